// ac_internal.h -- internal types of libac (not part of the ABI).
#pragma once

#include <cstdint>
#include <functional>
#include <string>
#include <vector>

#include "ac.h"

// Phase-1 result on the host (P:118 STT, P:137 built once on the host).
struct ac_table {
    uint32_t n_patterns = 0;
    uint32_t maxlen = 0;
    uint32_t n_states = 0;
    uint32_t n_classes = 0;
    uint32_t row_stride = 0;   // entries per row
    uint32_t info_col = 0;     // entry index of the output summary (payload u32, count)
    uint32_t max_out = 0;      // max |output(s)|: bounds matches per byte (32-bit chain counters)
    uint32_t entry_bytes = 2;
    uint32_t forward = 0;
    uint8_t class_map[256] = {0};
    std::vector<uint8_t> stt;          // n_states * row_stride * entry_bytes
    std::vector<uint32_t> out_off;     // n_states + 1
    std::vector<uint32_t> out_ids;     // output CSR (ids ascending per state)
    std::vector<uint32_t> lens;        // pattern lengths
    std::vector<uint32_t> fail;        // failure function, BFS ids
    std::vector<uint32_t> depth;       // state depth (trie level)

    // COMPACT encoding, built by compact_table():
    //   [dense rows: c_dense x c_dstride u16][sparse records: (S - c_dense) x 8 B][output table: n_out x 8 B]
    // in its own numbering: 0 = root, then the other dense states,
    // [c_dense - c_od, c_dense) = dense output states, [c_dense, c_dense +
    // c_os) = sparse output states, then the other sparse states.
    uint32_t c_dense = 0, c_od = 0, c_os = 0, c_dstride = 0;
    uint32_t c_sparse_off = 0, c_out_off = 0;  // byte offsets inside `compact`
    std::vector<uint8_t> compact;
    std::vector<uint32_t> c_perm;              // compact id -> BFS id

    // SPLIT tier (ac_split.cpp): dense rows for BFS ids [0, s_dense) (s_dstride
    // u16 entries each), then s_rec 8-byte records for ids [s_dense, s_dense +
    // s_rec); every other state is read from the global 32-bit table
    uint32_t s_dense = 0, s_rec = 0, s_dstride = 0, s_cold_rec = 0;
    std::vector<uint8_t> split;

    // two-byte table (NEXT-4), built by stride2_table(): row s, column
    // c1 * n_classes + c2 -> delta(delta(s,c1),c2) | final flag << 31 |
    // middle flag << 30; rows padded to an odd number of words
    uint32_t stride2 = 0;
    std::vector<uint32_t> stt2;
};

// Device-side STT (library owned).
struct ac_stt {
    ac_table host;        // keeps the host copy for query / re-upload
    int device = 0;
    uint32_t tier = AC_TIER_GLOBAL;
    uint32_t hot_rows = 0;
    void *d_stt = nullptr;           // entries
    uint32_t *d_stt2 = nullptr;      // two-byte table (NEXT-4) or NULL
    void *d_split = nullptr;         // SPLIT tier: the shared-memory part (dense rows + records)
    uint8_t *d_class_map = nullptr;  // 256 B
    uint8_t *d_cnt8 = nullptr;       // GLOBAL tier, 32-bit table: min(|output(s)|, 255) per state (staged)
    uint32_t *d_out_off = nullptr;
    uint32_t *d_out_ids = nullptr;
    uint32_t *d_lens = nullptr;
    int num_sms = 148;
    size_t smem_optin = 227 * 1024;
};

namespace acx {
void set_error(const std::string &msg);
uint32_t build_threads(const ac_build_opts *opts);
void parallel_for(size_t n, uint32_t T, const std::function<void(size_t, size_t)> &fn);
ac_status compile_table(const uint8_t *const *patterns, const uint32_t *lens, uint32_t n,
                        const ac_build_opts *opts, ac_table &t);
bool compact_table(ac_table &t, size_t budget);
bool stride2_table(ac_table &t, size_t max_bytes);
bool split_table(ac_table &t, size_t budget);
}  // namespace acx
