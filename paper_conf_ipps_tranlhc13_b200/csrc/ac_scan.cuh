// ac_scan.cuh -- launch interface between the ABI layer and the scan kernels.
#pragma once

#include <cstdint>

#include <cuda.h>
#include <cuda_runtime.h>

#include "ac.h"

namespace acx {

// COUNT_TOTAL: count only (atomic total).  COUNT_CHAINS: per-chain counts.
// EMIT: write records at known chain end offsets (second pass).
// EMIT_OPT: one pass -- per-chain counts AND the chain's first q records
// written into its scratch slot; k_gather moves them to their final place.
enum ScanMode { MODE_COUNT_TOTAL = 0, MODE_COUNT_CHAINS = 1, MODE_EMIT = 2, MODE_EMIT_OPT = 3 };

// Read-only automaton as the kernels see it.
struct SttView {
    const void *stt;          // entries, row-major, row_stride entries per row
    const uint8_t *cmap;      // byte -> class (256 B)
    const uint32_t *out_off;  // output CSR offsets [S + 1]
    const uint32_t *out_ids;  // output CSR ids (ascending per state)
    uint32_t stride;          // entries per row
    uint32_t n_states;
    uint32_t smem_rows;       // rows staged into shared memory
    uint32_t halo;            // maxlen - 1
    uint32_t info_col;        // entry index of the row's output summary (payload u32, count)
    uint32_t smem_bytes;      // STT bytes staged into shared memory
    // COMPACT tier (ac_compact.cpp): the dense/sparse split and byte offsets
    // inside the blob, pre-biased so that each address is one multiply-add
    // of the compact id x: dense row x at x * c_row_bytes, sparse record x at
    // c_sparse_x0 + 8 x, output slot of output state x at c_out_x0 + 8 x
    // (both x0 wrap around modulo 2^32 on purpose)
    uint32_t c_dense, c_row_bytes, c_sparse_x0, c_out_x0;
    // run-time constants of the COMPACT walk (see compact_next): 8, 2, -2,
    // 2^31, 2^16, 0x0101 -- multiplied, never shifted, to load the FMA pipe
    uint32_t c_rec_bytes, c_two, c_mtwo, c_half, c_k16, c_rep;
    // two-byte table (NEXT-4): row s, column c1 * n_classes + c2; NULL = off
    const uint32_t *stt2;
    uint32_t stride2, n_classes;
    // SPLIT tier (ac_split.cpp): shared-memory part staged from `sblob` --
    // dense rows r <= s_dense at r * s_row_bytes (row s_dense = the escape
    // row), the 8-byte records of the sparse hot ids [s_dense, s_rec) at
    // s_rec_x0 + 8 s (biased by -8 s_dense, wraps);
    // `stt` stays the full 32-bit table for the cold states
    const void *sblob;
    uint32_t s_dense, s_rec, s_row_bytes, s_rec_x0;
    uint32_t cmap_ident;  // the class map is the identity (every byte occurs in a pattern)
    // GLOBAL tier, staged kernel: `sblob` holds min(|output(s)|, 255) per state,
    // staged into shared memory -- a flagged lane reads its output count there
    // instead of from the table row in L1/L2 (255 = read the row)
    uint32_t cnt8;
};

// A run of equal-length chains over owned starts [lo, hi) of the shard.
struct Region {
    uint64_t lo, hi;       // owned byte range (shard coordinates)
    uint64_t chain_len;    // bytes owned per chain (last chain may be shorter)
    uint64_t n_chains;
    uint64_t chain0;       // global index of the region's first chain
};

// Where results go.
struct ScanOut {
    unsigned long long *total;      // MODE_COUNT_TOTAL: atomic sum
    uint64_t *chain_counts;         // MODE_COUNT_CHAINS
    const uint64_t *chain_end;      // MODE_EMIT: inclusive prefix (end offset) per chain
    const ac_result *res;           // MODE_EMIT: skip writing when res->status != AC_OK
    uint64_t *out;                  // MODE_EMIT: records
    uint64_t base;                  // global position of shard byte 0
    uint64_t *scratch;              // MODE_EMIT_OPT: q slots per chain
    uint32_t q;
    // MODE_EMIT_OPT, staged kernel's deferred emission only: > 0 = narrow
    // 4-byte scratch records (offset in chain << nbits | pattern), packed at
    // the end of the chain's 8q-byte slot; 0 = 8-byte final keys
    uint32_t nbits;
    // MODE_EMIT_OPT, staged kernel, when the main region starts the list
    // (NULL = off): each CTA publishes its match total in tile_state
    // [its ticket] (decoupled look-back) and writes the end offset of each of
    // its chains into chain_end_w -- the offset scan runs inside the scan
    unsigned long long *tile_state;
    uint64_t *chain_end_w;
    // with tile_state: zeroed counter from which each staged CTA takes its
    // tile index (an atomic ticket), so every look-back predecessor of a
    // running CTA is itself running or done -- CUDA does not promise that
    // CTAs start in blockIdx order
    unsigned int *ticket;
    // MODE_EMIT_OPT EVENTS (dense outputs, 32-bit tables, S < 2^24; NULL =
    // off): the scan parks one 8-byte event (start << 24 | state) per output
    // state reached instead of its records -- the slot holds a whole chain's
    // events (q >= chain length) -- counts the records for the offsets as
    // usual and writes the chain's event count here; k_gather expands the
    // events into records, warp-cooperatively and coalesced
    uint32_t *chain_events;
};

// What k_gather needs to expand events: the dense table's per-row output
// summary (32-bit entries: payload at entry info_col, count at info_col + 1;
// 16-bit entries: u32 payload at entries [info_col, info_col + 1], u16 count
// at info_col + 2, 0xFFFF = read the CSR offsets) and the CSR.
struct EventExpand {
    const uint32_t *events;   // per-chain event counts (NULL = record mode)
    const void *stt;
    uint32_t stride, info_col, entry_bytes;
    const uint32_t *out_off, *out_ids;
};

// Decoupled look-back words: 2-bit flag (aggregate / inclusive prefix) + value.
static constexpr uint64_t LB_AGG = 1ull << 62, LB_INC = 2ull << 62, LB_VAL = (1ull << 62) - 1;

// Where k_gather finds chain offsets when the staged kernel computed them:
// main chains from chain_end; the (few) tail chains behind the main total,
// which is the last staged CTA's inclusive look-back word.
// Main-region chains whose scratch records are narrow (k_gather widens them).
struct NarrowMain {
    uint32_t nbits;       // 0 = every chain is wide
    uint64_t c0, n;       // global ids of the main chains
    uint64_t lo0;         // global position of main chain 0's first byte (base + m0)
    uint64_t chain_len;   // L
};

struct TailPlace {
    const unsigned long long *tile_state;  // NULL: chain_end holds every chain (k_offsets ran)
    uint64_t n_tiles;                      // staged CTAs
    uint64_t tail_c0, tail_n;              // tail chains (global ids), tail_n <= 256
    uint64_t cap;
};

// Geometry of the TMA-staged main region.
struct StagedGeom {
    uint64_t m0;           // shard offset of the main region (16-byte aligned address)
    uint64_t chain_len;    // L, multiple of the tile width
    uint64_t n_chains;     // full chains in the main region
    uint64_t chain0;       // global index of main chain 0
    uint64_t n_readable;   // bytes readable from the main-region pointer (halo bound)
    uint32_t text_evict_first;  // L2 policy of the text's TMA loads: 0 normal, 1 evict-first, 2 per-sector pair
};

struct StagedConfig {
    int warps;       // warps per CTA (each owns 32*k chains and a private ring)
    int k;           // chains per lane
    int width;       // tile width W in bytes (16 / 32 / 64 = TMA swizzle span)
    int stages;      // ring slots per warp
    int swizzle;     // 1 = TMA swizzle (conflict-free lane reads), 0 = plain rows (NEXT-1 ablation)
};

// AC_STAGED_VARIANTS(X): X(index, warps, chains per lane, tile width, ring depth, swizzle)
#define AC_STAGED_VARIANTS(X) \
    X(1, 16, 1, 32, 3, 1)     \
    X(2, 16, 2, 32, 2, 1)     \
    X(3, 32, 1, 32, 2, 1)     \
    X(4, 32, 1, 16, 3, 1)     \
    X(5, 16, 2, 16, 3, 1)     \
    X(6, 32, 2, 16, 2, 1)     \
    X(7, 32, 1, 16, 2, 1)     \
    X(8, 32, 1, 32, 2, 0)     \
    X(9, 16, 2, 16, 2, 1)     \
    X(10, 32, 1, 32, 1, 1)    \
    X(11, 32, 1, 32, 1, 0)

// Kernel entry points (host side launchers); all return cudaError_t.
cudaError_t launch_scan_global(int mode, uint32_t entry_bytes, uint32_t tier, const uint8_t *text,
                               uint64_t n_total, const SttView &st, const Region &a, const Region &b,
                               const ScanOut &so, size_t smem_bytes, cudaStream_t stream);
cudaError_t launch_scan_staged(int mode, uint32_t entry_bytes, uint32_t tier, int variant, const CUtensorMap &tmap,
                               const uint8_t *main_text, const SttView &st, const StagedGeom &g, const ScanOut &so,
                               size_t smem_stt_bytes, cudaStream_t stream);
cudaError_t launch_offsets(const uint64_t *counts, uint64_t n, uint64_t *chain_end, uint64_t *tile_state,
                           unsigned int *tile_counter, ac_result *res, uint64_t cap, int emitting,
                           cudaStream_t stream);

size_t staged_smem_bytes(const StagedConfig &cfg, size_t smem_stt_bytes);

// Single-pass list mode helpers: k_gather copies every chain's scratch slot
// to its final position (or lists the chain when it overflowed); k_rewalk
// re-scans the listed chains in MODE_EMIT.
cudaError_t launch_gather(const uint64_t *counts, uint64_t *chain_end, uint64_t n_chains,
                          const uint64_t *scratch, uint32_t q, uint64_t *out, ac_result *res,
                          uint64_t *list, unsigned int *list_n, const TailPlace &tp, const NarrowMain &nm,
                          const EventExpand &ev, int num_sms, cudaStream_t stream);
cudaError_t launch_rewalk(uint32_t entry_bytes, uint32_t tier, const uint8_t *text, uint64_t n_total,
                          const SttView &st, const Region &a, const Region &b, const StagedGeom &g,
                          const ScanOut &so, const uint64_t *list, const unsigned int *list_n, size_t smem_stt,
                          int num_sms, cudaStream_t stream);

// per-tier instantiations (ac_tier_*.cu)
template <int TIER>
cudaError_t launch_global_tier(int mode, uint32_t eb, const uint8_t *text, uint64_t n_total, const SttView &st,
                               const Region &a, const Region &b, const ScanOut &so, size_t smem_stt,
                               cudaStream_t stream);
template <int TIER>
cudaError_t launch_staged_tier(int mode, uint32_t eb, int variant, const CUtensorMap &tmap, const uint8_t *mtext,
                               const SttView &st, const StagedGeom &g, const ScanOut &so, size_t smem_stt,
                               cudaStream_t stream);
template <int TIER>
cudaError_t launch_segments_tier(int mode, uint32_t eb, const uint8_t *text, const uint64_t *seg_off, uint64_t n_seg,
                                 const SttView &st, const ScanOut &so, size_t smem_stt, cudaStream_t stream);
cudaError_t launch_segments(int mode, uint32_t eb, uint32_t tier, const uint8_t *text, const uint64_t *seg_off,
                            uint64_t n_seg, const SttView &st, const ScanOut &so, size_t smem_stt, cudaStream_t stream);
template <int TIER>
cudaError_t launch_rewalk_tier(uint32_t eb, const uint8_t *text, uint64_t n_total, const SttView &st,
                               const Region &a, const Region &b, const StagedGeom &g, const ScanOut &so,
                               const uint64_t *list, const unsigned int *list_n, size_t smem_stt, int num_sms,
                               cudaStream_t stream);
int staged_variant_count();
const StagedConfig &staged_variant(int v);  // v in [1, staged_variant_count()]
size_t offsets_tiles(uint64_t n);

}  // namespace acx
