// ac_split.cpp -- the SPLIT STT tier: the hot part of a large automaton in
// shared memory, the cold part in L1/L2 (SURVEY 8(a)-a5 tier (ii), 8(f)
// NEXT-3 hot/cold two-level STT).
//
// The paper keeps the whole STT in texture memory and notes that its cache
// misses grow with the number of patterns.  On sm_100a
// a table read through L1TEX costs one tag lookup and one sector per lane,
// and for a 10,000-pattern byte dictionary (131K states x 256 columns x 4 B
// = 135 MB) the L1 -> L2 request path binds the scan (ncu: l1tex2xbar 81 %,
// 2.8 GB of DRAM reads per 1 GiB of text).  But a DFA walk over payload
// bytes spends almost all of its steps in a few shallow states (simulated
// on the C3 text: depth 1 = 60 %, depth 2 = 38 %, deeper 2 %), and in the AC
// automaton delta(s,c) = g(s,c) if the trie has that edge, else
// delta(f(s),c) (P:62 with the failure function of P:52).  So, in BFS order
// (states sorted by depth, the ids of the global dense table):
//
//   * ids [0, D)      DENSE rows in shared memory: C 16-bit entries each;
//   * ids [D, D + W)  8-byte RECORDS in shared memory: fd(s) = the first
//                     dense state on s's failure chain and two exceptions
//                     (c, delta(s,c)) -- the classes where delta(s,.)
//                     differs from delta(fd(s),.); states needing more are
//                     marked cold (fd = 0xFFFF);
//   * everything else COLD: the full dense 32-bit table in global memory,
//                     read through L1/L2.
//
// A shared-memory entry is 2 x + flag (x = BFS id of the next state, flag =
// output(x) != {}) when x < 32767, else 0xFFFF = "read this entry from the
// global table".  Records with fewer than two exceptions repeat a real one
// (or store delta(s, 0)) so no sentinel class is needed: every stored
// (c, t) pair is exactly delta(s, c).  Output enumeration always reads the
// global table's per-row output summary (matches are rare where this tier
// is chosen).
#include <algorithm>
#include <cstring>

#include "ac_internal.h"

namespace acx {

bool split_table(ac_table &t, size_t budget) {
    const uint32_t S = t.n_states, C = t.n_classes, stride = t.row_stride;
    if (t.entry_bytes != 4 || S == 0 || C > 256) return false;
    auto delta = [&](uint32_t s, uint32_t c) -> uint32_t {
        uint32_t e;
        std::memcpy(&e, &t.stt[((size_t)s * stride + c) * 4], 4);
        return e;
    };
    const uint32_t dstride = (C + 1) & ~1u;  // u16 entries per dense row (keeps records 4-byte aligned)
    const size_t row_bytes = (size_t)dstride * 2;
    uint32_t maxd = 0;
    for (uint32_t s = 0; s < S; s++) maxd = std::max(maxd, t.depth[s]);
    std::vector<uint32_t> level_end(maxd + 2, 0);  // BFS ids of depth <= d are [0, level_end[d])
    for (uint32_t s = 0; s < S; s++) level_end[t.depth[s]] = s + 1;
    for (uint32_t d = 1; d <= maxd; d++) level_end[d] = std::max(level_end[d], level_end[d - 1]);

    // fd(s) for a dense prefix [0, D): first state on the failure chain with id < D
    std::vector<uint32_t> fd(S, 0);
    auto exceptions = [&](uint32_t s, uint32_t f, uint32_t *cls, uint32_t cap) {
        uint32_t k = 0;
        for (uint32_t c = 0; c < C; c++)
            if ((delta(s, c) & 0x7fffffffu) != (delta(f, c) & 0x7fffffffu)) {
                if (k < cap) cls[k] = c;
                k++;
            }
        return k;
    };
    auto set_fd = [&](uint32_t D) {
        for (uint32_t s = 0; s < S; s++) fd[s] = s < D ? s : fd[t.fail[s]];
    };
    // Dense levels, shallowest first: a level is made dense while most of its
    // states would need more than two exceptions (shallow states have many
    // children) and the level fits; then records fill the rest of the budget.
    uint32_t D = 1;  // the root is always dense
    for (uint32_t d = 1; d <= maxd; d++) {
        const uint32_t lo = level_end[d - 1], hi = level_end[d];
        if ((size_t)hi * row_bytes > budget) break;
        set_fd(lo);
        uint32_t over = 0, tmp[3];
        for (uint32_t s = lo; s < hi; s++) over += exceptions(s, fd[s], tmp, 3) > 2;
        if (2 * over < hi - lo) break;  // mostly cheap as records
        D = hi;
    }
    if ((size_t)D * row_bytes > budget || D >= 0xFFFFu) return false;
    const size_t dense_bytes = (size_t)D * row_bytes;
    const uint32_t W = (uint32_t)std::min<size_t>(S - D, (budget - dense_bytes) / 8);
    set_fd(D);

    auto enc = [&](uint32_t e) -> uint16_t {  // 32-bit entry -> 2 x + flag, or the escape
        const uint32_t x = e & 0x7fffffffu;
        return x < 32767u ? (uint16_t)((x << 1) | (e >> 31)) : (uint16_t)0xFFFFu;
    };
    std::vector<uint8_t> blob(dense_bytes + (size_t)W * 8, 0);
    for (uint32_t s = 0; s < D; s++)
        for (uint32_t c = 0; c < C; c++) {
            const uint16_t e = enc(delta(s, c));
            std::memcpy(&blob[((size_t)s * dstride + c) * 2], &e, 2);
        }
    uint32_t n_cold = 0;
    for (uint32_t i = 0; i < W; i++) {
        const uint32_t s = D + i;
        uint32_t cls[2] = {0, 0};
        const uint32_t k = exceptions(s, fd[s], cls, 2);
        uint32_t lo, hi;
        if (k > 2) {  // cold record: the global table serves this state
            lo = 0xFFFFu;
            hi = 0;
            n_cold++;
        } else {
            if (k == 1) cls[1] = cls[0];
            // k == 0: (0, delta(s, 0)) twice -- equal to the dense fallback anyway
            lo = fd[s] | (cls[0] << 16) | (cls[1] << 24);
            hi = (uint32_t)enc(delta(s, cls[0])) | ((uint32_t)enc(delta(s, cls[1])) << 16);
        }
        std::memcpy(&blob[dense_bytes + (size_t)i * 8], &lo, 4);
        std::memcpy(&blob[dense_bytes + (size_t)i * 8 + 4], &hi, 4);
    }
    t.split.swap(blob);
    t.s_dense = D;
    t.s_rec = W;
    t.s_dstride = dstride;
    t.s_cold_rec = n_cold;
    return true;
}

}  // namespace acx
