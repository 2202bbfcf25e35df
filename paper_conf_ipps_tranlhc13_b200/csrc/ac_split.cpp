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
// (states sorted by depth, the ids of the global dense table), the HOT
// states [0, H) are served from shared memory by one rule:
//
//   record(s) = fd(s) | c1 << 16 | c2 << 24,  t1 | t2 << 16
//   delta(s, c) = t1 if c == c1, t2 if c == c2, else row[fd(s)][c]
//
// where row[] are dense 16-bit rows, also in shared memory:
//   * the shallow levels [0, D) are DENSE: no record is stored; the kernel
//     uses (fd = s, no exception class), i.e. reads the state's own row;
//   * the next states [D, H) are SPARSE: fd(s) = the first dense state on s's
//     failure chain, (c1, t1), (c2, t2) = the (at most two) classes where
//     delta(s,.) differs from delta(fd(s),.) -- repeated, or (0, delta(s, 0)),
//     when there are fewer, so every stored pair is exactly delta(s, c);
//   * a sparse state needing more exceptions is COLD: its record points at
//     row[D], the ESCAPE row (all 0xFFFF), with t1 = t2 = 0xFFFF;
//   * states >= H are COLD: the kernel does not read a record for them.
// A 16-bit entry is 2 x + flag (x = BFS id of the next state, flag =
// output(x) != {}) when x < 32767, else 0xFFFF; 0xFFFF (cold state, cold
// record, large id) sends the lane to the full 32-bit dense table in global
// memory (L1/L2; the paper's STT).  Output enumeration always reads
// that table's per-row output summary (matches are rare where this tier is
// chosen).
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
    const size_t dense_bytes = (size_t)(D + 1) * row_bytes;  // + the escape row
    if (dense_bytes > budget) return false;
    const uint32_t H = D + (uint32_t)std::min<size_t>(S - D, (budget - dense_bytes) / 8);
    set_fd(D);

    auto enc = [&](uint32_t e) -> uint16_t {  // 32-bit entry -> 2 x + flag, or the escape
        const uint32_t x = e & 0x7fffffffu;
        return x < 32767u ? (uint16_t)((x << 1) | (e >> 31)) : (uint16_t)0xFFFFu;
    };
    std::vector<uint8_t> blob(dense_bytes + (size_t)(H - D) * 8, 0);
    for (uint32_t s = 0; s < D; s++)
        for (uint32_t c = 0; c < C; c++) {
            const uint16_t e = enc(delta(s, c));
            std::memcpy(&blob[((size_t)s * dstride + c) * 2], &e, 2);
        }
    for (uint32_t c = 0; c < dstride; c++) {  // the escape row
        const uint16_t e = 0xFFFFu;
        std::memcpy(&blob[((size_t)D * dstride + c) * 2], &e, 2);
    }
    uint32_t n_cold = 0;
    for (uint32_t s = D; s < H; s++) {  // records of the sparse hot states
        uint32_t cls[2] = {0, 0}, lo, hi;
        {
            const uint32_t k = exceptions(s, fd[s], cls, 2);
            if (k > 2) {  // cold record: every class escapes to the global table
                lo = D;
                hi = 0xFFFFFFFFu;
                n_cold++;
            } else {
                if (k == 1) cls[1] = cls[0];
                // k == 0: (0, delta(s, 0)) twice -- equal to the dense fallback anyway
                lo = fd[s] | (cls[0] << 16) | (cls[1] << 24);
                hi = (uint32_t)enc(delta(s, cls[0])) | ((uint32_t)enc(delta(s, cls[1])) << 16);
            }
        }
        std::memcpy(&blob[dense_bytes + (size_t)(s - D) * 8], &lo, 4);
        std::memcpy(&blob[dense_bytes + (size_t)(s - D) * 8 + 4], &hi, 4);
    }
    t.split.swap(blob);
    t.s_dense = D;
    t.s_rec = H;
    t.s_dstride = dstride;
    t.s_cold_rec = n_cold;
    return true;
}

}  // namespace acx
