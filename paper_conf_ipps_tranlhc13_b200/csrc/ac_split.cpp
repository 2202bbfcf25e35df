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
//   * the shallow levels [0, D) are DENSE: 16-bit rows in shared memory
//     (the levels whose states mostly have more than four children);
//   * the next level [D, H) gets an 8-byte CHILDREN record per state:
//       lo = c1 | c2 << 8 | c3 << 16 | c4 << 24   (children's classes, ascending)
//       hi = fd | flags << 12 | (2 first - 1) << 16
//     delta(s, c) = first + k if c == c_k (k = 0..3: BFS numbers a state's
//     children consecutively in class order), else row[fd][c] -- fd = f(s),
//     which is dense, so the exceptions of s against fd are exactly its
//     goto children; flags bit k = output(first + k) != {}.  Fewer than four
//     children repeat the last class; a state with more (or ids that do not
//     fit) is COLD: fd = D (the ESCAPE row, all 0xFFFF) and 2 first - 1 =
//     0xFFFD, so any result escapes.  (first is stored doubled minus one: the
//     scan adds the match position p = 8 k + 7 as p >> 2 = 2 k + 1 and gets
//     2 (first + k) -- the 16-bit entry form -- in one instruction; first >= 1
//     because a child is never the root);
//   * states >= H are COLD.
// A 16-bit result is 2 x + flag (x = BFS id, flag = output(x) != {}) for
// x < 32767, and > 0xFFFD means "read the 32-bit dense table in global
// memory (L1/L2; the paper's STT)".  Output enumeration always reads
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
    // states have more than four children and the level fits; the next
    // level gets children records.
    auto children = [&](uint32_t s, uint32_t *cls, uint32_t *tgt, uint32_t cap) {
        uint32_t k = 0;
        for (uint32_t c = 0; c < C; c++) {
            const uint32_t x = delta(s, c) & 0x7fffffffu;
            if (t.depth[x] == t.depth[s] + 1) {  // a goto edge
                if (k < cap) cls[k] = c, tgt[k] = delta(s, c);
                k++;
            }
        }
        return k;
    };
    uint32_t D = 1, d0 = 0;  // the root is always dense
    for (uint32_t d = 1; d <= maxd; d++) {
        const uint32_t lo = level_end[d - 1], hi = level_end[d];
        if ((size_t)(hi + 1) * row_bytes > budget) break;
        uint32_t over = 0, tc[5], tt[5];
        for (uint32_t s = lo; s < hi; s++) over += children(s, tc, tt, 5) > 4;
        if (2 * over < hi - lo) break;  // mostly cheap as records
        D = hi;
        d0 = d;
    }
    if (D >= 4095u) return false;  // fd and the escape row index are 12-bit
    const size_t dense_bytes = (size_t)(D + 1) * row_bytes;  // + the escape row
    if (dense_bytes > budget) return false;
    const uint32_t H = std::min<uint32_t>(level_end[d0 + 1 <= maxd ? d0 + 1 : maxd],
                                          D + (uint32_t)std::min<size_t>(S - D, (budget - dense_bytes) / 8));
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
    for (uint32_t s = D; s < H; s++) {  // children records of the next level
        uint32_t cls[4] = {0, 0, 0, 0}, tgt[4] = {0, 0, 0, 0}, ex[1];
        const uint32_t k = children(s, cls, tgt, 4);
        bool ok = k <= 4 && fd[s] == t.fail[s] && exceptions(s, fd[s], ex, 0) == k;
        for (uint32_t i = 0; ok && i < k; i++) ok = (tgt[i] & 0x7fffffffu) == (tgt[0] & 0x7fffffffu) + i;
        ok = ok && (k == 0 || (tgt[0] & 0x7fffffffu) + k - 1 < 32767u);
        uint32_t lo, hi;
        const uint32_t kCold = D | (0xFFFDu << 16);  // cold: every result escapes
        if (!ok) {
            lo = 0;
            hi = kCold;
            n_cold++;
        } else if (k == 0) {
            // a leaf: every class falls back to row[fd]; the record names one
            // class c* (all four bytes) whose "child" is delta(s, c*) itself
            // -- a class whose target is not the root (first >= 1)
            uint32_t cs = C;
            for (uint32_t c = 0; c < C && cs == C; c++) {
                const uint32_t x = delta(s, c) & 0x7fffffffu;
                if (x >= 1 && x < 32767u) cs = c;
            }
            if (cs == C) {
                lo = 0;
                hi = kCold;
                n_cold++;
            } else {
                const uint32_t e = delta(s, cs);
                lo = cs * 0x01010101u;
                hi = fd[s] | ((e >> 31) << 12) | ((2 * (e & 0x7fffffffu) - 1) << 16);
            }
        } else {
            for (uint32_t i = k; i < 4; i++) cls[i] = cls[k - 1];  // repeats never win (lowest byte first)
            uint32_t flags = 0;
            for (uint32_t i = 0; i < k; i++) flags |= (tgt[i] >> 31) << i;
            lo = cls[0] | (cls[1] << 8) | (cls[2] << 16) | (cls[3] << 24);
            hi = fd[s] | (flags << 12) | ((2 * (tgt[0] & 0x7fffffffu) - 1) << 16);
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
