// ac_compact.cpp -- the COMPACT STT encoding.
//
// The paper keeps the whole STT in texture memory and notes that its cache
// misses grow with the number of patterns.  On sm_100a the
// fast tier is shared memory, but a dense AC table for ~1,000 English
// patterns (15K states x 31 classes x 2 B) is ~1 MB.  Most of those rows are
// near-copies: in the AC automaton delta(s,c) = g(s,c) if the trie has that
// edge, else delta(f(s),c) (P:62 with the failure function of P:52), and a
// deep trie state almost always has a single child.  So:
//
//   * DENSE states (the BFS prefix up to depth d, plus any state that needs
//     more than two exceptions) keep a full row of C entries.
//   * Every other (SPARSE) state s gets an 8-byte record: fd(s) = the first
//     dense state on its failure chain, and up to two exceptions (c, delta(s,c))
//     -- exactly the classes where delta(s,.) differs from delta(fd(s),.).
//     delta(s,c) = exception if c matches one, else dense[fd(s)][c]: at most
//     two shared-memory loads per byte, no loop.
//   * Output states are numbered last among the dense and first among the
//     sparse states, so their ids are contiguous and the output table index
//     is one subtraction: oidx = x - (c_dense - c_od); each table slot holds
//     (payload, count) exactly like the dense rows' output summary.
//
// Entries are 2 x + flag: x = the next state's compact id, flag =
// output(next) != {} (COMPACT requires <= 32768 states and C <= 127).
// The device class map of a COMPACT automaton holds 2 x class: the byte
// offset of the class's column inside a dense row, compared directly with
// the records' (doubled) exception classes.
#include <algorithm>
#include <cstring>

#include "ac_internal.h"

namespace acx {

// Size of the COMPACT encoding whose dense set is the depth-<= d prefix, the
// states marked in `seed` (may be NULL), and every state that would need more
// than two exceptions.
size_t compact_bytes_for(const ac_table &t, uint32_t d, const std::vector<uint8_t> *seed,
                         std::vector<uint8_t> *dense_out, uint32_t *n_dense) {
    const uint32_t S = t.n_states, C = t.n_classes, stride = t.row_stride;
    auto delta = [&](uint32_t s, uint32_t c) -> uint32_t {
        uint16_t e;
        std::memcpy(&e, &t.stt[((size_t)s * stride + c) * 2], 2);
        return e & 0x7fffu;
    };
    std::vector<uint8_t> dense(S, 0);
    std::vector<uint32_t> fd(S, 0);
    uint32_t nd = 0;
    for (uint32_t s = 0; s < S; s++) {  // BFS order: f(s) is decided before s
        if (s == 0 || t.depth[s] <= d || (seed && (*seed)[s])) {
            dense[s] = 1;
        } else {
            const uint32_t f = t.fail[s];
            fd[s] = dense[f] ? f : fd[f];
            uint32_t exc = 0;
            for (uint32_t c = 0; c < C && exc <= 2; c++) exc += delta(s, c) != delta(fd[s], c);
            if (exc > 2) dense[s] = 1;
        }
        nd += dense[s];
    }
    uint32_t words = (C + 1) / 2;
    if (words % 2 == 0) words++;
    uint32_t n_out = 0;
    for (uint32_t s = 0; s < S; s++) n_out += t.out_off[s + 1] > t.out_off[s];
    if (dense_out) dense_out->swap(dense);
    if (n_dense) *n_dense = nd;
    const size_t dense_bytes = (size_t)nd * words * 4;
    return (dense_bytes + 7) / 8 * 8 + (size_t)(S - nd) * 8 + (size_t)n_out * 8;
}

// Build the COMPACT encoding into t.compact if it fits `budget` bytes.
// Returns false (t unchanged) when the automaton cannot be compacted.
bool compact_table(ac_table &t, size_t budget) {
    const uint32_t S = t.n_states, C = t.n_classes, stride = t.row_stride;
    if (t.entry_bytes != 2 || S > 32768 || C > 127 || S == 0) return false;
    uint32_t maxd = 0;
    for (uint32_t s = 0; s < S; s++) maxd = std::max(maxd, t.depth[s]);
    // the deepest dense prefix that fits (the size is not monotonic in d:
    // shallow prefixes force many states with > 2 exceptions to be dense)
    // Dense set = the depth-<= d prefix + the first k of the deeper states
    // ordered by how many patterns they prefix (most first): a state that
    // prefixes many patterns is a common string (the patterns are words of
    // the text), so it is visited often, and making it dense also lets
    // its descendants' records fall back on it (fewer exceptions, fewer
    // exception-forced dense states -- the size is not monotonic in d or k).
    // Take the deepest prefix that fits and fill the rest of the budget; if
    // no prefix fits, the (d, k) with the most dense states that does.
    // Measured on the C2 text (simulated walk): sparse visits 48 % -> 34 %.
    std::vector<uint32_t> parent(S, 0), below(S, 0);
    for (uint32_t s = 0; s < S; s++)
        for (uint32_t c = 0; c < C; c++) {
            uint16_t e;
            std::memcpy(&e, &t.stt[((size_t)s * stride + c) * 2], 2);
            const uint32_t u = e & 0x7fffu;
            if (u && t.depth[u] == t.depth[s] + 1) parent[u] = s;  // the goto edge (unique)
        }
    for (uint32_t s = 1; s < S; s++)  // patterns ending exactly at s
        for (uint32_t j = t.out_off[s]; j < t.out_off[s + 1]; j++) below[s] += t.lens[t.out_ids[j]] == t.depth[s];
    for (uint32_t s = S - 1; s > 0; s--) below[parent[s]] += below[s];  // BFS order: children after parents
    std::vector<uint8_t> seed(S, 0);
    std::vector<uint32_t> cand;
    auto candidates = [&](uint32_t d) {
        cand.clear();
        for (uint32_t s = 1; s < S; s++)
            if (t.depth[s] > d) cand.push_back(s);
        std::stable_sort(cand.begin(), cand.end(), [&](uint32_t a, uint32_t b) {
            return below[a] != below[b] ? below[a] > below[b] : t.depth[a] < t.depth[b];
        });
    };
    uint32_t nd_try = 0;
    auto fits = [&](uint32_t d, size_t k) {
        std::fill(seed.begin(), seed.end(), 0);
        for (size_t i = 0; i < k; i++) seed[cand[i]] = 1;
        return compact_bytes_for(t, d, &seed, nullptr, &nd_try) <= budget;
    };
    // the largest fitting k, given that k = lo fits (bisection; near-monotone)
    auto widest = [&](uint32_t d, size_t lo) {
        size_t hi = cand.size();
        while (lo < hi) {
            const size_t mid = (lo + hi + 1) / 2;
            if (fits(d, mid)) lo = mid; else hi = mid - 1;
        }
        return lo;
    };
    int best = -1;
    for (uint32_t d = 0; d <= maxd; d++)
        if (compact_bytes_for(t, d, nullptr, nullptr, nullptr) <= budget) best = (int)d;
    size_t best_k = 0;
    if (best >= 0) {
        candidates((uint32_t)best);
        best_k = widest((uint32_t)best, 0);
    } else {
        uint32_t best_nd = 0;
        for (uint32_t d = 0; d <= std::min<uint32_t>(maxd, 6); d++) {
            candidates(d);
            size_t k0 = SIZE_MAX;  // the first fitting k on a doubling grid
            for (size_t k = 1; k <= cand.size(); k = k * 2) {
                if (fits(d, k)) { k0 = k; break; }
                if (k * 2 > cand.size() && k != cand.size() && fits(d, cand.size())) { k0 = cand.size(); break; }
            }
            if (k0 == SIZE_MAX) continue;
            const size_t k = widest(d, k0);
            fits(d, k);
            if (nd_try > best_nd) best_nd = nd_try, best = (int)d, best_k = k;
        }
        if (best < 0) return false;
        candidates((uint32_t)best);
    }
    fits((uint32_t)best, best_k);
    std::vector<uint8_t> dense;
    uint32_t nd = 0;
    const size_t total = compact_bytes_for(t, (uint32_t)best, &seed, &dense, &nd);
    auto delta_e = [&](uint32_t s, uint32_t c) -> uint16_t {
        uint16_t e;
        std::memcpy(&e, &t.stt[((size_t)s * stride + c) * 2], 2);
        return e;
    };
    auto is_out = [&](uint32_t s) { return t.out_off[s + 1] > t.out_off[s]; };
    // numbering: root, other dense, dense outputs, sparse outputs, other
    // sparse -- the output states form ONE contiguous id range
    // [c_dense - c_od, c_dense + c_os), so oidx = x - (c_dense - c_od)
    std::vector<uint32_t> perm;  // compact id -> BFS id
    perm.reserve(S);
    perm.push_back(0);
    uint32_t od = 0, os = 0;
    for (uint32_t s = 1; s < S; s++)
        if (dense[s] && !is_out(s)) perm.push_back(s);
    for (uint32_t s = 1; s < S; s++)
        if (dense[s] && is_out(s)) perm.push_back(s), od++;
    for (uint32_t s = 1; s < S; s++)
        if (!dense[s] && is_out(s)) perm.push_back(s), os++;
    for (uint32_t s = 1; s < S; s++)
        if (!dense[s] && !is_out(s)) perm.push_back(s);
    std::vector<uint32_t> inv(S);
    for (uint32_t x = 0; x < S; x++) inv[perm[x]] = x;
    // COMPACT entry = 2 x + flag (x = compact id of the next state)
    auto enc = [&](uint16_t e) -> uint16_t { return (uint16_t)((inv[e & 0x7fffu] << 1) | (e >> 15)); };

    uint32_t words = (C + 1) / 2;
    if (words % 2 == 0) words++;
    const uint32_t dstride = words * 2;
    const size_t dense_bytes = ((size_t)nd * dstride * 2 + 7) / 8 * 8;
    std::vector<uint8_t> blob(total, 0);
    for (uint32_t x = 0; x < nd; x++) {
        const uint32_t s = perm[x];
        for (uint32_t c = 0; c < C; c++) {
            const uint16_t e = enc(delta_e(s, c));
            std::memcpy(&blob[((size_t)x * dstride + c) * 2], &e, 2);
        }
    }
    // sparse records: lo = 2 c1 | 2 c2 << 8 | fd << 16, hi = t1 | t2 << 16
    // (classes doubled, as in the COMPACT class map: a doubled class is the
    // byte offset of its column in a dense row; 0xFF = no exception; fd is a
    // plain compact id, t1 and t2 are entries)
    std::vector<uint32_t> fd(S, 0);
    for (uint32_t s = 1; s < S; s++)
        if (!dense[s]) fd[s] = dense[t.fail[s]] ? t.fail[s] : fd[t.fail[s]];
    for (uint32_t x = nd; x < S; x++) {
        const uint32_t s = perm[x];
        uint32_t cls[2] = {0xFF, 0xFF};
        uint16_t tgt[2] = {0, 0};
        uint32_t k = 0;
        for (uint32_t c = 0; c < C; c++) {
            const uint16_t e = delta_e(s, c);
            if ((e & 0x7fffu) != (delta_e(fd[s], c) & 0x7fffu)) {
                cls[k] = 2 * c;
                tgt[k] = enc(e);
                k++;
            }
        }
        const uint32_t lo = cls[0] | (cls[1] << 8) | (inv[fd[s]] << 16);
        const uint32_t hi = (uint32_t)tgt[0] | ((uint32_t)tgt[1] << 16);
        uint8_t *r = &blob[dense_bytes + (size_t)(x - nd) * 8];
        std::memcpy(r, &lo, 4);
        std::memcpy(r + 4, &hi, 4);
    }
    // output table
    const size_t out_base = dense_bytes + (size_t)(S - nd) * 8;
    auto put_out = [&](uint32_t oidx, uint32_t s) {
        const uint32_t a = t.out_off[s], z = t.out_off[s + 1];
        const uint32_t payload = (z - a == 1) ? t.out_ids[a] : a, count = z - a;
        std::memcpy(&blob[out_base + (size_t)oidx * 8], &payload, 4);
        std::memcpy(&blob[out_base + (size_t)oidx * 8 + 4], &count, 4);
    };
    for (uint32_t i = 0; i < od + os; i++) put_out(i, perm[nd - od + i]);

    t.compact.swap(blob);
    t.c_perm.swap(perm);
    t.c_dense = nd;
    t.c_od = od;
    t.c_os = os;
    t.c_dstride = dstride;
    t.c_sparse_off = (uint32_t)dense_bytes;
    t.c_out_off = (uint32_t)out_base;
    return true;
}

// NEXT-4: the two-byte next-move table, T2(s, c1 c2) =
// delta(delta(s, c1), c2), so a small-alphabet scan does one dependent gather
// per TWO bytes (the paper's O(n) walk, with half the steps).  Bit 31
// flags output(final) != {}, bit 30 flags output(middle) != {} (the kernel
// recovers the middle state from the one-byte table in that rare case).
// Built from the dense one-byte table; requires 32-bit entries.
bool stride2_table(ac_table &t, size_t max_bytes) {
    const uint32_t S = t.n_states, C = t.n_classes, stride = t.row_stride;
    if (t.entry_bytes != 4 || S == 0 || S >= (1u << 30)) return false;
    const uint64_t cols = (uint64_t)C * C;
    const uint32_t stride2 = (uint32_t)(cols | 1u);
    if ((uint64_t)S * stride2 * 4 > max_bytes || (uint64_t)S * stride2 >= (1ull << 32)) return false;
    auto delta = [&](uint32_t s, uint32_t c) -> uint32_t {
        uint32_t e;
        std::memcpy(&e, &t.stt[((size_t)s * stride + c) * 4], 4);
        return e;
    };
    std::vector<uint32_t> tab((size_t)S * stride2, 0);
    for (uint32_t s = 0; s < S; s++) {
        uint32_t *row = &tab[(size_t)s * stride2];
        for (uint32_t c1 = 0; c1 < C; c1++) {
            const uint32_t e1 = delta(s, c1);
            const uint32_t mid = e1 & 0x7fffffffu;
            for (uint32_t c2 = 0; c2 < C; c2++) {
                const uint32_t e2 = delta(mid, c2);
                row[c1 * C + c2] = (e2 & 0x7fffffffu) | ((e2 >> 31) << 31) | ((e1 >> 31) << 30);
            }
        }
    }
    t.stt2.swap(tab);
    t.stride2 = stride2;
    return true;
}

}  // namespace acx
