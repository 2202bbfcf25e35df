// ac_build.cpp -- phase 1 on the host: dictionary -> dense STT.
//
// The paper builds "a 2-dimensional matrix (called State Transition Table:
// STT)" whose rows are DFA states and whose columns are the input symbols,
// plus a column M flagging matched states (Fig. 5), on a single CPU
// core.  The DFA's next-move function delta replaces both goto and
// failure functions.  What differs here:
//
//   * Alphabet compaction: the 256 byte columns collapse to C classes; class
//     0 = every byte that occurs in no pattern (its column is all-root), the
//     others are the bytes that occur, in byte order.
//   * Orientation: by default the automaton is built over the REVERSED
//     patterns and the scan walks right to left, so a state's output set is
//     the set of patterns STARTING at the current position and the matches
//     leave each chain already in canonical (start, pattern) order.  The
//     forward (paper) orientation is kept for builder tests.
//   * Column M is folded into each entry: the top bit of delta(s,c) says
//     "output(delta(s,c)) is non-empty" (reading R10), so the hot loop
//     learns about a match from the same load that moves it.
//   * BFS state numbering: shallow (hot) states form a prefix of the table,
//     which is what a shared-memory hot prefix keeps resident.
//   * Rows are padded to an odd number of 4-byte words (bank spreading).
//   * output(s) is stored as CSR with ids ascending (the closure over the
//     failure function).
//
// Construction is the textbook one (AC'75 Alg. 2-4) on a dense goto table;
// everything after the trie runs on host threads, one BFS level at a time
// (a faster build).
#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <new>
#include <thread>

#include "ac_internal.h"

namespace acx {

// Host threads for phase 1: ac_build_opts.threads, else $AC_BUILD_THREADS,
// else the hardware concurrency (capped at 32).
uint32_t build_threads(const ac_build_opts *opts) {
    uint32_t t = opts ? opts->threads : 0;
    if (t == 0) {
        const char *e = std::getenv("AC_BUILD_THREADS");
        if (e && *e) t = (uint32_t)std::strtoul(e, nullptr, 10);
    }
    if (t == 0) t = std::min(32u, std::max(1u, std::thread::hardware_concurrency()));
    return std::max(1u, std::min(t, 256u));
}

// fn(lo, hi) over [0, n) in T contiguous ranges; small ranges stay on the
// calling thread (a level of a few hundred states is not worth a spawn).
void parallel_for(size_t n, uint32_t T, const std::function<void(size_t, size_t)> &fn) {
    const size_t kMinPerThread = 2048;
    size_t k = std::min<size_t>(T, (n + kMinPerThread - 1) / kMinPerThread);
    if (k <= 1) {
        if (n) fn(0, n);
        return;
    }
    std::vector<std::thread> pool;
    pool.reserve(k - 1);
    for (size_t j = 1; j < k; j++) pool.emplace_back(fn, n * j / k, n * (j + 1) / k);
    fn(0, n / k);
    for (auto &th : pool) th.join();
}

ac_status compile_table(const uint8_t *const *patterns, const uint32_t *lens, uint32_t n,
                        const ac_build_opts *opts, ac_table &t) {
    if (n > 0 && (!patterns || !lens)) {
        set_error("patterns/lens is NULL");
        return AC_ERR_INVALID_ARG;
    }
    if (n >= AC_MAX_PATTERNS) {
        set_error("n_patterns must be < 2^24");
        return AC_ERR_TOO_LARGE;
    }
    uint32_t want_eb = opts ? opts->entry_bytes : 0;
    if (want_eb != 0 && want_eb != 2 && want_eb != 4) {
        set_error("entry_bytes must be 0, 2 or 4");
        return AC_ERR_INVALID_ARG;
    }
    t.forward = opts ? (opts->forward ? 1u : 0u) : 0u;
    t.n_patterns = n;
    t.lens.assign(lens, lens + n);
    uint64_t total = 0;
    t.maxlen = 0;
    bool used[256] = {false};
    for (uint32_t p = 0; p < n; p++) {
        if (lens[p] == 0) {
            set_error("pattern " + std::to_string(p) + " is empty");
            return AC_ERR_EMPTY_PATTERN;
        }
        if (!patterns[p]) {
            set_error("patterns[" + std::to_string(p) + "] is NULL");
            return AC_ERR_INVALID_ARG;
        }
        t.maxlen = std::max(t.maxlen, lens[p]);
        total += lens[p];
        for (uint32_t j = 0; j < lens[p]; j++) used[patterns[p][j]] = true;
    }
    if (total + 1 >= (1ull << 31)) {
        set_error("too many states");
        return AC_ERR_TOO_LARGE;
    }
    // ---- alphabet classes
    uint32_t C = 1;
    for (int b = 0; b < 256; b++) t.class_map[b] = 0;
    for (int b = 0; b < 256; b++)
        if (used[b]) t.class_map[b] = (uint8_t)std::min<uint32_t>(C++, 255);
    // C can reach 257 when every byte occurs; class ids then need 9 bits.
    // We keep class 0 only if some byte is unused: with all 256 bytes used the
    // map is the identity shifted by one, which would overflow uint8, so map
    // byte b -> b and drop the empty class.
    if (C == 257) {
        for (int b = 0; b < 256; b++) t.class_map[b] = (uint8_t)b;
        C = 256;
    }
    t.n_classes = C;

    const uint32_t T = build_threads(opts);
    try {
        // ---- goto function (AC'75 Alg. 2) on a dense table, creation order.
        // The trie is sequential (one pass over the patterns); every later
        // phase runs on T threads, level by level where a state depends on
        // shallower ones (NEXT-3 "faster build"; the table is identical for
        // any T).
        std::vector<int32_t> go;
        go.reserve((size_t)std::min<uint64_t>(total + 1, 1u << 22) * C);
        go.assign(C, -1);
        std::vector<uint32_t> end_state(n);
        uint32_t S = 1;
        for (uint32_t p = 0; p < n; p++) {
            uint32_t s = 0;
            for (uint32_t j = 0; j < lens[p]; j++) {
                uint8_t b = t.forward ? patterns[p][j] : patterns[p][lens[p] - 1 - j];
                uint32_t c = t.class_map[b];
                int32_t nx = go[(size_t)s * C + c];
                if (nx < 0) {
                    nx = (int32_t)S++;
                    go[(size_t)s * C + c] = nx;
                    go.insert(go.end(), C, -1);
                }
                s = (uint32_t)nx;
            }
            end_state[p] = s;
        }
        // own(s): the patterns ending in s, ids ascending (counting sort)
        std::vector<uint32_t> own_off(S + 1, 0), own_ids(n);
        for (uint32_t p = 0; p < n; p++) own_off[end_state[p] + 1]++;
        for (uint32_t s = 0; s < S; s++) own_off[s + 1] += own_off[s];
        {
            std::vector<uint32_t> fill(own_off.begin(), own_off.end() - 1);
            for (uint32_t p = 0; p < n; p++) own_ids[fill[end_state[p]]++] = p;
        }
        // ---- BFS order, failure function and delta (AC'75 Alg. 3/4), one
        // level at a time: a state's failure state is shallower, so its delta
        // row is final before the level that reads it.
        std::vector<uint32_t> order;
        order.reserve(S);
        std::vector<uint32_t> fail(S, 0), depth(S, 0), level_start;
        order.push_back(0);
        std::vector<uint32_t> nch;
        for (size_t lo = 0, hi = 1; lo < hi; lo = hi, hi = order.size()) {
            level_start.push_back((uint32_t)lo);
            const size_t L = hi - lo;
            nch.assign(L + 1, 0);
            parallel_for(L, T, [&](size_t a, size_t b) {
                for (size_t i = a; i < b; i++) {
                    const int32_t *row = &go[(size_t)order[lo + i] * C];
                    uint32_t k = 0;
                    for (uint32_t c = 0; c < C; c++) k += row[c] >= 0;
                    nch[i + 1] = k;
                }
            });
            for (size_t i = 0; i < L; i++) nch[i + 1] += nch[i];
            order.resize(hi + nch[L]);
            parallel_for(L, T, [&](size_t a, size_t b) {
                for (size_t i = a; i < b; i++) {
                    const uint32_t r = order[lo + i];
                    int32_t *row = &go[(size_t)r * C];
                    const int32_t *frow = &go[(size_t)fail[r] * C];
                    size_t w = hi + nch[i];
                    for (uint32_t c = 0; c < C; c++) {
                        const int32_t child = row[c];
                        if (child >= 0) {
                            order[w++] = (uint32_t)child;
                            depth[child] = depth[r] + 1;
                            fail[child] = (r == 0) ? 0u : (uint32_t)frow[c];
                        } else {
                            // delta(r,c) = delta(f(r),c); the root loops to itself
                            row[c] = (r == 0) ? 0 : frow[c];
                        }
                    }
                }
            });
        }
        level_start.push_back(S);
        // after this loop go[] holds delta (all entries >= 0)
        // ---- renumber in BFS order
        std::vector<uint32_t> rank(S);
        parallel_for(S, T, [&](size_t a, size_t b) {
            for (size_t i = a; i < b; i++) rank[order[i]] = (uint32_t)i;
        });
        t.fail.resize(S);
        t.depth.resize(S);
        parallel_for(S, T, [&](size_t a, size_t b) {
            for (size_t i = a; i < b; i++) {
                t.fail[i] = rank[fail[order[i]]];
                t.depth[i] = depth[order[i]];
            }
        });
        // ---- output closure output(s) = own(s) U output(f(s)),
        // as CSR in BFS numbering; |output(s)| and the fill go level by level
        std::vector<uint64_t> osz(S, 0);  // by BFS id
        for (size_t d = 0; d + 1 < level_start.size(); d++)
            parallel_for(level_start[d + 1] - level_start[d], T, [&](size_t a, size_t b) {
                for (size_t i = level_start[d] + a; i < level_start[d] + b; i++) {
                    const uint32_t s = order[i];
                    osz[i] = (own_off[s + 1] - own_off[s]) + (i ? osz[rank[fail[s]]] : 0);
                }
            });
        uint32_t eb = want_eb ? want_eb : (S <= 32768 ? 2u : 4u);
        if (eb == 2 && S > 32768) {
            set_error("entry_bytes=2 needs <= 32768 states");
            return AC_ERR_TOO_LARGE;
        }
        // Row = C transition entries, then the state's output summary (so a
        // flagged transition learns |output(next)| and, when it is 1, the
        // pattern id from the row it is about to walk anyway):
        //   eb=2: entries [P, P+1] = u32 payload (P = C rounded to even), [P+2] = u16 count
        //   eb=4: entry C = u32 payload, entry C+1 = u32 count
        // payload = the pattern id if count == 1, else the CSR offset.
        // The row is padded to an odd number of 4-byte words.
        uint32_t stride, info_col;
        if (eb == 2) {
            info_col = (C + 1) & ~1u;
            uint32_t words = (info_col + 3 + 1) / 2;
            if (words % 2 == 0) words++;
            stride = words * 2;
        } else {
            info_col = C;
            stride = (C + 2) | 1u;
        }
        t.n_states = S;
        t.row_stride = stride;
        t.info_col = info_col;
        t.entry_bytes = eb;
        t.out_off.assign(S + 1, 0);
        uint64_t n_out = 0;
        t.max_out = 0;
        for (uint32_t i = 0; i < S; i++) {
            t.out_off[i] = (uint32_t)n_out;
            n_out += osz[i];
            t.max_out = (uint32_t)std::max<uint64_t>(t.max_out, osz[i]);
            if (n_out >= (1ull << 32)) {
                set_error("output closure too large");
                return AC_ERR_TOO_LARGE;
            }
        }
        t.out_off[S] = (uint32_t)n_out;
        t.out_ids.resize(n_out);
        for (size_t d = 0; d + 1 < level_start.size(); d++)
            parallel_for(level_start[d + 1] - level_start[d], T, [&](size_t a, size_t b) {
                for (size_t i = level_start[d] + a; i < level_start[d] + b; i++) {
                    const uint32_t s = order[i];
                    uint32_t *dst = t.out_ids.data() + t.out_off[i];
                    if (i == 0) {
                        std::copy(own_ids.begin() + own_off[s], own_ids.begin() + own_off[s + 1], dst);
                    } else {
                        const uint32_t f = rank[fail[s]];  // shallower: already filled
                        std::merge(own_ids.begin() + own_off[s], own_ids.begin() + own_off[s + 1],
                                   t.out_ids.begin() + t.out_off[f], t.out_ids.begin() + t.out_off[f + 1], dst);
                    }
                }
            });
        // ---- the table: entry = BFS id of delta(s,c) | flag (output non-empty)
        std::vector<uint32_t> code(S);  // by creation id
        parallel_for(S, T, [&](size_t a, size_t b) {
            for (size_t s = a; s < b; s++)
                code[s] = rank[s] | (osz[rank[s]] ? (eb == 2 ? 0x8000u : 0x80000000u) : 0u);
        });
        t.stt.assign((size_t)S * stride * eb, 0);
        parallel_for(S, T, [&](size_t a, size_t b) {
            for (size_t i = a; i < b; i++) {
                const int32_t *row = &go[(size_t)order[i] * C];
                const uint64_t cnt = osz[i];
                const uint32_t payload = cnt == 1 ? t.out_ids[t.out_off[i]] : t.out_off[i];
                uint8_t *r = &t.stt[(size_t)i * stride * eb];
                std::memcpy(r + (size_t)info_col * eb, &payload, 4);
                if (eb == 2) {
                    uint16_t c16 = (uint16_t)std::min<uint64_t>(cnt, 0xFFFF);
                    std::memcpy(r + (size_t)(info_col + 2) * 2, &c16, 2);
                    uint16_t *e = reinterpret_cast<uint16_t *>(r);
                    for (uint32_t c = 0; c < C; c++) e[c] = (uint16_t)code[(uint32_t)row[c]];
                } else {
                    uint32_t c32 = (uint32_t)cnt;
                    std::memcpy(r + (size_t)(info_col + 1) * 4, &c32, 4);
                    uint32_t *e = reinterpret_cast<uint32_t *>(r);
                    for (uint32_t c = 0; c < C; c++) e[c] = code[(uint32_t)row[c]];
                }
            }
        });
    } catch (const std::bad_alloc &) {
        set_error("host allocation failed while building the STT");
        return AC_ERR_NO_MEMORY;
    }
    return AC_OK;
}

}  // namespace acx
