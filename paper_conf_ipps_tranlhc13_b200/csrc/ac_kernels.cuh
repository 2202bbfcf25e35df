// ac_kernels.cuh -- device code of the Aho-Corasick scan for sm_100a
// (templates; instantiated once per STT tier in ac_tier_*.cu).
//
// The hot loop is the DFA walk of P:60-70: one dependent STT gather per text
// byte (state <- delta(state, text[i]), O(n) transitions), with the
// output function consulted when the entry's match flag (the paper's column
// M) is set.  Text decomposition follows the paper's chunking: each
// thread walks its own chunk, extended by the longest pattern so straddling
// matches are found, with ownership by START position so every
// occurrence is reported once (reading R9).  Because the automaton is built
// over reversed patterns, every chain walks right to left: the (maxlen - 1)
// halo to the right of the chunk is consumed first as a warm-up (no output)
// and the chunk's matches then come out in descending (start, pattern) order,
// which the emitter writes backwards from the chain's end offset -- the list
// is canonical without any sort.
//
// Kernels:
//   k_scan_staged  the paper's "shared memory approach" rebuilt
//                  for sm_100a.  Each WARP owns 32*K chains of L bytes and a
//                  private ring of NST shared-memory slots; one lane streams
//                  the warp's text with 2-D TMA boxes (W bytes x 32*K chains,
//                  plus one box of the next chains' first bytes for the
//                  halo), each slot guarded by its own mbarrier.  Warps never
//                  wait for each other (the only CTA barrier is after the STT
//                  is staged), so the irregular gather latency of one warp
//                  does not stall the SM.  The TMA swizzle (32B/64B) is the
//                  hardware form of the paper's diagonal, bank-conflict-free
//                  store: lane l reads its chain 16 B at a time
//                  with conflict-free LDS.128.
//   k_scan_global  the paper's "global memory only approach":
//                  each thread reads its chain straight from global memory
//                  (16-byte vector loads, L1-cached).  Also covers the
//                  unaligned head and the ragged tail of the staged path.
//
// STT tiers: SMEM (whole table staged once per CTA),
// HYBRID (BFS-prefix rows in shared memory, the rest through L1/L2 with a
// generic load), GLOBAL (L1/L2 only), COMPACT (dense rows + default-transition
// records, all in shared memory), SPLIT (COMPACT-like hot part in shared
// memory, the cold states through L1/L2).
#pragma once

#include <type_traits>

#include "ac_scan.cuh"

namespace acx {

#ifdef AC_DEBUG_TIMES
// debug builds (AC_EXTRA_NVCC_FLAGS=-DAC_DEBUG_TIMES): per-warp walk times of
// the staged scan (one copy per translation unit; ac_tier_split.cu exports
// ac_debug_times() for its own)
static __device__ unsigned long long ac_dbg_times[1024 * 32 * 2];
#endif

static constexpr int GT = 256;  // k_scan_global block size
// SPLIT list mode: flag-mask walk + re-walk of flagged lanes (default) or the
// emission inline at each flagged byte (-DAC_SPLIT_INLINE_EMIT, ablation)
#ifdef AC_SPLIT_INLINE_EMIT
static constexpr bool kSplitInlineEmit = true;
#else
static constexpr bool kSplitInlineEmit = false;
#endif

template <typename E>
struct EntryBits;
template <>
struct EntryBits<uint16_t> {
    static constexpr uint32_t FLAG = 0x8000u, MASK = 0x7fffu;
};
template <>
struct EntryBits<uint32_t> {
    static constexpr uint32_t FLAG = 0x80000000u, MASK = 0x7fffffffu;
};

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

// ------------------------------------------------------------------ tables
template <typename E>
__device__ __forceinline__ void stage_tables(uint8_t *s_cmap, E *s_stt, const SttView &st) {
    const uint4 *c4 = reinterpret_cast<const uint4 *>(st.cmap);
    uint4 *d4 = reinterpret_cast<uint4 *>(s_cmap);
    for (int i = threadIdx.x; i < 16; i += blockDim.x) d4[i] = __ldg(c4 + i);
    const size_t words = ((size_t)st.smem_bytes + 15) / 16;
    // SPLIT stages its own blob (hot rows + records); the others a prefix of the table
    const uint4 *src = reinterpret_cast<const uint4 *>(st.sblob ? st.sblob : st.stt);
    uint4 *dst = reinterpret_cast<uint4 *>(s_stt);
    for (size_t i = threadIdx.x; i < words; i += blockDim.x) dst[i] = __ldg(src + i);
}

template <typename E, int TIER>
__device__ __forceinline__ uint32_t stt_load(const E *s_stt, const E *g_stt, uint32_t hot, uint32_t s,
                                             uint32_t idx) {
    if constexpr (TIER == AC_TIER_SMEM) {
        return s_stt[idx];
    } else if constexpr (TIER == AC_TIER_GLOBAL || TIER == AC_TIER_SPLIT) {
        return __ldg(g_stt + idx);  // (SPLIT: the output summaries live in the global table)
    } else {
        // HYBRID: two predicated loads, one per address space.  (A generic
        // load would send the shared-memory lanes through the L1TEX tag
        // stage too -- the stage that binds this tier, ncu: 97 % busy.)
        const uint32_t in_smem = s < hot;
        const uint32_t sa = smem_u32(s_stt + idx);
        const uint64_t ga = reinterpret_cast<uint64_t>(g_stt + idx);
        uint32_t v = 0;
        if constexpr (sizeof(E) == 2)
            asm("{\n\t.reg .pred p;\n\tsetp.ne.u32 p, %1, 0;\n\t@p ld.shared.u16 %0, [%2];\n\t"
                "@!p ld.global.nc.u16 %0, [%3];\n\t}"
                : "+r"(v)
                : "r"(in_smem), "r"(sa), "l"(ga));
        else
            asm("{\n\t.reg .pred p;\n\tsetp.ne.u32 p, %1, 0;\n\t@p ld.shared.u32 %0, [%2];\n\t"
                "@!p ld.global.nc.u32 %0, [%3];\n\t}"
                : "+r"(v)
                : "r"(in_smem), "r"(sa), "l"(ga));
        return v;
    }
}

// The entry delta(s, cls).  Dense tiers: next state in the low bits, output
// flag on top.  COMPACT: e = 2 x + flag (x = next state, compact id).
// COMPACT: a dense row, or a sparse record's exception, or the dense row of
// the record's default state fd(s) -- at most two shared-memory loads, issued
// as predicated loads so lanes in dense and sparse states never diverge.
// (Each predicated load's destination register is pre-loaded with a value
// that is dead afterwards -- its own address -- so no zeroing moves are
// needed; write-only "=r" outputs made ptxas spill 372 B per thread.)
// The COMPACT walk is bound by the ALU pipe (ncu: 86-89 % busy, FMA pipe
// 14 %), so its shifts, masks and field extractions are written as
// multiply-adds and multiply-highs by RUN-TIME constants (SttView c_*), which
// the compiler can neither strength-reduce back to shifts nor fold: they
// issue on the otherwise idle FMA pipe.
__device__ __forceinline__ uint32_t compact_next(uint32_t base, const SttView &st, uint32_t s, uint32_t cls2) {
    // cls2 = 2 x class (the COMPACT class map is pre-doubled): the byte
    // offset of column cls inside a dense row, and the form in which the
    // sparse records store their exception classes
    const uint32_t sp = s >= st.c_dense;
    uint32_t hi = cls2 + s * st.c_row_bytes;                   // dense entry (s, cls) (garbage if sparse)
    uint32_t lo = s * st.c_rec_bytes + (base + st.c_sparse_x0);  // sparse record of s (garbage if dense)
    asm("{\n\t.reg .pred p;\n\t.reg .u32 a;\n\tsetp.ne.u32 p, %2, 0;\n\t"
        "add.u32 a, %1, %3;\n\t"
        "@p ld.shared.v2.u32 {%0, %1}, [%0];\n\t"
        "@!p ld.shared.u16 %0, [a];\n\t}"
        : "+r"(lo), "+r"(hi)
        : "r"(sp), "r"(base));
    // sparse: lo = c1 | c2 << 8 | fd << 16 (exception classes doubled), hi = t1 | t2 << 16
    const uint32_t rep = cls2 * st.c_rep;                      // cls2 in bytes 0 and 1
    const uint32_t h1 = ((lo ^ rep) & 0xFFu) == 0, h2 = ((lo ^ rep) & 0xFF00u) == 0;
    const uint32_t need = sp & (1u ^ (h1 | h2));                // sparse and no exception hit
    uint32_t e3 = cls2 + __umulhi(lo, st.c_k16) * st.c_row_bytes;  // dense entry (fd, cls)
    asm("{\n\t.reg .pred p;\n\t.reg .u32 a;\n\tsetp.ne.u32 p, %1, 0;\n\tadd.u32 a, %0, %2;\n\t@p ld.shared.u16 %0, [a];\n\t}"
        : "+r"(e3)
        : "r"(need), "r"(base));
    const uint32_t ex = __byte_perm(hi, 0, h1 ? 0x4410 : 0x4432);
    return sp ? (need ? e3 : ex) : lo;
}

// SPLIT tier (ac_split.cpp): delta(s, cls) as a 32-bit entry (BFS id | flag
// << 31).  A hot state of the record level (s_dense <= s < s_rec) loads its
// children record {c1..c4 | fd, first, flags}: delta = first + k if cls ==
// c_k, else row[fd][cls]; a dense state reads row[s][cls]; a cold state
// (s >= s_rec) reads the escape row.  Every lane runs the same instructions
// (the class bytes of a non-record lane are cls ^ 0x80, which never match).
// A 16-bit result above 0xFFFD -- cold state, cold record or a next id >=
// 32767 -- is replaced by the full entry from the global table (L1/L2).
// IDENT: identity class map, so C = 256 and the 32-bit table's row stride is
// the compile-time (256 + 2) | 1 = 259 (one constant-bank load less per step).
static constexpr uint32_t kIdentStride = 259;
template <bool IDENT = false>
__device__ __forceinline__ uint32_t split_next(uint32_t base, const SttView &st, uint32_t s, uint32_t cls) {
    const uint32_t rep = cls * 0x01010101u;
    const uint32_t sparse = (s - st.s_dense) < (st.s_rec - st.s_dense);
    uint32_t lo = base + st.s_rec_x0 + s * 8u;  // record address (biased by -8 s_dense)
    uint32_t hi = min(s, st.s_dense);           // fd of a dense state (itself) or of a cold one (escape row)
    asm("{\n\t.reg .pred p;\n\tsetp.ne.u32 p, %2, 0;\n\t@p ld.shared.v2.u32 {%0, %1}, [%0];\n\t"
        "@!p xor.b32 %0, %3, 0x80808080;\n\t}"
        : "+r"(lo), "+r"(hi)
        : "r"(sparse), "r"(rep));
    // lo = c1 | c2 << 8 | c3 << 16 | c4 << 24, hi = fd | flags << 12 | (2 first - 1) << 16
    const uint32_t x = lo ^ rep;                                  // a zero byte where a class matches
    const uint32_t z = (x - 0x01010101u) & ~x & 0x80808080u;      // lowest set bit: the first match
    const uint32_t p = __ffs(z) - 1u;                              // 8 k + 7 (garbage if no match)
    // 2 (first + k) = (2 first - 1) + (p >> 2), then child k's output flag
    const uint32_t child = ((hi >> 16) + (p >> 2)) | ((hi >> (12u + (p >> 3))) & 1u);
    // e16 = child if a class matched, else the shared row entry row[fd][cls]:
    // one predicate for the load and the select
    uint32_t e16 = base + (hi & 0xFFFu) * st.s_row_bytes + cls * 2u;
    asm("{\n\t.reg .pred p;\n\tsetp.eq.u32 p, %1, 0;\n\t@p ld.shared.u16 %0, [%0];\n\t@!p mov.b32 %0, %2;\n\t}"
        : "+r"(e16)
        : "r"(z), "r"(child));
    uint32_t g = (e16 >> 1) | (e16 << 31);  // 2 x + flag -> x | flag << 31
    // (a warp-uniform skip of this block -- a vote over the active lanes --
    // was measured slower than the predicated form: C3 count 0.48 -> 0.51 ms,
    // list 0.63 -> 0.69 ms per 256 MiB)
    if (e16 > 0xFFFDu) {
        // cold: the full entry from the dense table through L1/L2.  (Measured
        // slower: a 16-byte L2-resident cold record per state answering three
        // exceptions over the shared-memory rows first -- the extra dependent
        // load doubled the long-scoreboard stalls, C3 list 3.2 -> 5.4 ms/GiB;
        // an L2 evict-last hint on this load: no change.)
        // (S x row_stride < 2^32 entries, checked by ac_build: a 32-bit index)
        const uint32_t *gp = static_cast<const uint32_t *>(st.stt) + (s * (IDENT ? kIdentStride : st.stride) + cls);
        asm volatile("ld.global.nc.u32 %0, [%1];" : "=r"(g) : "l"(gp));
    }
    return g;
}

// Class of a text byte (a4): the 256-byte class map in shared
// memory; SPLIT automata whose map is the identity (every byte occurs in a
// pattern, e.g. C3) skip the load -- one shared-memory wavefront group less
// per byte.
template <int TIER>
__device__ __forceinline__ uint32_t class_of(const uint8_t *s_cmap, uint32_t byte, const SttView &st) {
    if constexpr (TIER == AC_TIER_SPLIT) {
        uint32_t c = byte;
        asm("{\n\t.reg .pred p;\n\tsetp.eq.u32 p, %1, 0;\n\t@p ld.shared.u8 %0, [%2];\n\t}"
            : "+r"(c)
            : "r"(st.cmap_ident), "r"(smem_u32(s_cmap) + byte));
        return c;
    } else {
        return s_cmap[byte];
    }
}

// The same with the identity known at compile time (the SPLIT auto variant
// is also instantiated for identity class maps, e.g. C3: no predicated load).
template <int TIER, bool IDENT>
__device__ __forceinline__ uint32_t class_of_k(const uint8_t *s_cmap, uint32_t byte, const SttView &st) {
    if constexpr (IDENT)
        return byte;
    else
        return class_of<TIER>(s_cmap, byte, st);
}

// Entry -> next state and output flag.
template <typename E, int TIER>
__device__ __forceinline__ uint32_t state_of(uint32_t e, const SttView &st) {
    if constexpr (TIER == AC_TIER_COMPACT)
        return __umulhi(e, st.c_half);  // e >> 1 on the FMA pipe
    else
        return e & EntryBits<E>::MASK;
}
template <typename E, int TIER>
__device__ __forceinline__ uint32_t flag_of(uint32_t e, uint32_t x, const SttView &st) {
    if constexpr (TIER == AC_TIER_COMPACT)
        return e + x * st.c_mtwo;  // e - 2 x (IMAD)
    else
        return e >> (8 * sizeof(E) - 1);
}

template <typename E, int TIER, bool IDENT = false>
__device__ __forceinline__ uint32_t next_entry(const E *s_stt, const SttView &st, uint32_t s, uint32_t cls) {
    if constexpr (TIER == AC_TIER_COMPACT) {
        return compact_next(smem_u32(s_stt), st, s, cls);
    } else if constexpr (TIER == AC_TIER_SPLIT) {
        return split_next<IDENT>(smem_u32(s_stt), st, s, cls);
    } else {
        return stt_load<E, TIER>(s_stt, static_cast<const E *>(st.stt), st.smem_rows, s, s * st.stride + cls);
    }
}

// One transition with no output (halo warm-up).
template <typename E, int TIER>
__device__ __forceinline__ uint32_t ac_move(uint32_t s, uint32_t byte, const uint8_t *s_cmap, const E *s_stt,
                                            const SttView &st) {
    return state_of<E, TIER>(next_entry<E, TIER>(s_stt, st, s, class_of<TIER>(s_cmap, byte, st)), st);
}

// COMPACT output table slot of output state s: (payload, count).
template <typename E>
__device__ __forceinline__ uint2 compact_out(const E *s_stt, const SttView &st, uint32_t s) {
    return *reinterpret_cast<const uint2 *>(reinterpret_cast<const uint8_t *>(s_stt) + (st.c_out_x0 + (s << 3)));
}

// Output summary of state s, stored in the padding of its own STT row
// (builder: payload u32 at info_col, then the count), read through the same
// residency tier as the transitions -- no dependent global CSR loads for the
// common single-output case.
template <typename E, int TIER>
__device__ __forceinline__ uint32_t out_count(const E *s_stt, const SttView &st, uint32_t s) {
    if constexpr (TIER == AC_TIER_COMPACT) {
        return compact_out<E>(s_stt, st, s).y;
    } else {
        if constexpr (TIER == AC_TIER_GLOBAL) {
            if (st.cnt8) {  // staged counts (GLOBAL tier, staged kernel)
                const uint32_t c8 = reinterpret_cast<const uint8_t *>(s_stt)[s];
                if (c8 != 255u) return c8;
            }
        }
        const uint32_t idx = s * st.stride + st.info_col + (sizeof(E) == 2 ? 2 : 1);
        uint32_t c = stt_load<E, TIER>(s_stt, static_cast<const E *>(st.stt), st.smem_rows, s, idx);
        if (sizeof(E) == 2 && c == 0xFFFFu) c = __ldg(st.out_off + s + 1) - __ldg(st.out_off + s);
        return c;
    }
}

template <typename E, int TIER>
__device__ __forceinline__ uint32_t out_payload(const E *s_stt, const SttView &st, uint32_t s) {
    if constexpr (TIER == AC_TIER_COMPACT) {
        return compact_out<E>(s_stt, st, s).x;
    } else {
        const uint32_t idx = s * st.stride + st.info_col;  // 4-byte aligned by construction
        const uint32_t *sp = reinterpret_cast<const uint32_t *>(s_stt + idx);
        const uint32_t *gp = reinterpret_cast<const uint32_t *>(static_cast<const E *>(st.stt) + idx);
        if constexpr (TIER == AC_TIER_SMEM) {
            return *sp;
        } else if constexpr (TIER == AC_TIER_GLOBAL || TIER == AC_TIER_SPLIT) {
            return __ldg(gp);
        } else {
            return *((s < st.smem_rows) ? sp : gp);
        }
    }
}

// (payload, count) of output state s through its tier; a saturated 16-bit
// count falls back to the CSR offsets.
template <typename E, int TIER>
__device__ __forceinline__ uint2 compact_or_row_out(const E *s_stt, const SttView &st, uint32_t s) {
    if constexpr (TIER == AC_TIER_COMPACT) {
        return compact_out<E>(s_stt, st, s);
    } else {
        return make_uint2(out_payload<E, TIER>(s_stt, st, s), out_count<E, TIER>(s_stt, st, s));
    }
}

// (payload, count) of state s if f != 0, else (0, 0) -- predicated loads
// through the state's residency tier, so lanes never branch on a match.
template <typename E, int TIER, bool PAYLOAD>
__device__ __forceinline__ uint2 out_info_pred(const E *s_stt, const SttView &st, uint32_t s, uint32_t f) {
    uint32_t pay = 0, c = 0;
    if constexpr (TIER == AC_TIER_COMPACT) {
        const uint32_t a = smem_u32(s_stt) + st.c_out_x0 + (s << 3);
        asm("{\n\t.reg .pred p;\n\tsetp.ne.u32 p, %3, 0;\n\t@p ld.shared.v2.u32 {%0, %1}, [%2];\n\t}"
            : "+r"(pay), "+r"(c)
            : "r"(a), "r"(f));
    } else {
        const uint32_t ip = s * st.stride + st.info_col;            // payload (u32, 4-byte aligned)
        const uint32_t ic = ip + (sizeof(E) == 2 ? 2 : 1);           // count (E)
        if constexpr (TIER == AC_TIER_SMEM) {
            const uint32_t b = smem_u32(s_stt);
            if constexpr (sizeof(E) == 2)
                asm("{\n\t.reg .pred p;\n\tsetp.ne.u32 p, %2, 0;\n\t@p ld.shared.u16 %0, [%1];\n\t}"
                    : "+r"(c)
                    : "r"(b + ic * 2), "r"(f));
            else
                asm("{\n\t.reg .pred p;\n\tsetp.ne.u32 p, %2, 0;\n\t@p ld.shared.u32 %0, [%1];\n\t}"
                    : "+r"(c)
                    : "r"(b + ic * 4), "r"(f));
            if constexpr (PAYLOAD)
                asm("{\n\t.reg .pred p;\n\tsetp.ne.u32 p, %2, 0;\n\t@p ld.shared.u32 %0, [%1];\n\t}"
                    : "+r"(pay)
                    : "r"(b + ip * (uint32_t)sizeof(E)), "r"(f));
        } else {
            // GLOBAL: read-only global path; HYBRID: generic address (smem prefix or global)
            const E *g = static_cast<const E *>(st.stt);
            const E *base = (TIER == AC_TIER_HYBRID && s < st.smem_rows) ? s_stt : g;
            const uint64_t pc = reinterpret_cast<uint64_t>(base + ic), pp = reinterpret_cast<uint64_t>(base + ip);
            if constexpr (TIER == AC_TIER_GLOBAL || TIER == AC_TIER_SPLIT) {
                if constexpr (sizeof(E) == 2)
                    asm("{\n\t.reg .pred p;\n\tsetp.ne.u32 p, %2, 0;\n\t@p ld.global.nc.u16 %0, [%1];\n\t}"
                        : "+r"(c)
                        : "l"(pc), "r"(f));
                else
                    asm("{\n\t.reg .pred p;\n\tsetp.ne.u32 p, %2, 0;\n\t@p ld.global.nc.u32 %0, [%1];\n\t}"
                        : "+r"(c)
                        : "l"(pc), "r"(f));
                if constexpr (PAYLOAD)
                    asm("{\n\t.reg .pred p;\n\tsetp.ne.u32 p, %2, 0;\n\t@p ld.global.nc.u32 %0, [%1];\n\t}"
                        : "+r"(pay)
                        : "l"(pp), "r"(f));
            } else {
                if constexpr (sizeof(E) == 2)
                    asm("{\n\t.reg .pred p;\n\tsetp.ne.u32 p, %2, 0;\n\t@p ld.u16 %0, [%1];\n\t}"
                        : "+r"(c)
                        : "l"(pc), "r"(f));
                else
                    asm("{\n\t.reg .pred p;\n\tsetp.ne.u32 p, %2, 0;\n\t@p ld.u32 %0, [%1];\n\t}"
                        : "+r"(c)
                        : "l"(pc), "r"(f));
                if constexpr (PAYLOAD)
                    asm("{\n\t.reg .pred p;\n\tsetp.ne.u32 p, %2, 0;\n\t@p ld.u32 %0, [%1];\n\t}"
                        : "+r"(pay)
                        : "l"(pp), "r"(f));
            }
        }
    }
    return make_uint2(pay, c);
}

// Count or emit every pattern of output(x) at key0 (the branchy path).
template <typename E, int TIER, int MODE>
__device__ __forceinline__ void emit_outputs(uint32_t x, uint64_t key0, uint32_t &cnt, uint64_t &wp, const E *s_stt,
                                             const SttView &st, const ScanOut &so) {
    const uint32_t c = out_count<E, TIER>(s_stt, st, x);
    if constexpr (MODE == MODE_EMIT) {
        const uint32_t p = out_payload<E, TIER>(s_stt, st, x);
        if (c == 1) {
            so.out[--wp] = key0 | p;
        } else {
            for (uint32_t j = p + c; j > p; --j) so.out[--wp] = key0 | __ldg(st.out_ids + j - 1);
        }
    } else if constexpr (MODE == MODE_EMIT_OPT) {
        if (so.chain_events) {
            // EVENTS (dense outputs): one entry per output state reached, the
            // slot pointer moves down (a slot holds a whole chain's events)
            // Events are written with an L2 evict-first policy: 0.6 GB of them
            // per 256 MiB of English text otherwise pushed the 32-bit table
            // out of L2 (ncu: 2.2 GB of DRAM reads per launch instead of 0.6;
            // the same time -- the walk is bound by L1, not DRAM).  An
            // evict-last hint changed nothing; gathering four events per lane
            // in shared memory for one 32-byte store was no faster either
            // (English 5K 2.75 -> 2.83 ms, 20K 5.70 -> 5.45 ms).
            uint64_t pol;
            asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
            asm volatile("st.global.L2::cache_hint.u64 [%0], %1, %2;" ::"l"(wp), "l"(key0 | x), "l"(pol) : "memory");
            wp -= 8;
            cnt += c;
            return;
        }
        uint64_t *last = reinterpret_cast<uint64_t *>(wp);
        const uint32_t p = out_payload<E, TIER>(s_stt, st, x);
        if (c == 1) {
            if (cnt < so.q) last[-(int64_t)cnt] = key0 | p;
            cnt++;
        } else {
            for (uint32_t j = p + c; j > p; --j) {
                if (cnt < so.q) last[-(int64_t)cnt] = key0 | __ldg(st.out_ids + j - 1);
                cnt++;
            }
        }
    } else {
        cnt += c;
    }
}

// Predicated 8-byte global store to base[k] (k signed; one IMAD.WIDE for
// the address, no branch around the store).
__device__ __forceinline__ void st_global_if(const uint64_t *base, int32_t k, uint64_t v, bool pred) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t.reg .u64 a;\n\tsetp.ne.u32 p, %3, 0;\n\t"
        "mad.wide.s32 a, %1, 8, %0;\n\t@p st.global.u64 [a], %2;\n\t}" ::"l"(base),
        "r"(k), "l"(v), "r"((uint32_t)pred)
        : "memory");
}

// Predicated 4-byte global store to base[k] (narrow scratch records).
__device__ __forceinline__ void st_global32_if(const uint32_t *base, int32_t k, uint32_t v, bool pred) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t.reg .u64 a;\n\tsetp.ne.u32 p, %3, 0;\n\t"
        "mad.wide.s32 a, %1, 4, %0;\n\t@p st.global.u32 [a], %2;\n\t}" ::"l"(base),
        "r"(k), "r"(v), "r"((uint32_t)pred)
        : "memory");
}

// One transition inside the owned chunk: count or emit output(s) at the
// byte whose record key is key0 = (global start) << 24.  cnt is the chain's
// running count (32-bit: the planner keeps chain_len x max|output| < 2^31).
// wp: MODE_EMIT -> the chain's next output index (counts down);
//     MODE_EMIT_OPT -> the address of the LAST slot of the chain's scratch
//     slot (record k goes to wp - 8k).
template <typename E, int TIER, int MODE>
__device__ __forceinline__ void ac_step(uint32_t &s, uint32_t &cnt, uint64_t &wp, uint32_t byte, uint64_t key0,
                                        bool live, const uint8_t *s_cmap, const E *s_stt, const SttView &st,
                                        const ScanOut &so) {
    const uint32_t e = next_entry<E, TIER>(s_stt, st, s, class_of<TIER>(s_cmap, byte, st));
    s = state_of<E, TIER>(e, st);
    const uint32_t flag = flag_of<E, TIER>(e, s, st);
    // Predication pays where matches are dense (C2-like dictionaries, which are
    // what land in COMPACT); with rare flags (C1/C3/C4) the predicated loads
    // and store cost issue slots on every byte (measured: C1 list 2.6x slower),
    // so the dense tiers keep the branch.
    constexpr bool kPred = TIER == AC_TIER_COMPACT && MODE != MODE_EMIT;
    if constexpr (kPred) {
        // Branch-free for the common cases: predicated loads of the output
        // summary and a predicated store of a single-output match; only
        // multi-output states (and saturated counts) take a branch.
        const uint32_t f = flag & (live ? 1u : 0u);
        const uint2 o = out_info_pred<E, TIER, MODE == MODE_EMIT_OPT>(s_stt, st, s, f);
        uint32_t c = o.y;
        if (TIER != AC_TIER_COMPACT && sizeof(E) == 2 && c == 0xFFFFu)
            c = __ldg(st.out_off + s + 1) - __ldg(st.out_off + s);
        if constexpr (MODE == MODE_EMIT_OPT) {
            uint64_t *last = reinterpret_cast<uint64_t *>(wp);
            const uint32_t one = (c == 1u) & (cnt < so.q ? 1u : 0u);
            asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.u32 p, %2, 0;\n\t@p st.global.u64 [%0], %1;\n\t}" ::"l"(
                             last - cnt),
                         "l"(key0 | o.x), "r"(one)
                         : "memory");
            if (c > 1u) {
                for (uint32_t j = o.x + c; j > o.x; --j) {
                    if (cnt < so.q) last[-(int64_t)cnt] = key0 | __ldg(st.out_ids + j - 1);
                    cnt++;
                }
            } else {
                cnt += c;
            }
        } else {
            cnt += c;
        }
        return;
    }
    // (Dense outputs, the two-pass MODE_EMIT pass: a warp-uniform loop of
    // max-over-lanes |output(s)| predicated loads and stores instead of this
    // per-lane branch was measured slower -- C5 English 5K list 4.33 -> 4.72
    // ms, 20K 2x -- the per-record dependent loads of the output CSR, not the
    // divergence, bind that pass.)
    if (flag && live) emit_outputs<E, TIER, MODE>(s, key0, cnt, wp, s_stt, st, so);
}

// Two-pass emission (MODE_EMIT) from a CONVERGED warp -- used by the SPLIT
// re-walk only (a full-mask vote in the divergent callers, halo warm-ups and
// re-walks, would deadlock).  f = this lane reaches output state x at key0.
// States with fewer than AC_COOP_MIN outputs are written by their own lane;
// the records of larger output sets are written by the whole warp,
// AC_COOP_BATCH such states at a time: 32 consecutive ids read and 32
// consecutive records written per instruction, where a per-lane loop costs
// one L1 wavefront per record for the id and another for the store (each
// lane writes its own chain's range: 32 lines per instruction).  Measured
// (C5 English, 256 MiB, list): SPLIT 20K patterns (13.5 outputs per flagged
// byte) 11.8 -> 8.2 ms; in the GLOBAL tier's per-byte loop (English 5K,
// 4.3 outputs per flagged byte, 64-register kernel) every form was slower
// than the per-lane branch -- 4.30 ms vs 4.7 (all multi-output states
// cooperative), 5.0-5.4 (thresholds 6-12), 5.6-16 (batches of 2-8 states:
// register pressure) -- so that loop keeps emit_outputs.
#ifndef AC_COOP_MIN
#define AC_COOP_MIN 8  // smallest |output(x)| written by the whole warp
#endif
#ifndef AC_COOP_BATCH
#define AC_COOP_BATCH 2  // multi-output states whose id loads are in flight together
#endif
#ifndef AC_COOP
#define AC_COOP 1  // 0: per-lane emission in the SPLIT two-pass re-walk (ablation)
#endif
template <typename E, int TIER>
__device__ __forceinline__ void emit_coop(uint32_t x, uint32_t f, uint64_t key0, uint64_t &wp, const E *s_stt,
                                          const SttView &st, const ScanOut &so) {
    if (!__any_sync(0xffffffffu, f)) return;
    const uint2 o = out_info_pred<E, TIER, true>(s_stt, st, x, f);
    uint32_t c = o.y;
    if (TIER != AC_TIER_COMPACT && sizeof(E) == 2 && c == 0xFFFFu)
        c = __ldg(st.out_off + x + 1) - __ldg(st.out_off + x);
    const bool coop = c >= (uint32_t)AC_COOP_MIN;
    if (!coop) {  // one lane, few records
        if (c == 1u) {
            so.out[--wp] = key0 | o.x;
        } else {
            for (uint32_t j = o.x + c; j > o.x; --j) so.out[--wp] = key0 | __ldg(st.out_ids + j - 1);
        }
    }
    uint32_t multi = __ballot_sync(0xffffffffu, coop);
    const uint32_t lane = threadIdx.x & 31u;
    while (multi) {
        // up to AC_COOP_BATCH states: their (count, payload, key, first
        // record) broadcast, then every id load issued before any store
        uint32_t cc[AC_COOP_BATCH], pp[AC_COOP_BATCH];
        uint64_t kk[AC_COOP_BATCH], dd[AC_COOP_BATCH];
        uint32_t big = 0;
#pragma unroll
        for (int u = 0; u < AC_COOP_BATCH; u++) {
            const int i = multi ? __ffs(multi) - 1 : 0;
            const uint32_t has = multi != 0;
            multi &= multi - 1u;
            cc[u] = __shfl_sync(0xffffffffu, c, i) * has;
            pp[u] = __shfl_sync(0xffffffffu, o.x, i);
            kk[u] = __shfl_sync(0xffffffffu, key0, i);
            dd[u] = __shfl_sync(0xffffffffu, wp, i) - cc[u];
            big |= cc[u] > 32u;
        }
        if (!big) {
            uint32_t id[AC_COOP_BATCH];
#pragma unroll
            for (int u = 0; u < AC_COOP_BATCH; u++) id[u] = lane < cc[u] ? __ldg(st.out_ids + pp[u] + lane) : 0u;
#pragma unroll
            for (int u = 0; u < AC_COOP_BATCH; u++)
                if (lane < cc[u]) so.out[dd[u] + lane] = kk[u] | id[u];
        } else {
#pragma unroll
            for (int u = 0; u < AC_COOP_BATCH; u++)
                for (uint32_t b = lane; b < cc[u]; b += 32u) so.out[dd[u] + b] = kk[u] | __ldg(st.out_ids + pp[u] + b);
        }
    }
    if (coop) wp -= c;
}

// NEXT-4: one lookup for two bytes.  T2[s][c1*C + c2] =
// delta(delta(s,c1),c2) with bit 31 = output(final) != {} and bit 30 =
// output(middle) != {}; the (rare) middle state is recovered from the
// one-byte table.  b1 is the byte at key1's position, b2 the next one to the
// left (the walk is right to left).
static constexpr uint32_t T2_FIN = 1u << 31, T2_MID = 1u << 30, T2_MASK = (1u << 30) - 1;

template <typename E, int TIER, int MODE>
__device__ __forceinline__ void ac_step2(uint32_t &s, uint32_t &cnt, uint64_t &wp, uint32_t b1, uint32_t b2,
                                         uint64_t key1, uint64_t key2, bool live, const uint8_t *s_cmap,
                                         const E *s_stt, const SttView &st, const ScanOut &so) {
    const uint32_t c1 = s_cmap[b1], c2 = s_cmap[b2];
    const uint32_t e = __ldg(st.stt2 + s * st.stride2 + c1 * st.n_classes + c2);
    if ((e & (T2_FIN | T2_MID)) && live) {
        if (e & T2_MID) {
            const uint32_t mid = state_of<E, TIER>(next_entry<E, TIER>(s_stt, st, s, c1), st);
            emit_outputs<E, TIER, MODE>(mid, key1, cnt, wp, s_stt, st, so);
        }
        if (e & T2_FIN) emit_outputs<E, TIER, MODE>(e & T2_MASK, key2, cnt, wp, s_stt, st, so);
    }
    s = e & T2_MASK;
}

__device__ __forceinline__ uint32_t byte_of(const uint4 &v, int bb) {
    const uint32_t w = (bb >> 2) == 0 ? v.x : (bb >> 2) == 1 ? v.y : (bb >> 2) == 2 ? v.z : v.w;
    return __byte_perm(w, 0, 0x4440 | (bb & 3));  // one PRMT: zero-extended byte bb & 3
}

__device__ __forceinline__ unsigned long long warp_sum(unsigned long long v) {
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

// ------------------------------------------------------- k_scan_global (K1)
// Walk text[a, b) right to left; OWNED selects emission (else warm-up).
template <typename E, int TIER, int MODE, bool OWNED>
__device__ __forceinline__ void walk_global(const uint8_t *__restrict__ text, uint64_t a, uint64_t b, uint32_t &s,
                                            uint32_t &cnt, uint64_t &wp, const uint8_t *s_cmap, const E *s_stt,
                                            const SttView &st, const ScanOut &so) {
    auto one = [&](uint32_t byte, uint64_t pos) {
        if constexpr (OWNED)
            ac_step<E, TIER, MODE>(s, cnt, wp, byte, (so.base + pos) << 24, true, s_cmap, s_stt, st, so);
        else
            s = ac_move<E, TIER>(s, byte, s_cmap, s_stt, st);
    };
    uint64_t i = b;
    while (i > a && (reinterpret_cast<uintptr_t>(text + i) & 15u)) {
        --i;
        one(__ldg(text + i), i);
    }
    while (i >= a + 16) {
        const uint4 v = __ldg(reinterpret_cast<const uint4 *>(text + i - 16));
#pragma unroll
        for (int bb = 15; bb >= 0; --bb) one(byte_of(v, bb), i - 16 + bb);
        i -= 16;
    }
    while (i > a) {
        --i;
        one(__ldg(text + i), i);
    }
}

template <typename E, int TIER, int MODE>
__global__ void __launch_bounds__(GT) k_scan_global(const uint8_t *__restrict__ text, uint64_t n_total, SttView st,
                                                    Region ra, Region rb, ScanOut so) {
    extern __shared__ __align__(16) uint8_t smem[];
    uint8_t *s_cmap = smem;
    E *s_stt = reinterpret_cast<E *>(smem + 256);
    stage_tables<E>(s_cmap, s_stt, st);
    __syncthreads();
    if constexpr (MODE == MODE_EMIT) {
        if (so.res->status != AC_OK) return;  // capacity exceeded: write nothing
    }
    const uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const bool in_a = t < ra.n_chains;
    const uint64_t ci = in_a ? t : t - ra.n_chains;
    const uint64_t r_lo = in_a ? ra.lo : rb.lo, r_hi = in_a ? ra.hi : rb.hi;
    const uint64_t r_len = in_a ? ra.chain_len : rb.chain_len, r_n = in_a ? ra.n_chains : rb.n_chains;
    const uint64_t r_c0 = in_a ? ra.chain0 : rb.chain0;
    uint32_t cnt = 0;
    if (ci < r_n) {
        const uint64_t lo = r_lo + ci * r_len;
        const uint64_t own_hi = min(lo + r_len, r_hi);
        const uint64_t walk_hi = min(own_hi + (uint64_t)st.halo, n_total);
        const uint64_t g = r_c0 + ci;
        uint64_t wp = 0;
        if constexpr (MODE == MODE_EMIT) wp = so.chain_end[g];
        if constexpr (MODE == MODE_EMIT_OPT) wp = reinterpret_cast<uint64_t>(so.scratch + (g + 1) * so.q - 1);
        uint32_t s = 0;
        walk_global<E, TIER, MODE, false>(text, own_hi, walk_hi, s, cnt, wp, s_cmap, s_stt, st, so);
        walk_global<E, TIER, MODE, true>(text, lo, own_hi, s, cnt, wp, s_cmap, s_stt, st, so);
        if constexpr (MODE == MODE_COUNT_CHAINS || MODE == MODE_EMIT_OPT) so.chain_counts[g] = cnt;
        if constexpr (MODE == MODE_EMIT_OPT)
            if (so.chain_events)
                so.chain_events[g] =
                    (uint32_t)((reinterpret_cast<uint64_t>(so.scratch + (g + 1) * so.q - 1) - wp) >> 3);
    }
    if constexpr (MODE == MODE_COUNT_TOTAL) {
        const unsigned long long tot = warp_sum((unsigned long long)cnt);
        if ((threadIdx.x & 31) == 0 && tot) atomicAdd(so.total, tot);
    }
}

// Packet batches (the NIDS workload of P:108): segment i
// is text[seg_off[i], seg_off[i+1]) and is scanned from the start state on
// its own -- no halo, no occurrence crosses a boundary.  One thread per
// segment, right to left, so its records are canonical within the segment.
template <typename E, int TIER, int MODE>
__global__ void __launch_bounds__(GT) k_scan_segments(const uint8_t *__restrict__ text,
                                                      const uint64_t *__restrict__ seg_off, uint64_t n_seg,
                                                      SttView st, ScanOut so) {
    extern __shared__ __align__(16) uint8_t smem[];
    uint8_t *s_cmap = smem;
    E *s_stt = reinterpret_cast<E *>(smem + 256);
    stage_tables<E>(s_cmap, s_stt, st);
    __syncthreads();
    if constexpr (MODE == MODE_EMIT) {
        if (so.res->status != AC_OK) return;
    }
    const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    uint32_t cnt = 0;
    if (i < n_seg) {
        const uint64_t lo = seg_off[i], hi = seg_off[i + 1];
        uint64_t wp = 0;
        if constexpr (MODE == MODE_EMIT) wp = so.chain_end[i];
        uint32_t s = 0;
        walk_global<E, TIER, MODE, true>(text, lo, hi, s, cnt, wp, s_cmap, s_stt, st, so);
        if constexpr (MODE == MODE_COUNT_CHAINS) so.chain_counts[i] = cnt;
    }
    if constexpr (MODE == MODE_COUNT_TOTAL) {
        const unsigned long long tot = warp_sum((unsigned long long)cnt);
        if ((threadIdx.x & 31) == 0 && tot) atomicAdd(so.total, tot);
    }
}

// Re-scan the chains listed by k_gather (their matches overflowed the
// scratch slot) straight into their final positions.  One CTA per listed
// chain: the chain is split into GT sub-chains (each with its own halo
// warm-up, P:163-164 again one level down), counted, block-scanned and
// emitted -- so a dense chain costs ~2 x (L/GT + halo) steps, not L.
template <typename E, int TIER>
__global__ void __launch_bounds__(GT) k_rewalk(const uint8_t *__restrict__ text, uint64_t n_total, SttView st,
                                               Region ra, Region rb, StagedGeom g, ScanOut so,
                                               const uint64_t *__restrict__ list, const unsigned int *list_n) {
    const uint32_t nl = *list_n;
    if (nl == 0 || so.res->status != AC_OK) return;  // uniform: skip staging entirely
    extern __shared__ __align__(16) uint8_t smem[];
    __shared__ unsigned long long s_warp[GT / 32];
    uint8_t *s_cmap = smem;
    E *s_stt = reinterpret_cast<E *>(smem + 256);
    stage_tables<E>(s_cmap, s_stt, st);
    __syncthreads();
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    for (uint32_t i = blockIdx.x; i < nl; i += gridDim.x) {
        const uint64_t gi = list[i];
        uint64_t lo, own_hi;
        if (gi < ra.n_chains) {
            lo = ra.lo + gi * ra.chain_len;
            own_hi = min(lo + ra.chain_len, ra.hi);
        } else if (g.n_chains && gi >= g.chain0 && gi < g.chain0 + g.n_chains) {
            lo = g.m0 + (gi - g.chain0) * g.chain_len;
            own_hi = lo + g.chain_len;
        } else {
            lo = rb.lo + (gi - rb.chain0) * rb.chain_len;
            own_hi = min(lo + rb.chain_len, rb.hi);
        }
        const uint64_t sub = (own_hi - lo + GT - 1) / GT;
        const uint64_t a = min(lo + threadIdx.x * sub, own_hi), b = min(a + sub, own_hi);
        const uint64_t walk_hi = min(b + (uint64_t)st.halo, n_total);
        uint64_t wp = 0;
        uint32_t s = 0, cnt = 0;
        if (a < b) {
            walk_global<E, TIER, MODE_COUNT_CHAINS, false>(text, b, walk_hi, s, cnt, wp, s_cmap, s_stt, st, so);
            walk_global<E, TIER, MODE_COUNT_CHAINS, true>(text, a, b, s, cnt, wp, s_cmap, s_stt, st, so);
        }
        // suffix sum: records of later sub-chains come later in canonical order
        unsigned long long incl = cnt;
        for (int o = 1; o < 32; o <<= 1) {
            const unsigned long long y = __shfl_down_sync(0xffffffffu, incl, o);
            if (lane + o < 32) incl += y;
        }
        if (lane == 0) s_warp[w] = incl;
        __syncthreads();
        unsigned long long after = incl - cnt;
        for (int j = w + 1; j < GT / 32; j++) after += s_warp[j];
        __syncthreads();
        if (a < b && cnt) {
            wp = so.chain_end[gi] - after;
            s = 0;
            walk_global<E, TIER, MODE_EMIT, false>(text, b, walk_hi, s, cnt, wp, s_cmap, s_stt, st, so);
            walk_global<E, TIER, MODE_EMIT, true>(text, a, b, s, cnt, wp, s_cmap, s_stt, st, so);
        }
    }
}

// --------------------------------------------------------- TMA / mbarrier
__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
    uint32_t done;
    do {
        asm volatile(
            "{\n\t.reg .pred p;\n\t"
            "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
            "selp.u32 %0, 1, 0, p;\n\t}"
            : "=r"(done)
            : "r"(smem_u32(bar)), "r"(parity)
            : "memory");
    } while (!done);
}
// L2 policy of the text's TMA loads (chosen by the planner, StagedGeom).
// The text is streamed once: where the automaton lives in L2 (GLOBAL,
// HYBRID) its loads are evict-first so they do not push the STT out (C3:
// count 2,251 -> 2,860 Gbps).  For the shared-memory tiers they are
// evict-normal: a 16-byte box uses half of each 32-B sector and the next box
// the other half, so evict-first text lines are re-read from DRAM (C2 list
// scan, ncu: 839 MB DRAM reads vs 341 MB; step 0.5324 vs 0.5294 ms; with
// 32-byte boxes evict-first was also slower, 0.697 vs 0.683 ms).
__device__ __forceinline__ uint64_t text_l2_policy(uint32_t evict_first) {
    uint64_t pol;
    if (evict_first)
        asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    else
        asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}
__device__ __forceinline__ void tma_load_2d(void *dst, const CUtensorMap *map, int x, int y, uint64_t *bar,
                                            uint64_t policy) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes.L2::cache_hint "
        "[%0], [%1, {%2, %3}], [%4], %5;" ::"r"(smem_u32(dst)),
        "l"(reinterpret_cast<uint64_t>(map)), "r"(x), "r"(y), "r"(smem_u32(bar)), "l"(policy)
        : "memory");
}

// ------------------------------------------------- in-kernel offsets (a9)
// Epilogue of the single emitting pass when the main region starts the list
// (no head chains): a CTA's chains are consecutive in canonical order, so
// the CTA needs only the match total of the CTAs before it -- a decoupled
// look-back over one word per CTA (tile indices come from an atomic ticket
// taken at CTA start, so every predecessor is running or done; warp 0 reads
// 32 predecessors per step) -- to write every chain's end offset.  This replaces the k_offsets
// launch.  Shared memory for the exchange is the warps' own (finished) TMA
// ring slots.
__device__ __forceinline__ uint64_t ld_acquire_u64(const unsigned long long *p) {
    uint64_t v;
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_u64(unsigned long long *p, uint64_t v) {
    asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

template <int K>
__device__ __forceinline__ void place_chains(const ScanOut &so, const StagedGeom &g, uint8_t *wring, uint8_t *ring,
                                             int warp_ring, int warps, uint32_t tile, uint64_t row0,
                                             const uint32_t (&cnt)[K], const bool (&live)[K]) {
    const int lane = threadIdx.x & 31;
    // warp-level inclusive scan in canonical chain order (k major, lane minor)
    uint64_t incl[K];
    uint64_t run = 0;
#pragma unroll
    for (int k = 0; k < K; k++) {
        uint64_t v = live[k] ? cnt[k] : 0;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint64_t y = __shfl_up_sync(0xffffffffu, v, o);
            if (lane >= o) v += y;
        }
        incl[k] = run + v;
        run += __shfl_sync(0xffffffffu, v, 31);
    }
    uint64_t *wslot = reinterpret_cast<uint64_t *>(wring);
    __syncwarp();
    if (lane == 0) wslot[0] = run;  // this warp's total
    __syncthreads();
    if (threadIdx.x < 32) {
        uint64_t tot = 0;
        for (int w = 0; w < warps; w++) tot += reinterpret_cast<uint64_t *>(ring + w * warp_ring)[0];
        uint64_t prefix = 0;
        if (tile == 0) {
            if (lane == 0) st_release_u64(&so.tile_state[0], LB_INC | tot);
        } else {
            if (lane == 0) st_release_u64(&so.tile_state[tile], LB_AGG | tot);
            int64_t p = (int64_t)tile - 1;  // nearest predecessor of the window
            while (true) {
                const int64_t idx = p - lane;
                uint64_t st = idx >= 0 ? ld_acquire_u64(&so.tile_state[idx]) : LB_INC;  // before CTA 0: 0
                while (__any_sync(0xffffffffu, (st >> 62) == 0))
                    if ((st >> 62) == 0) st = ld_acquire_u64(&so.tile_state[idx]);  // not yet published
                const uint32_t inc = __ballot_sync(0xffffffffu, (st & LB_INC) == LB_INC);
                const int stop = inc ? __ffs(inc) - 1 : 31;  // lanes 0..stop contribute
                uint64_t val = lane <= stop ? (st & LB_VAL) : 0;
                for (int o = 16; o > 0; o >>= 1) val += __shfl_xor_sync(0xffffffffu, val, o);
                prefix += val;
                if (inc) break;
                p -= 32;
            }
            if (lane == 0) st_release_u64(&so.tile_state[tile], LB_INC | (prefix + tot));
        }
        if (lane == 0)  // exclusive prefix of every warp, into its slot (word 1)
            for (int w = 0; w < warps; w++) {
                uint64_t *ws = reinterpret_cast<uint64_t *>(ring + w * warp_ring);
                ws[1] = prefix;
                prefix += ws[0];
            }
    }
    __syncthreads();
    const uint64_t wpre = wslot[1];
#pragma unroll
    for (int k = 0; k < K; k++)
        if (live[k]) so.chain_end_w[g.chain0 + row0 + k * 32 + lane] = wpre + incl[k];
}

// ------------------------------------------- k_scan_staged (warp-private TMA)
template <int WARPS, int K, int W, int NST, int SWIZZLE>
struct StagedShape {
    static constexpr int ROWS = 32 * K;               // chains per warp = TMA box rows (<= 256)
    static constexpr int SLOT = ROWS * W;             // bytes per ring slot
    static constexpr int WARP_RING = NST * SLOT;
    static constexpr int RING = WARPS * WARP_RING;
    // mbarriers, then one 16-byte word for the CTA's tile ticket (dynamic
    // shared memory: a static __shared__ variable would push the 1024-B
    // aligned dynamic base by a whole 1 KB)
    static constexpr int BARS = (WARPS * NST * 8 + 16 + 15) / 16 * 16;
    static constexpr uint32_t SWZ = !SWIZZLE ? 0u : W == 128 ? 7u : W == 64 ? 3u : W == 32 ? 1u : 0u;
    static_assert(ROWS <= 256, "TMA box rows");
    static_assert(W == 16 || W == 32 || W == 64 || W == 128, "tile width");
    static_assert(SLOT % 512 == 0 || W == 16, "slots must keep the swizzle atom aligned");
};

// DENSE (SPLIT, EVENTS): emit inline at each flagged byte instead of the
// flag walk + re-walk, which for dense dictionaries walks most chunks twice
template <typename E, int TIER, int MODE, int WARPS, int K, int W, int NST, int SWIZZLE, int STRIDE = 1,
          bool IDENT = false, bool DENSE = false>
__global__ void __launch_bounds__(WARPS * 32, 1)
    k_scan_staged(const __grid_constant__ CUtensorMap tmap, const uint8_t *__restrict__ mtext, SttView st,
                  StagedGeom g, ScanOut so) {
    using Sh = StagedShape<WARPS, K, W, NST, SWIZZLE>;
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    // Swizzled tiles need their 1024-B atom alignment at run time; unswizzled
    // (W = 16) tiles only need TMA's 128 B, which the dynamic base has, so the
    // whole layout -- and the STT base -- is a compile-time constant.
    uint8_t *ring = Sh::SWZ ? smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u) : smem_raw;
    uint64_t *bars = reinterpret_cast<uint64_t *>(ring + Sh::RING);
    uint8_t *s_cmap = ring + Sh::RING + Sh::BARS;
    E *s_stt = reinterpret_cast<E *>(s_cmap + 256);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

    // in-kernel placement (look-back) takes the CTA's tile from a ticket
    const bool place = MODE == MODE_EMIT_OPT && so.tile_state != nullptr;
    uint32_t &s_tile = *reinterpret_cast<uint32_t *>(bars + WARPS * NST);
    if (threadIdx.x < WARPS * NST) mbar_init(&bars[threadIdx.x], 1);
    if (threadIdx.x == 0) {
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmap)) : "memory");
        s_tile = place ? atomicAdd(so.ticket, 1u) : blockIdx.x;
    }
    stage_tables<E>(s_cmap, s_stt, st);
    __syncthreads();  // the only CTA-wide barrier: tables staged, barriers initialised, tile taken
    if constexpr (MODE == MODE_EMIT) {
        if (so.res->status != AC_OK) return;  // capacity exceeded: write nothing
    }
    const uint32_t tile = s_tile;
#ifdef AC_DEBUG_TIMES
    uint64_t dbg_t0;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(dbg_t0));
#endif
    const uint64_t row0 = (uint64_t)tile * (WARPS * Sh::ROWS) + (uint64_t)warp * Sh::ROWS;
    // in-kernel placement ends with CTA barriers: idle warps stay (no tiles)
    const bool idle = row0 >= g.n_chains;
    if (idle && !place) return;  // idle warp (no later CTA barrier)

    uint8_t *wring = ring + warp * Sh::WARP_RING;
    uint64_t *wbar = bars + warp * NST;
    const uint64_t L = g.chain_len;
    const uint32_t H = st.halo;
    const uint32_t nh0 = (H + W - 1) / W;
    const bool tma_halo = (uint64_t)nh0 * W <= L;  // the halo window lies inside the next chain
    const uint32_t nh = tma_halo ? nh0 : 0;
    const uint32_t m = idle ? 0u : nh + (uint32_t)(L / W);
    // text_evict_first: 0 = evict-normal, 1 = evict-first, 2 = per 32-byte
    // sector: the half a chain reads first (the upper one, the walk is right
    // to left) evict-normal, the second half evict-first -- a 16-byte box
    // pulls a whole sector, so the first half keeps it for the second
    const uint64_t pol = text_l2_policy(g.text_evict_first != 0);
    const uint64_t pol_first_half = g.text_evict_first == 2 ? text_l2_policy(0) : pol;

    auto issue = [&](uint32_t j) {
        const uint32_t slot = j % NST;
        int x, y;
        if (j < nh) {  // halo: first bytes of the next chains (the row below)
            x = (int)((nh - 1 - j) * W);
            y = (int)(row0 + 1);
        } else {
            x = (int)(L - (uint64_t)(j - nh + 1) * W);
            y = (int)row0;
        }
        mbar_expect_tx(&wbar[slot], Sh::SLOT);
        tma_load_2d(wring + slot * Sh::SLOT, &tmap, x, y, &wbar[slot], (x & 16) ? pol_first_half : pol);
    };
    if (lane == 0)
        for (uint32_t j = 0; j < (uint32_t)NST && j < m; j++) issue(j);

    uint32_t s[K], hlen[K], cnt[K];
    uint64_t wp[K], cbase[K];
    bool live[K];
#pragma unroll
    for (int k = 0; k < K; k++) {
        const uint64_t c = row0 + k * 32 + lane;
        live[k] = c < g.n_chains;
        s[k] = 0;
        cnt[k] = 0;
        wp[k] = 0;
        cbase[k] = c * L;  // main-region offset of the chain's first byte
        const uint64_t rest = live[k] ? g.n_readable - (c + 1) * L : 0;
        hlen[k] = (uint32_t)(rest < H ? rest : H);
        if constexpr (MODE == MODE_EMIT)
            if (live[k]) wp[k] = so.chain_end[g.chain0 + c];
        if constexpr (MODE == MODE_EMIT_OPT)
            wp[k] = reinterpret_cast<uint64_t>(so.scratch + (g.chain0 + c + 1) * so.q - 1);
        // the last chain's halo row is outside the tensor map (and any halo
        // wider than the next chain): warm up from global memory instead
        if (live[k] && (!tma_halo || c + 1 == g.n_chains)) {
            for (int h = (int)hlen[k] - 1; h >= 0; --h)
                s[k] = ac_move<E, TIER>(s[k], __ldg(mtext + cbase[k] + L + h), s_cmap, s_stt, st);
            hlen[k] = 0;
        }
    }

    for (uint32_t j = 0; j < m; j++) {
        const uint32_t slot = j % NST;
        mbar_wait(&wbar[slot], (j / NST) & 1u);
        const uint8_t *tile = wring + slot * Sh::SLOT;
        if (j < nh) {
            const uint32_t col0 = (nh - 1 - j) * W;  // offset inside the halo window
#pragma unroll
            for (int q = W / 16 - 1; q >= 0; --q) {
                uint4 v[K];
#pragma unroll
                for (int k = 0; k < K; k++) {
                    const uint32_t logical = (k * 32 + lane) * W + q * 16;
                    v[k] = *reinterpret_cast<const uint4 *>(tile + (logical ^ (((logical >> 7) & Sh::SWZ) << 4)));
                }
#pragma unroll
                for (int bb = 15; bb >= 0; --bb) {
#pragma unroll
                    for (int k = 0; k < K; k++)
                        if (col0 + q * 16 + bb < hlen[k])
                            s[k] = ac_move<E, TIER>(s[k], byte_of(v[k], bb), s_cmap, s_stt, st);
                }
            }
        } else {
            const uint64_t col0 = L - (uint64_t)(j - nh + 1) * W;
            // single-slot ring (NST = 1): the lane copies its whole W-byte
            // row into registers and the slot is refilled at once, so the
            // next box's TMA overlaps the walk of this one; with 32-byte
            // boxes every 32-byte sector of the text is fetched exactly once
            // (a 16-byte box pulls a whole sector, and with the text's
            // evict-first policy the second half was often re-fetched)
            uint4 vall[NST == 1 ? W / 16 : 1][K];
            if constexpr (NST == 1) {
#pragma unroll
                for (int q = 0; q < W / 16; q++)
#pragma unroll
                    for (int k = 0; k < K; k++) {
                        const uint32_t logical = (k * 32 + lane) * W + q * 16;
                        vall[q][k] =
                            *reinterpret_cast<const uint4 *>(tile + (logical ^ (((logical >> 7) & Sh::SWZ) << 4)));
                    }
                // the slot may be overwritten only once every lane's loads have
                // landed: an opaque zero computed from the loaded words,
                // OR-reduced over the warp (the scoreboard waits for every
                // lane's loads), feeds the next box index; then the
                // generic-to-async proxy fence before the TMA write
                uint32_t dep = 0;
#pragma unroll
                for (int q = 0; q < W / 16; q++)
#pragma unroll
                    for (int k = 0; k < K; k++) dep |= vall[q][k].x | vall[q][k].y | vall[q][k].z | vall[q][k].w;
                dep &= (uint32_t)(g.n_chains >> 63);  // 0, but not a compile-time constant
                dep = __reduce_or_sync(0xffffffffu, dep);
                if (lane == 0 && j + 1 < m) {
                    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                    issue(j + 1 + dep);
                }
            }
#pragma unroll
            for (int q = W / 16 - 1; q >= 0; --q) {
                uint4 v[K];
                uint64_t kb[K];  // record key of the chunk's first byte: (global start) << 24
#pragma unroll
                for (int k = 0; k < K; k++) {
                    const uint32_t logical = (k * 32 + lane) * W + q * 16;
                    if constexpr (NST == 1)
                        v[k] = vall[q][k];
                    else
                        v[k] = *reinterpret_cast<const uint4 *>(tile + (logical ^ (((logical >> 7) & Sh::SWZ) << 4)));
                    kb[k] = (so.base + g.m0 + cbase[k] + col0 + q * 16) << 24;
                }
                // (COMPACT counting keeps its predicated per-byte count: measured faster)
                constexpr bool kDeferred = STRIDE == 1 && K == 1 && sizeof(E) == 2 &&
                                           (TIER != AC_TIER_COMPACT || MODE == MODE_EMIT || MODE == MODE_EMIT_OPT);
                // (a deferred-by-rewalk variant for 32-bit tables -- flag mask only,
                // re-walk the chunk in lanes that matched -- was measured slower on
                // C3, count 3.81 -> 4.95 ms: the L1-bound walk lost its overlap)
                if constexpr (kDeferred) {
                    // Deferred emission: walk the 16 bytes recording the
                    // flag bits and the (16-bit) states in registers, then
                    // emit in a warp-uniform loop that runs max-over-lanes
                    // popcount times (~3 for C2) instead of 16 times.
                    uint32_t hist[8], fm = 0, st0 = s[0], odd = 0;
#pragma unroll
                    for (int bb = 15; bb >= 0; --bb) {
                        const uint32_t e = next_entry<E, TIER>(s_stt, st, st0, s_cmap[byte_of(v[0], bb)]);
                        st0 = state_of<E, TIER>(e, st);
                        const uint32_t f = flag_of<E, TIER>(e, st0, st);
                        // byte bb's flag ends at bit bb; hist[i] = (state at 2i+1, state at 2i << 16)
                        if constexpr (TIER == AC_TIER_COMPACT) {
                            fm = fm * st.c_two + f;  // FMA pipe
                            if (bb & 1)
                                odd = st0;
                            else
                                hist[bb >> 1] = odd + st0 * st.c_k16;
                        } else {
                            fm = (fm << 1) | f;
                            if (bb & 1)
                                odd = st0;
                            else
                                hist[bb >> 1] = __byte_perm(odd, st0, 0x5410);
                        }
                    }
                    s[0] = st0;
                    if (!live[0]) fm = 0;
                    if constexpr (MODE == MODE_EMIT_OPT) {
                        // record k of the chain goes to slot last - k (if k < q);
                        // nk = -k keeps the address one IMAD.WIDE away.  Wide
                        // records are the final 8-byte keys; narrow ones (so.nbits
                        // > 0) are (offset in chain << nbits | pattern), 4 bytes,
                        // widened by k_gather -- half the scratch traffic
                        const uint64_t *const last = reinterpret_cast<const uint64_t *>(wp[0]);
                        const uint32_t *const last32 = reinterpret_cast<const uint32_t *>(wp[0] + 4);
                        int32_t nk = -(int32_t)cnt[0];
                        int32_t nq = -(int32_t)so.q;
                        // COMPACT output-table base kept in a register (ptxas
                        // may still re-derive nq from the constant bank)
                        uint32_t ob = smem_u32(s_stt) + st.c_out_x0;
                        asm volatile("" : "+r"(ob), "+r"(nq));
                        const uint32_t nb = so.nbits;
                        const uint32_t kn = ((uint32_t)col0 + (uint32_t)q * 16u) << nb;  // chunk offset, narrow
                        // A warp-uniform trip count (the most flags any lane
                        // holds) instead of a divergent while-any loop: no
                        // reconvergence bookkeeping, predicated body.
                        const uint32_t iters = __reduce_max_sync(0xffffffffu, (uint32_t)__popc(fm));
                        auto emit_loop = [&](auto narrow_tag) {
                            constexpr bool NARROW = decltype(narrow_tag)::value;
                            for (uint32_t it = 0; it < iters; ++it) {
                                uint32_t bb;  // highest flagged byte left (0xffffffff if none)
                                asm("bfind.u32 %0, %1;" : "=r"(bb) : "r"(fm));
                                const uint32_t act = fm != 0;
                                fm &= ~(1u << (bb & 31u));
                                const uint32_t i = bb >> 1;
                                const uint32_t a0 = (i & 1) ? hist[1] : hist[0], a1 = (i & 1) ? hist[3] : hist[2];
                                const uint32_t a2 = (i & 1) ? hist[5] : hist[4], a3 = (i & 1) ? hist[7] : hist[6];
                                const uint32_t b0 = (i & 2) ? a1 : a0, b1 = (i & 2) ? a3 : a2;
                                const uint32_t pr = (i & 4) ? b1 : b0;
                                const uint32_t x = __byte_perm(pr, 0, (bb & 1) ? 0x4410 : 0x4432);
                                uint2 o;
                                if constexpr (TIER == AC_TIER_COMPACT) {
                                    o = make_uint2(0u, 0u);
                                    asm("{\n\t.reg .pred p;\n\tsetp.ne.u32 p, %3, 0;\n\t@p ld.shared.v2.u32 {%0, %1}, [%2];\n\t}"
                                        : "+r"(o.x), "+r"(o.y)
                                        : "r"(ob + x * 8u), "r"(act));
                                } else {
                                    o = out_info_pred<E, TIER, true>(s_stt, st, x, act);
                                }
                                uint32_t c = o.y;
                                if (TIER != AC_TIER_COMPACT && sizeof(E) == 2 && c == 0xFFFFu)
                                    c = __ldg(st.out_off + x + 1) - __ldg(st.out_off + x);
                                // wide key = (start << 24) | pid with start = chunk start +
                                // bb: bb << 24 | pid < 2^32 (bb <= 15, pid < 2^24) is added
                                // to the chunk's key as ONE 32-bit addend; narrow: the same
                                // with the chain-relative offset and nb pattern bits
                                // (garbage, and never stored, in lanes with no flag left)
                                const uint32_t add = NARROW ? (bb << nb) + kn : bb * (1u << 24);
                                auto put = [&](int32_t k, uint32_t pid, bool pred) {
                                    if constexpr (NARROW)
                                        st_global32_if(last32, k, add + pid, pred);
                                    else
                                        st_global_if(last, k, kb[0] + (add + pid), pred);
                                };
                                put(nk, o.x, (c == 1u) & (nk > nq));
                                if (__any_sync(0xffffffffu, c > 1u)) {  // multi-output states (rare)
                                    for (uint32_t j = 0; j < c && c > 1u; ++j)
                                        put(nk - (int32_t)j, __ldg(st.out_ids + o.x + c - 1 - j), nk - (int32_t)j > nq);
                                }
                                nk -= (int32_t)c;
                            }
                        };
                        bool done = false;
                        if constexpr (TIER != AC_TIER_COMPACT) {
                            if (so.chain_events) {
                                // EVENTS (dense outputs): one event per flagged byte
                                // (start << 24 | state), the slot pointer moves down;
                                // only the output count is read here
                                uint64_t pol;
                                asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
                                for (uint32_t it = 0; it < iters; ++it) {
                                    uint32_t bb;
                                    asm("bfind.u32 %0, %1;" : "=r"(bb) : "r"(fm));
                                    const uint32_t act = fm != 0;
                                    fm &= ~(1u << (bb & 31u));
                                    const uint32_t i = bb >> 1;
                                    const uint32_t a0 = (i & 1) ? hist[1] : hist[0], a1 = (i & 1) ? hist[3] : hist[2];
                                    const uint32_t a2 = (i & 1) ? hist[5] : hist[4], a3 = (i & 1) ? hist[7] : hist[6];
                                    const uint32_t b0 = (i & 2) ? a1 : a0, b1 = (i & 2) ? a3 : a2;
                                    const uint32_t pr = (i & 4) ? b1 : b0;
                                    const uint32_t x = __byte_perm(pr, 0, (bb & 1) ? 0x4410 : 0x4432);
                                    uint32_t c = out_info_pred<E, TIER, false>(s_stt, st, x, act).y;
                                    if (sizeof(E) == 2 && c == 0xFFFFu)
                                        c = __ldg(st.out_off + x + 1) - __ldg(st.out_off + x);
                                    asm volatile(
                                        "{\n\t.reg .pred p;\n\tsetp.ne.u32 p, %3, 0;\n\t"
                                        "@p st.global.L2::cache_hint.u64 [%0], %1, %2;\n\t}" ::"l"(wp[0]),
                                        "l"((kb[0] + ((uint64_t)(bb & 15u) << 24)) | x), "l"(pol), "r"(act)
                                        : "memory");
                                    wp[0] -= (uint64_t)act << 3;
                                    nk -= (int32_t)c;
                                }
                                done = true;
                            }
                        }
                        if (done) {
                        } else if (nb)
                            emit_loop(std::true_type{});
                        else
                            emit_loop(std::false_type{});
                        cnt[0] = (uint32_t)(-nk);
                    } else
                    while (__any_sync(0xffffffffu, fm)) {
                        if (fm) {
                            const int bb = 31 - __clz(fm);
                            fm &= ~(1u << bb);
                            const int i = bb >> 1;
                            const uint32_t a0 = (i & 1) ? hist[1] : hist[0], a1 = (i & 1) ? hist[3] : hist[2];
                            const uint32_t a2 = (i & 1) ? hist[5] : hist[4], a3 = (i & 1) ? hist[7] : hist[6];
                            const uint32_t b0 = (i & 2) ? a1 : a0, b1 = (i & 2) ? a3 : a2;
                            const uint32_t pr = (i & 4) ? b1 : b0;
                            const uint32_t x = (bb & 1) ? (pr & 0xFFFFu) : (pr >> 16);
                            emit_outputs<E, TIER, MODE>(x, kb[0] + ((uint64_t)bb << 24), cnt[0], wp[0], s_stt, st,
                                                        so);
                        }
                    }
                } else if constexpr (STRIDE == 2) {
#pragma unroll
                    for (int bb = 15; bb >= 1; bb -= 2) {
#pragma unroll
                        for (int k = 0; k < K; k++)
                            ac_step2<E, TIER, MODE>(s[k], cnt[k], wp[k], byte_of(v[k], bb), byte_of(v[k], bb - 1),
                                                    kb[k] + ((uint64_t)bb << 24), kb[k] + ((uint64_t)(bb - 1) << 24),
                                                    live[k], s_cmap, s_stt, st, so);
                    }
                } else if constexpr (TIER == AC_TIER_SPLIT && (MODE == MODE_EMIT || MODE == MODE_EMIT_OPT) &&
                                     !kSplitInlineEmit && !DENSE) {
                    // rare matches (the tier is chosen for large byte
                    // dictionaries): the 16 steps only collect the flag bits
                    // -- the count-mode loop, no record keys or slot
                    // pointers live in it -- and a lane that saw a flag
                    // re-walks the chunk from its first state, emitting
                    // (C3: 0.5 % of lane-chunks, 15 % of warp-chunks)
#pragma unroll
                    for (int k = 0; k < K; k++) {
                        const uint32_t s_in = s[k];
                        uint32_t fm = 0;
#pragma unroll
                        for (int bb = 15; bb >= 0; --bb) {
                            const uint32_t e =
                                next_entry<E, TIER, IDENT>(s_stt, st, s[k], class_of_k<TIER, IDENT>(s_cmap, byte_of(v[k], bb), st));
                            s[k] = state_of<E, TIER>(e, st);
                            fm |= flag_of<E, TIER>(e, s[k], st) << bb;
                        }
                        if constexpr (MODE == MODE_EMIT && AC_COOP) {
                            // two-pass emission (dense outputs): every lane
                            // re-walks in step so the warp can write the
                            // multi-output states' records together (emit_coop)
                            if (!live[k]) fm = 0;
                            if (__any_sync(0xffffffffu, fm != 0)) {
                                uint32_t x = s_in;
#pragma unroll 1
                                for (int bb = 15; bb >= 0; --bb) {
                                    const uint32_t e = next_entry<E, TIER, IDENT>(
                                        s_stt, st, x, class_of_k<TIER, IDENT>(s_cmap, byte_of(v[k], bb), st));
                                    x = state_of<E, TIER>(e, st);
                                    emit_coop<E, TIER>(x, (fm >> bb) & 1u, kb[k] + ((uint64_t)bb << 24), wp[k], s_stt,
                                                       st, so);
                                }
                            }
                        } else if (__any_sync(0xffffffffu, fm != 0 && live[k]) && fm != 0 && live[k]) {
                            uint32_t x = s_in;
#pragma unroll 1
                            for (int bb = 15; bb >= 0; --bb) {
                                const uint32_t e = next_entry<E, TIER, IDENT>(
                                    s_stt, st, x, class_of_k<TIER, IDENT>(s_cmap, byte_of(v[k], bb), st));
                                x = state_of<E, TIER>(e, st);
                                if ((fm >> bb) & 1u)
                                    emit_outputs<E, TIER, MODE>(x, kb[k] + ((uint64_t)bb << 24), cnt[k], wp[k], s_stt,
                                                                st, so);
                            }
                        }
                    }
                } else if constexpr (TIER == AC_TIER_SPLIT) {
                    // counting with rare matches, or emitting inline (DENSE):
                    // the walk is the whole loop
#pragma unroll
                    for (int bb = 15; bb >= 0; --bb) {
#pragma unroll
                        for (int k = 0; k < K; k++) {
                            const uint32_t e =
                                next_entry<E, TIER, IDENT>(s_stt, st, s[k], class_of_k<TIER, IDENT>(s_cmap, byte_of(v[k], bb), st));
                            s[k] = state_of<E, TIER>(e, st);
                            if (__builtin_expect(flag_of<E, TIER>(e, s[k], st) != 0, 0) && live[k])
                                emit_outputs<E, TIER, MODE>(s[k], kb[k] + ((uint64_t)bb << 24), cnt[k], wp[k], s_stt,
                                                            st, so);
                        }
                    }
                } else {
#pragma unroll
                    for (int bb = 15; bb >= 0; --bb) {
#pragma unroll
                        for (int k = 0; k < K; k++)
                            ac_step<E, TIER, MODE>(s[k], cnt[k], wp[k], byte_of(v[k], bb),
                                                   kb[k] + ((uint64_t)bb << 24), live[k], s_cmap, s_stt, st, so);
                    }
                }
            }
        }
        if (NST > 1 || j < nh) {  // (NST = 1 main boxes refilled their slot above)
            __syncwarp();              // every lane is done with this slot
            if (lane == 0 && j + NST < m) issue(j + NST);
        }
    }

#ifdef AC_DEBUG_TIMES
    if (lane == 0 && tile < 1024 && warp < 32) {  // debug build only: walk time of each warp
        uint64_t t1;
        uint32_t smid;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t1));
        asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
        ac_dbg_times[(tile * 32 + warp) * 2] = dbg_t0;
        ac_dbg_times[(tile * 32 + warp) * 2 + 1] = (t1 - dbg_t0) | ((uint64_t)smid << 48);
    }
#endif
    if constexpr (MODE == MODE_COUNT_CHAINS || MODE == MODE_EMIT_OPT) {
#pragma unroll
        for (int k = 0; k < K; k++)
            if (live[k]) so.chain_counts[g.chain0 + row0 + k * 32 + lane] = cnt[k];
    }
    if constexpr (MODE == MODE_EMIT_OPT) {
        if (so.chain_events) {
#pragma unroll
            for (int k = 0; k < K; k++) {
                const uint64_t c = g.chain0 + row0 + k * 32 + lane;
                const uint64_t last = reinterpret_cast<uint64_t>(so.scratch + (c + 1) * so.q - 1);
                if (live[k]) so.chain_events[c] = (uint32_t)((last - wp[k]) >> 3);
            }
        }
    }
    if constexpr (MODE == MODE_EMIT_OPT) {
        if (place) place_chains<K>(so, g, wring, ring, Sh::WARP_RING, WARPS, tile, row0, cnt, live);
    }

    if constexpr (MODE == MODE_COUNT_TOTAL) {
        unsigned long long sum = 0;
#pragma unroll
        for (int k = 0; k < K; k++) sum += cnt[k];
        sum = warp_sum(sum);
        if (lane == 0 && sum) atomicAdd(so.total, sum);
    }
}

// ---------------------------------------------------------------- launchers
// Dispatch a runtime scan mode to a template argument.
template <typename F>
static cudaError_t with_mode(int mode, F &&f) {
    switch (mode) {
        case MODE_COUNT_TOTAL: return f(std::integral_constant<int, MODE_COUNT_TOTAL>{});
        case MODE_COUNT_CHAINS: return f(std::integral_constant<int, MODE_COUNT_CHAINS>{});
        case MODE_EMIT: return f(std::integral_constant<int, MODE_EMIT>{});
        case MODE_EMIT_OPT: return f(std::integral_constant<int, MODE_EMIT_OPT>{});
    }
    return cudaErrorInvalidValue;
}

template <typename E, int TIER, int MODE>
static cudaError_t launch_global_m(const uint8_t *text, uint64_t n_total, const SttView &st, const Region &a,
                                   const Region &b, const ScanOut &so, size_t smem, cudaStream_t stream) {
    auto kern = k_scan_global<E, TIER, MODE>;
    if (smem > 48 * 1024) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
    }
    const uint64_t threads = a.n_chains + b.n_chains;
    const unsigned grid = (unsigned)((threads + GT - 1) / GT);
    if (grid == 0) return cudaSuccess;
    kern<<<grid, GT, smem, stream>>>(text, n_total, st, a, b, so);
    return cudaGetLastError();
}

template <int TIER>
cudaError_t launch_global_tier(int mode, uint32_t eb, const uint8_t *text, uint64_t n_total, const SttView &st,
                               const Region &a, const Region &b, const ScanOut &so, size_t smem_stt,
                               cudaStream_t stream) {
    const size_t smem = 256 + smem_stt;
    if (eb == 2)
        return with_mode(mode, [&](auto m) {
            return launch_global_m<uint16_t, TIER, decltype(m)::value>(text, n_total, st, a, b, so, smem, stream);
        });
    if constexpr (TIER == AC_TIER_COMPACT) {
        return cudaErrorInvalidValue;  // COMPACT is 16-bit only
    } else {
        return with_mode(mode, [&](auto m) {
            return launch_global_m<uint32_t, TIER, decltype(m)::value>(text, n_total, st, a, b, so, smem, stream);
        });
    }
}

template <typename E, int TIER, int MODE>
static cudaError_t launch_segments_m(const uint8_t *text, const uint64_t *seg_off, uint64_t n_seg, const SttView &st,
                                     const ScanOut &so, size_t smem, cudaStream_t stream) {
    auto kern = k_scan_segments<E, TIER, MODE>;
    if (smem > 48 * 1024) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
    }
    const unsigned grid = (unsigned)((n_seg + GT - 1) / GT);
    if (grid == 0) return cudaSuccess;
    kern<<<grid, GT, smem, stream>>>(text, seg_off, n_seg, st, so);
    return cudaGetLastError();
}

template <typename E, int TIER>
static cudaError_t launch_segments_e(int mode, const uint8_t *text, const uint64_t *seg_off, uint64_t n_seg,
                                     const SttView &st, const ScanOut &so, size_t smem, cudaStream_t stream) {
    switch (mode) {
        case MODE_COUNT_TOTAL: return launch_segments_m<E, TIER, MODE_COUNT_TOTAL>(text, seg_off, n_seg, st, so, smem, stream);
        case MODE_COUNT_CHAINS: return launch_segments_m<E, TIER, MODE_COUNT_CHAINS>(text, seg_off, n_seg, st, so, smem, stream);
        case MODE_EMIT: return launch_segments_m<E, TIER, MODE_EMIT>(text, seg_off, n_seg, st, so, smem, stream);
    }
    return cudaErrorInvalidValue;
}

template <int TIER>
cudaError_t launch_segments_tier(int mode, uint32_t eb, const uint8_t *text, const uint64_t *seg_off, uint64_t n_seg,
                                 const SttView &st, const ScanOut &so, size_t smem_stt, cudaStream_t stream) {
    const size_t smem = 256 + smem_stt;
    if (eb == 2) return launch_segments_e<uint16_t, TIER>(mode, text, seg_off, n_seg, st, so, smem, stream);
    if constexpr (TIER == AC_TIER_COMPACT) {
        return cudaErrorInvalidValue;
    } else {
        return launch_segments_e<uint32_t, TIER>(mode, text, seg_off, n_seg, st, so, smem, stream);
    }
}

template <typename E, int TIER>
static cudaError_t launch_rewalk_e(const uint8_t *text, uint64_t n_total, const SttView &st, const Region &a,
                                   const Region &b, const StagedGeom &g, const ScanOut &so, const uint64_t *list,
                                   const unsigned int *list_n, size_t smem, int num_sms, cudaStream_t stream) {
    auto kern = k_rewalk<E, TIER>;
    if (smem > 48 * 1024) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
    }
    kern<<<num_sms, GT, smem, stream>>>(text, n_total, st, a, b, g, so, list, list_n);
    return cudaGetLastError();
}

template <int TIER>
cudaError_t launch_rewalk_tier(uint32_t eb, const uint8_t *text, uint64_t n_total, const SttView &st,
                               const Region &a, const Region &b, const StagedGeom &g, const ScanOut &so,
                               const uint64_t *list, const unsigned int *list_n, size_t smem_stt, int num_sms,
                               cudaStream_t stream) {
    const size_t smem = 256 + smem_stt;
    if (eb == 2)
        return launch_rewalk_e<uint16_t, TIER>(text, n_total, st, a, b, g, so, list, list_n, smem, num_sms, stream);
    if constexpr (TIER == AC_TIER_COMPACT) {
        return cudaErrorInvalidValue;
    } else {
        return launch_rewalk_e<uint32_t, TIER>(text, n_total, st, a, b, g, so, list, list_n, smem, num_sms, stream);
    }
}

template <typename E, int TIER, int MODE, int WARPS, int K, int W, int NST, int SWIZZLE, int STRIDE = 1,
          bool IDENT = false, bool DENSE = false>
static cudaError_t launch_staged_v(const CUtensorMap &tmap, const uint8_t *mtext, const SttView &st,
                                   const StagedGeom &g, const ScanOut &so, size_t smem_stt, cudaStream_t stream) {
    auto kern = k_scan_staged<E, TIER, MODE, WARPS, K, W, NST, SWIZZLE, STRIDE, IDENT, DENSE>;
    const StagedConfig cfg{WARPS, K, W, NST, SWIZZLE};
    const size_t smem = staged_smem_bytes(cfg, smem_stt);
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    const uint64_t R = (uint64_t)WARPS * 32 * K;
    const unsigned grid = (unsigned)((g.n_chains + R - 1) / R);
    if (grid == 0) return cudaSuccess;
    kern<<<grid, WARPS * 32, smem, stream>>>(tmap, mtext, st, g, so);
    return cudaGetLastError();
}

template <typename E, int TIER, int MODE>
static cudaError_t launch_staged_m(int variant, const CUtensorMap &tmap, const uint8_t *mtext, const SttView &st,
                                   const StagedGeom &g, const ScanOut &so, size_t smem_stt, cudaStream_t s) {
    if (st.stt2) {
        // the two-byte walk is instantiated for the L1/L2 tier with 32-bit
        // entries (large small-alphabet automata, e.g. DNA) and two shapes
        if constexpr (TIER == AC_TIER_GLOBAL && sizeof(E) == 4) {
            if (variant == 4) return launch_staged_v<E, TIER, MODE, 32, 1, 16, 3, 1, 2>(tmap, mtext, st, g, so, smem_stt, s);
            if (variant == 7) return launch_staged_v<E, TIER, MODE, 32, 1, 16, 2, 1, 2>(tmap, mtext, st, g, so, smem_stt, s);
        }
        return cudaErrorInvalidValue;
    }
    if constexpr (TIER == AC_TIER_SPLIT && (MODE == MODE_EMIT || MODE == MODE_EMIT_OPT)) {
        // the SPLIT auto variant (10) for identity class maps: no class-map
        // load in the walk (list modes; ptxas spills the count-mode forms)
        // EVENTS (dense outputs) on the auto variant: inline emission
        if constexpr (MODE == MODE_EMIT_OPT) {
            if (variant == 10 && so.chain_events)
                return launch_staged_v<E, TIER, MODE, 32, 1, 32, 1, 1, 1, false, true>(tmap, mtext, st, g, so,
                                                                                     smem_stt, s);
        }
        if (variant == 10 && st.cmap_ident && st.stride == kIdentStride)
            return launch_staged_v<E, TIER, MODE, 32, 1, 32, 1, 1, 1, true>(tmap, mtext, st, g, so, smem_stt, s);
    }
    switch (variant) {
#define AC_CASE(i, w, k, wd, ns, sw) \
    case i: return launch_staged_v<E, TIER, MODE, w, k, wd, ns, sw>(tmap, mtext, st, g, so, smem_stt, s);
        AC_STAGED_VARIANTS(AC_CASE)
#undef AC_CASE
    }
    return cudaErrorInvalidValue;
}

template <int TIER>
cudaError_t launch_staged_tier(int mode, uint32_t eb, int variant, const CUtensorMap &tmap, const uint8_t *mtext,
                               const SttView &st, const StagedGeom &g, const ScanOut &so, size_t smem_stt,
                               cudaStream_t stream) {
    if constexpr (TIER == AC_TIER_SPLIT) {  // the cold part is the 32-bit global table
        if (eb != 4) return cudaErrorInvalidValue;
        return with_mode(mode, [&](auto m) {
            return launch_staged_m<uint32_t, TIER, decltype(m)::value>(variant, tmap, mtext, st, g, so, smem_stt,
                                                                       stream);
        });
    } else if (eb == 2)
        return with_mode(mode, [&](auto m) {
            return launch_staged_m<uint16_t, TIER, decltype(m)::value>(variant, tmap, mtext, st, g, so, smem_stt,
                                                                       stream);
        });
    if constexpr (TIER == AC_TIER_COMPACT) {
        return cudaErrorInvalidValue;  // COMPACT is 16-bit only
    } else {
        return with_mode(mode, [&](auto m) {
            return launch_staged_m<uint32_t, TIER, decltype(m)::value>(variant, tmap, mtext, st, g, so, smem_stt,
                                                                       stream);
        });
    }
}

}  // namespace acx
