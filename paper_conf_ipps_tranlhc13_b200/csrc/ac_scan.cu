// ac_scan.cu -- phase-2 kernels of the Aho-Corasick scan for sm_100a.
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
//                  for sm_100a: a persistent-style CTA owns R = T*K chains of
//                  L bytes each; 2-D TMA boxes (W bytes x up to 256 chains)
//                  stream the chains' text into a swizzled shared-memory ring
//                  (the TMA swizzle is the hardware form of the paper's
//                  diagonal, bank-conflict-avoiding store), an
//                  mbarrier per stage replaces the load/compute barrier
//                  (P:216), and every lane reads its own chain 16 B at a time
//                  conflict free.
//   k_scan_global  the paper's "global memory only approach":
//                  chains read straight from global memory.  Also covers the
//                  unaligned head and the ragged tail of the staged path.
//   k_offsets      single-pass chained scan (decoupled look-back) of the
//                  per-chain counts -> per-chain end offsets + total.
//
// STT tiers: SMEM (whole table staged once per CTA),
// HYBRID (BFS-prefix rows in shared memory, the rest through L1/L2 with a
// generic load), GLOBAL (L1/L2 only).
#include <cuda/atomic>

#include "ac_scan.cuh"

namespace acx {

static constexpr int GT = 256;  // k_scan_global block size

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

// ------------------------------------------------------------------ helpers
template <typename E>
__device__ __forceinline__ void stage_tables(uint8_t *s_cmap, E *s_stt, const SttView &st) {
    const uint4 *c4 = reinterpret_cast<const uint4 *>(st.cmap);
    uint4 *d4 = reinterpret_cast<uint4 *>(s_cmap);
    for (int i = threadIdx.x; i < 16; i += blockDim.x) d4[i] = __ldg(c4 + i);
    size_t words = ((size_t)st.smem_rows * st.stride * sizeof(E) + 15) / 16;
    const uint4 *src = reinterpret_cast<const uint4 *>(st.stt);
    uint4 *dst = reinterpret_cast<uint4 *>(s_stt);
    for (size_t i = threadIdx.x; i < words; i += blockDim.x) dst[i] = __ldg(src + i);
}

template <typename E, int TIER>
__device__ __forceinline__ uint32_t stt_load(const E *s_stt, const E *g_stt, uint32_t hot, uint32_t s,
                                             uint32_t idx) {
    if constexpr (TIER == AC_TIER_SMEM) {
        return s_stt[idx];
    } else if constexpr (TIER == AC_TIER_GLOBAL) {
        return __ldg(g_stt + idx);
    } else {
        const E *p = (s < hot) ? (s_stt + idx) : (g_stt + idx);
        return *p;
    }
}

// One transition with no output (halo warm-up).
template <typename E, int TIER>
__device__ __forceinline__ uint32_t ac_move(uint32_t s, uint32_t byte, const uint8_t *s_cmap, const E *s_stt,
                                            const SttView &st) {
    uint32_t cls = s_cmap[byte];
    uint32_t e = stt_load<E, TIER>(s_stt, static_cast<const E *>(st.stt), st.smem_rows, s, s * st.stride + cls);
    return e & EntryBits<E>::MASK;
}

// Output summary of state s, stored in the padding of its own STT row
// (builder: payload u32 at info_col, then the count), read through the same
// residency tier as the transitions -- no dependent global CSR loads for the
// common single-output case.
template <typename E, int TIER>
__device__ __forceinline__ uint32_t out_count(const E *s_stt, const SttView &st, uint32_t s) {
    const uint32_t idx = s * st.stride + st.info_col + (sizeof(E) == 2 ? 2 : 1);
    uint32_t c = stt_load<E, TIER>(s_stt, static_cast<const E *>(st.stt), st.smem_rows, s, idx);
    if (sizeof(E) == 2 && c == 0xFFFFu) c = __ldg(st.out_off + s + 1) - __ldg(st.out_off + s);
    return c;
}

template <typename E, int TIER>
__device__ __forceinline__ uint32_t out_payload(const E *s_stt, const SttView &st, uint32_t s) {
    const uint32_t idx = s * st.stride + st.info_col;  // 4-byte aligned by construction
    const uint32_t *sp = reinterpret_cast<const uint32_t *>(s_stt + idx);
    const uint32_t *gp = reinterpret_cast<const uint32_t *>(static_cast<const E *>(st.stt) + idx);
    if constexpr (TIER == AC_TIER_SMEM) {
        return *sp;
    } else if constexpr (TIER == AC_TIER_GLOBAL) {
        return __ldg(gp);
    } else {
        return *((s < st.smem_rows) ? sp : gp);
    }
}

// One transition inside the owned chunk: count or emit output(s) at pos.
template <typename E, int TIER, int MODE>
__device__ __forceinline__ void ac_step(uint32_t &s, uint64_t &cnt, uint64_t &wp, uint32_t byte, uint64_t pos,
                                        bool live, const uint8_t *s_cmap, const E *s_stt, const SttView &st,
                                        const ScanOut &so) {
    uint32_t cls = s_cmap[byte];
    uint32_t e = stt_load<E, TIER>(s_stt, static_cast<const E *>(st.stt), st.smem_rows, s, s * st.stride + cls);
    s = e & EntryBits<E>::MASK;
    if ((e & EntryBits<E>::FLAG) && live) {
        const uint32_t c = out_count<E, TIER>(s_stt, st, s);
        if constexpr (MODE == MODE_EMIT) {
            const uint64_t key0 = (so.base + pos) << 24;
            const uint32_t p = out_payload<E, TIER>(s_stt, st, s);
            if (c == 1) {
                so.out[--wp] = key0 | p;
            } else {
                for (uint32_t j = p + c; j > p; --j) so.out[--wp] = key0 | __ldg(st.out_ids + j - 1);
            }
        } else {
            cnt += c;
        }
    }
}

__device__ __forceinline__ unsigned long long block_sum(unsigned long long v) {
    __shared__ unsigned long long red[32];
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    int w = threadIdx.x >> 5, l = threadIdx.x & 31;
    if (l == 0) red[w] = v;
    __syncthreads();
    unsigned long long r = 0;
    if (w == 0) {
        r = (l < (int)(blockDim.x >> 5)) ? red[l] : 0ull;
        for (int o = 16; o > 0; o >>= 1) r += __shfl_xor_sync(0xffffffffu, r, o);
    }
    return r;  // valid in thread 0
}

// ------------------------------------------------------- k_scan_global (K1)
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
    uint64_t cnt = 0;
    if (ci < r_n) {
        const uint64_t lo = r_lo + ci * r_len;
        const uint64_t own_hi = min(lo + r_len, r_hi);
        const uint64_t walk_hi = min(own_hi + (uint64_t)st.halo, n_total);
        const uint64_t g = r_c0 + ci;
        uint64_t wp = 0;
        if constexpr (MODE == MODE_EMIT) wp = so.chain_end[g];
        uint32_t s = 0;
        for (uint64_t i = walk_hi; i > own_hi;) {
            --i;
            s = ac_move<E, TIER>(s, __ldg(text + i), s_cmap, s_stt, st);
        }
        uint64_t i = own_hi;
        // 8 bytes at a time so the text loads are independent of the chain
        while (i >= lo + 8) {
            uint8_t b[8];
#pragma unroll
            for (int u = 0; u < 8; u++) b[u] = __ldg(text + i - 1 - u);
#pragma unroll
            for (int u = 0; u < 8; u++) ac_step<E, TIER, MODE>(s, cnt, wp, b[u], i - 1 - u, true, s_cmap, s_stt, st, so);
            i -= 8;
        }
        while (i > lo) {
            --i;
            ac_step<E, TIER, MODE>(s, cnt, wp, __ldg(text + i), i, true, s_cmap, s_stt, st, so);
        }
        if constexpr (MODE == MODE_COUNT_CHAINS) so.chain_counts[g] = cnt;
    }
    if constexpr (MODE == MODE_COUNT_TOTAL) {
        unsigned long long tot = block_sum(cnt);
        if (threadIdx.x == 0 && tot) atomicAdd(so.total, tot);
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
__device__ __forceinline__ void tma_load_2d(void *dst, const CUtensorMap *map, int x, int y, uint64_t *bar) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], "
        "[%4];" ::"r"(smem_u32(dst)),
        "l"(reinterpret_cast<uint64_t>(map)), "r"(x), "r"(y), "r"(smem_u32(bar))
        : "memory");
}

__device__ __forceinline__ uint32_t word_of(const uint4 &v, int q) {
    return q == 0 ? v.x : q == 1 ? v.y : q == 2 ? v.z : v.w;
}

// ---------------------------------------------- k_scan_staged (shared/TMA)
template <int T, int K, int W, int NST>
struct StagedShape {
    static constexpr int R = T * K;                      // chains per CTA
    static constexpr int STAGE_BYTES = R * W;            // one ring slot
    static constexpr int BOXR = R < 256 ? R : 256;       // TMA box rows (<= 256)
    static constexpr int NBOX = R / BOXR;
    static constexpr uint32_t SWZ = W == 128 ? 7u : (W == 64 ? 3u : 1u);
    static constexpr int HDR = NST * STAGE_BYTES + 128 + 256;  // ring + barriers + class map
};

template <typename E, int TIER, int MODE, int T, int K, int W, int NST>
__global__ void __launch_bounds__(T, 1)
    k_scan_staged(const __grid_constant__ CUtensorMap tmap, const uint8_t *__restrict__ mtext, SttView st,
                  StagedGeom g, ScanOut so) {
    using Sh = StagedShape<T, K, W, NST>;
    extern __shared__ uint8_t smem_raw[];
    // 1024-byte alignment for the 128B/64B swizzle atoms
    uint8_t *ring = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
    uint64_t *bars = reinterpret_cast<uint64_t *>(ring + NST * Sh::STAGE_BYTES);
    uint8_t *s_cmap = ring + NST * Sh::STAGE_BYTES + 128;
    E *s_stt = reinterpret_cast<E *>(s_cmap + 256);

    const uint64_t c_first = (uint64_t)blockIdx.x * Sh::R;
    const uint32_t m = (uint32_t)(g.chain_len / W);
    if (threadIdx.x == 0) {
        for (int i = 0; i < NST; i++) mbar_init(&bars[i], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmap)) : "memory");
    }
    stage_tables<E>(s_cmap, s_stt, st);
    __syncthreads();
    bool skip = false;
    if constexpr (MODE == MODE_EMIT) skip = so.res->status != AC_OK;  // uniform
    if (skip) return;

    auto issue = [&](uint32_t j) {
        const int slot = j % NST;
        mbar_expect_tx(&bars[slot], Sh::STAGE_BYTES);
        const int x = (int)(g.chain_len - (uint64_t)(j + 1) * W);
#pragma unroll
        for (int bx = 0; bx < Sh::NBOX; bx++)
            tma_load_2d(ring + slot * Sh::STAGE_BYTES + bx * Sh::BOXR * W, &tmap, x,
                        (int)(c_first + bx * Sh::BOXR), &bars[slot]);
    };
    if (threadIdx.x == 0)
        for (uint32_t j = 0; j < (uint32_t)NST && j < m; j++) issue(j);

    uint32_t s[K];
    uint64_t cnt[K], wp[K], cbase[K];
    bool live[K];
#pragma unroll
    for (int k = 0; k < K; k++) {
        const uint64_t c = c_first + k * T + threadIdx.x;
        live[k] = c < g.n_chains;
        s[k] = 0;
        cnt[k] = 0;
        wp[k] = 0;
        cbase[k] = c * g.chain_len;  // main-region offset of the chain's first byte
        if constexpr (MODE == MODE_EMIT)
            if (live[k]) wp[k] = so.chain_end[g.chain0 + c];
    }
    // halo warm-up (right of each chain, read from global), no output
    for (int h = (int)st.halo - 1; h >= 0; --h) {
#pragma unroll
        for (int k = 0; k < K; k++) {
            const uint64_t p = cbase[k] + g.chain_len + h;
            if (live[k] && p < g.n_readable) s[k] = ac_move<E, TIER>(s[k], __ldg(mtext + p), s_cmap, s_stt, st);
        }
    }

    for (uint32_t j = 0; j < m; j++) {
        const int slot = j % NST;
        mbar_wait(&bars[slot], (j / NST) & 1u);
        const uint8_t *tile = ring + slot * Sh::STAGE_BYTES;
        const uint64_t col0 = g.chain_len - (uint64_t)(j + 1) * W;  // chain-relative offset of tile column 0
#pragma unroll
        for (int q = W / 16 - 1; q >= 0; --q) {
            uint4 v[K];
#pragma unroll
            for (int k = 0; k < K; k++) {
                const uint32_t row = k * T + threadIdx.x;
                const uint32_t logical = row * W + q * 16;
                const uint32_t phys = logical ^ (((logical >> 7) & Sh::SWZ) << 4);
                v[k] = *reinterpret_cast<const uint4 *>(tile + phys);
            }
#pragma unroll
            for (int bb = 15; bb >= 0; --bb) {
#pragma unroll
                for (int k = 0; k < K; k++) {
                    const uint32_t byte = (word_of(v[k], bb >> 2) >> (8 * (bb & 3))) & 0xffu;
                    const uint64_t pos = g.m0 + cbase[k] + col0 + q * 16 + bb;
                    ac_step<E, TIER, MODE>(s[k], cnt[k], wp[k], byte, pos, live[k], s_cmap, s_stt, st, so);
                }
            }
        }
        __syncthreads();  // every lane is done with this slot
        if (threadIdx.x == 0 && j + NST < m) issue(j + NST);
    }

    if constexpr (MODE == MODE_COUNT_CHAINS) {
#pragma unroll
        for (int k = 0; k < K; k++)
            if (live[k]) so.chain_counts[g.chain0 + c_first + k * T + threadIdx.x] = cnt[k];
    }
    if constexpr (MODE == MODE_COUNT_TOTAL) {
        unsigned long long sum = 0;
#pragma unroll
        for (int k = 0; k < K; k++) sum += cnt[k];
        unsigned long long tot = block_sum(sum);
        if (threadIdx.x == 0 && tot) atomicAdd(so.total, tot);
    }
}

// ----------------------------------------------------- k_offsets (scan)
static constexpr int OT = 256, OITEMS = 8, OTILE = OT * OITEMS;
static constexpr uint64_t FLAG_AGG = 1ull << 62, FLAG_INC = 2ull << 62, VAL_MASK = (1ull << 62) - 1;

__global__ void __launch_bounds__(OT) k_offsets(const uint64_t *__restrict__ counts, uint64_t n,
                                                uint64_t *__restrict__ chain_end, uint64_t *tile_state,
                                                unsigned int *tile_counter, ac_result *res, uint64_t cap,
                                                int emitting) {
    __shared__ uint32_t s_tile;
    __shared__ uint64_t s_prefix;
    __shared__ uint64_t s_warp[OT / 32];
    if (threadIdx.x == 0) s_tile = atomicAdd(tile_counter, 1u);
    __syncthreads();
    const uint64_t tile = s_tile;
    const uint64_t first = tile * OTILE + (uint64_t)threadIdx.x * OITEMS;
    uint64_t v[OITEMS];
    uint64_t tsum = 0;
#pragma unroll
    for (int k = 0; k < OITEMS; k++) {
        v[k] = (first + k < n) ? counts[first + k] : 0;
        tsum += v[k];
    }
    // block exclusive scan of per-thread sums
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    uint64_t incl = tsum;
    for (int o = 1; o < 32; o <<= 1) {
        uint64_t y = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += y;
    }
    if (lane == 31) s_warp[w] = incl;
    __syncthreads();
    uint64_t wpre = 0, btot = 0;
    for (int i = 0; i < OT / 32; i++) {
        if (i < w) wpre += s_warp[i];
        btot += s_warp[i];
    }
    if (threadIdx.x == 0) {
        cuda::atomic_ref<unsigned long long, cuda::thread_scope_device> me(
            *reinterpret_cast<unsigned long long *>(&tile_state[tile]));
        uint64_t prefix = 0;
        if (tile == 0) {
            me.store(FLAG_INC | btot, cuda::memory_order_release);
        } else {
            me.store(FLAG_AGG | btot, cuda::memory_order_release);
            int64_t p = (int64_t)tile - 1;
            while (p >= 0) {
                cuda::atomic_ref<unsigned long long, cuda::thread_scope_device> other(
                    *reinterpret_cast<unsigned long long *>(&tile_state[p]));
                uint64_t st = other.load(cuda::memory_order_acquire);
                if ((st >> 62) == 0) continue;  // not yet published: spin
                prefix += st & VAL_MASK;
                if ((st & FLAG_INC) == FLAG_INC) break;
                --p;
            }
            me.store(FLAG_INC | (prefix + btot), cuda::memory_order_release);
        }
        s_prefix = prefix;
    }
    __syncthreads();
    uint64_t run = s_prefix + wpre + incl - tsum;
#pragma unroll
    for (int k = 0; k < OITEMS; k++) {
        run += v[k];
        if (first + k < n) chain_end[first + k] = run;
    }
    const uint64_t ntiles = (n + OTILE - 1) / OTILE;
    if (tile == ntiles - 1 && threadIdx.x == 0) {
        const uint64_t total = s_prefix + btot;
        res->count = total;
        res->status = (emitting && total > cap) ? (uint32_t)AC_ERR_CAPACITY : (uint32_t)AC_OK;
    }
}

size_t offsets_tiles(uint64_t n) { return (size_t)((n + OTILE - 1) / OTILE); }

// ---------------------------------------------------------------- launchers
template <typename E, int TIER, int MODE>
static cudaError_t launch_global_t(const uint8_t *text, uint64_t n_total, const SttView &st, const Region &a,
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

template <typename E, int MODE>
static cudaError_t launch_global_e(uint32_t tier, const uint8_t *text, uint64_t n_total, const SttView &st,
                                   const Region &a, const Region &b, const ScanOut &so, size_t smem,
                                   cudaStream_t s) {
    switch (tier) {
        case AC_TIER_SMEM: return launch_global_t<E, AC_TIER_SMEM, MODE>(text, n_total, st, a, b, so, smem, s);
        case AC_TIER_HYBRID: return launch_global_t<E, AC_TIER_HYBRID, MODE>(text, n_total, st, a, b, so, smem, s);
        default: return launch_global_t<E, AC_TIER_GLOBAL, MODE>(text, n_total, st, a, b, so, smem, s);
    }
}

cudaError_t launch_scan_global(int mode, uint32_t eb, uint32_t tier, const uint8_t *text, uint64_t n_total,
                               const SttView &st, const Region &a, const Region &b, const ScanOut &so,
                               size_t smem_stt, cudaStream_t stream) {
    const size_t smem = 256 + smem_stt;
    if (eb == 2) {
        if (mode == MODE_COUNT_TOTAL) return launch_global_e<uint16_t, MODE_COUNT_TOTAL>(tier, text, n_total, st, a, b, so, smem, stream);
        if (mode == MODE_COUNT_CHAINS) return launch_global_e<uint16_t, MODE_COUNT_CHAINS>(tier, text, n_total, st, a, b, so, smem, stream);
        return launch_global_e<uint16_t, MODE_EMIT>(tier, text, n_total, st, a, b, so, smem, stream);
    }
    if (mode == MODE_COUNT_TOTAL) return launch_global_e<uint32_t, MODE_COUNT_TOTAL>(tier, text, n_total, st, a, b, so, smem, stream);
    if (mode == MODE_COUNT_CHAINS) return launch_global_e<uint32_t, MODE_COUNT_CHAINS>(tier, text, n_total, st, a, b, so, smem, stream);
    return launch_global_e<uint32_t, MODE_EMIT>(tier, text, n_total, st, a, b, so, smem, stream);
}

// Staged kernel shapes (threads, chains per thread, tile width, ring depth).
// Variant 0 is "auto"; the table index is ac_match_opts.variant.
static const StagedConfig kVariants[] = {
    {256, 2, 64, 3},  // 1: 512 chains, 96 KB ring (SMEM-tier default)
    {256, 2, 32, 2},  // 2: 512 chains, 32 KB ring (largest STT budget)
    {512, 2, 32, 2},  // 3: 1024 chains, 64 KB ring
    {256, 4, 32, 2},  // 4: 1024 chains (4 per thread), 64 KB ring
    {512, 1, 64, 2},  // 5: 512 chains, 64 KB ring, 1 chain per thread
};

int staged_variant_count() { return (int)(sizeof(kVariants) / sizeof(kVariants[0])); }
const StagedConfig &staged_variant(int v) { return kVariants[v - 1]; }

size_t staged_smem_bytes(const StagedConfig &cfg, size_t smem_stt) {
    return 1024 + (size_t)cfg.stages * cfg.threads * cfg.k * cfg.width + 128 + 256 + smem_stt;
}

template <typename E, int TIER, int MODE, int T, int K, int W, int NST>
static cudaError_t launch_staged_v(const CUtensorMap &tmap, const uint8_t *mtext, const SttView &st,
                                   const StagedGeom &g, const ScanOut &so, size_t smem_stt, cudaStream_t stream) {
    auto kern = k_scan_staged<E, TIER, MODE, T, K, W, NST>;
    const StagedConfig cfg{T, K, W, NST};
    const size_t smem = staged_smem_bytes(cfg, smem_stt);
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    const uint64_t R = (uint64_t)T * K;
    const unsigned grid = (unsigned)((g.n_chains + R - 1) / R);
    if (grid == 0) return cudaSuccess;
    kern<<<grid, T, smem, stream>>>(tmap, mtext, st, g, so);
    return cudaGetLastError();
}

template <typename E, int TIER, int MODE>
static cudaError_t launch_staged_t(int variant, const CUtensorMap &tmap, const uint8_t *mtext, const SttView &st,
                                   const StagedGeom &g, const ScanOut &so, size_t smem_stt, cudaStream_t s) {
    switch (variant) {
        case 1: return launch_staged_v<E, TIER, MODE, 256, 2, 64, 3>(tmap, mtext, st, g, so, smem_stt, s);
        case 2: return launch_staged_v<E, TIER, MODE, 256, 2, 32, 2>(tmap, mtext, st, g, so, smem_stt, s);
        case 3: return launch_staged_v<E, TIER, MODE, 512, 2, 32, 2>(tmap, mtext, st, g, so, smem_stt, s);
        case 4: return launch_staged_v<E, TIER, MODE, 256, 4, 32, 2>(tmap, mtext, st, g, so, smem_stt, s);
        case 5: return launch_staged_v<E, TIER, MODE, 512, 1, 64, 2>(tmap, mtext, st, g, so, smem_stt, s);
    }
    return cudaErrorInvalidValue;
}

template <typename E, int MODE>
static cudaError_t launch_staged_e(int variant, uint32_t tier, const CUtensorMap &tmap, const uint8_t *mtext,
                                   const SttView &st, const StagedGeom &g, const ScanOut &so, size_t smem_stt,
                                   cudaStream_t s) {
    switch (tier) {
        case AC_TIER_SMEM: return launch_staged_t<E, AC_TIER_SMEM, MODE>(variant, tmap, mtext, st, g, so, smem_stt, s);
        case AC_TIER_HYBRID: return launch_staged_t<E, AC_TIER_HYBRID, MODE>(variant, tmap, mtext, st, g, so, smem_stt, s);
        default: return launch_staged_t<E, AC_TIER_GLOBAL, MODE>(variant, tmap, mtext, st, g, so, smem_stt, s);
    }
}

cudaError_t launch_scan_staged(int mode, uint32_t eb, uint32_t tier, int variant, const CUtensorMap &tmap,
                               const uint8_t *mtext, const SttView &st, const StagedGeom &g, const ScanOut &so,
                               size_t smem_stt, cudaStream_t stream) {
    if (eb == 2) {
        if (mode == MODE_COUNT_TOTAL) return launch_staged_e<uint16_t, MODE_COUNT_TOTAL>(variant, tier, tmap, mtext, st, g, so, smem_stt, stream);
        if (mode == MODE_COUNT_CHAINS) return launch_staged_e<uint16_t, MODE_COUNT_CHAINS>(variant, tier, tmap, mtext, st, g, so, smem_stt, stream);
        return launch_staged_e<uint16_t, MODE_EMIT>(variant, tier, tmap, mtext, st, g, so, smem_stt, stream);
    }
    if (mode == MODE_COUNT_TOTAL) return launch_staged_e<uint32_t, MODE_COUNT_TOTAL>(variant, tier, tmap, mtext, st, g, so, smem_stt, stream);
    if (mode == MODE_COUNT_CHAINS) return launch_staged_e<uint32_t, MODE_COUNT_CHAINS>(variant, tier, tmap, mtext, st, g, so, smem_stt, stream);
    return launch_staged_e<uint32_t, MODE_EMIT>(variant, tier, tmap, mtext, st, g, so, smem_stt, stream);
}

cudaError_t launch_offsets(const uint64_t *counts, uint64_t n, uint64_t *chain_end, uint64_t *tile_state,
                           unsigned int *tile_counter, ac_result *res, uint64_t cap, int emitting,
                           cudaStream_t stream) {
    const size_t tiles = offsets_tiles(n);
    if (tiles == 0) return cudaSuccess;
    k_offsets<<<(unsigned)tiles, OT, 0, stream>>>(counts, n, chain_end, tile_state, tile_counter, res, cap, emitting);
    return cudaGetLastError();
}

}  // namespace acx
