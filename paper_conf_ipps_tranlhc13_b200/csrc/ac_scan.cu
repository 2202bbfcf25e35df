// ac_scan.cu -- scan dispatch (tier x entry width x mode x variant) and the
// chained offset scan that turns per-chain counts into output positions.
// The scan kernels themselves are in ac_kernels.cuh, instantiated per STT
// tier by ac_tier_{smem,hybrid,global}.cu (compiled in parallel).
#include <cuda/atomic>

#include "ac_scan.cuh"

namespace acx {

static const StagedConfig kVariants[] = {
#define AC_ROW(i, w, k, wd, ns, sw) {w, k, wd, ns, sw},
    AC_STAGED_VARIANTS(AC_ROW)
#undef AC_ROW
};

int staged_variant_count() { return (int)(sizeof(kVariants) / sizeof(kVariants[0])); }
const StagedConfig &staged_variant(int v) { return kVariants[v - 1]; }

size_t staged_smem_bytes(const StagedConfig &cfg, size_t smem_stt) {
    const size_t ring = (size_t)cfg.warps * cfg.stages * 32 * cfg.k * cfg.width;
    const size_t bars = ((size_t)cfg.warps * cfg.stages * 8 + 16 + 15) / 16 * 16;  // + the tile ticket word
    // swizzled tiles (W >= 32) align the ring to the 1024-B swizzle atom at run time
    const size_t align = cfg.swizzle && cfg.width >= 32 ? 1024 : 0;
    return align + ring + bars + 256 + smem_stt;
}

cudaError_t launch_scan_global(int mode, uint32_t eb, uint32_t tier, const uint8_t *text, uint64_t n_total,
                               const SttView &st, const Region &a, const Region &b, const ScanOut &so,
                               size_t smem_stt, cudaStream_t stream) {
    switch (tier) {
        case AC_TIER_SMEM: return launch_global_tier<AC_TIER_SMEM>(mode, eb, text, n_total, st, a, b, so, smem_stt, stream);
        case AC_TIER_HYBRID: return launch_global_tier<AC_TIER_HYBRID>(mode, eb, text, n_total, st, a, b, so, smem_stt, stream);
        case AC_TIER_COMPACT: return launch_global_tier<AC_TIER_COMPACT>(mode, eb, text, n_total, st, a, b, so, smem_stt, stream);
        default: return launch_global_tier<AC_TIER_GLOBAL>(mode, eb, text, n_total, st, a, b, so, smem_stt, stream);
    }
}

cudaError_t launch_scan_staged(int mode, uint32_t eb, uint32_t tier, int variant, const CUtensorMap &tmap,
                               const uint8_t *mtext, const SttView &st, const StagedGeom &g, const ScanOut &so,
                               size_t smem_stt, cudaStream_t stream) {
    switch (tier) {
        case AC_TIER_SMEM: return launch_staged_tier<AC_TIER_SMEM>(mode, eb, variant, tmap, mtext, st, g, so, smem_stt, stream);
        case AC_TIER_HYBRID: return launch_staged_tier<AC_TIER_HYBRID>(mode, eb, variant, tmap, mtext, st, g, so, smem_stt, stream);
        case AC_TIER_COMPACT: return launch_staged_tier<AC_TIER_COMPACT>(mode, eb, variant, tmap, mtext, st, g, so, smem_stt, stream);
        case AC_TIER_SPLIT: return launch_staged_tier<AC_TIER_SPLIT>(mode, eb, variant, tmap, mtext, st, g, so, smem_stt, stream);
        default: return launch_staged_tier<AC_TIER_GLOBAL>(mode, eb, variant, tmap, mtext, st, g, so, smem_stt, stream);
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

// ------------------------------------------------------------- k_gather
// One warp per chain (grid-stride): a chain whose count fits its scratch slot
// is copied, coalesced, from the tail of the slot to [chain_end - cnt,
// chain_end); an overflowed chain is appended to the re-walk list.  With a
// TailPlace (the staged kernel already placed the main chains) every CTA
// also derives the grand total and the tail chains' offsets itself and CTA 0
// writes the count and the capacity status.
static constexpr uint64_t kMaxTail = 256;

// EV: the chains hold events (EVENTS single pass), else records; the record
// copy keeps 32 registers (8 CTAs of 256 threads per SM: one wave)
template <bool EV>
__global__ void __launch_bounds__(256, EV ? 1 : 8) k_gather(const uint64_t *__restrict__ counts, uint64_t *chain_end,
                                                uint64_t n_chains, const uint64_t *__restrict__ scratch, uint32_t q,
                                                uint64_t *__restrict__ out, ac_result *res, uint64_t *list,
                                                unsigned int *list_n, TailPlace tp, NarrowMain nm, EventExpand ev) {
    const int lane = threadIdx.x & 31;
    uint64_t main_total = 0;
    if (tp.tile_state) {
        __shared__ unsigned long long s_tail[256 / 32];
        main_total = tp.tile_state[tp.n_tiles - 1] & LB_VAL;
        unsigned long long t = threadIdx.x < tp.tail_n ? counts[tp.tail_c0 + threadIdx.x] : 0;
        for (int o = 16; o > 0; o >>= 1) t += __shfl_xor_sync(0xffffffffu, t, o);
        if (lane == 0) s_tail[threadIdx.x >> 5] = t;
        __syncthreads();
        uint64_t total = main_total;
        for (int i = 0; i < 256 / 32; i++) total += s_tail[i];
        if (blockIdx.x == 0 && threadIdx.x == 0) {
            res->count = total;
            res->status = total > tp.cap ? (uint32_t)AC_ERR_CAPACITY : (uint32_t)AC_OK;
        }
        if (total > tp.cap) return;  // capacity exceeded: write nothing
    } else if (res->status != AC_OK) {
        return;
    }
    const uint64_t warps = (uint64_t)gridDim.x * (blockDim.x >> 5);
    for (uint64_t c = (uint64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); c < n_chains; c += warps) {
        // count and end offset are loaded together (one round trip, not two);
        // the end read for an empty chain is not used.
        // (prefetching the next chain's pair during this chain's copy was
        // measured slower on C2: 0.048 -> 0.059 ms)
        const uint64_t cnt = counts[c];
        const bool tail = tp.tile_state && c >= tp.tail_c0;  // its end is not written yet: derive it
        uint64_t end = tail ? 0 : chain_end[c];
        if (tail) {
            // tail chain: main total + inclusive sum of the tail counts up to c
            unsigned long long v = 0;
            for (uint64_t j = tp.tail_c0 + lane; j <= c; j += 32) v += counts[j];
            for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
            end = main_total + v;
            if (lane == 0) chain_end[c] = end;  // k_rewalk reads it for listed chains
        }
        if (cnt == 0) continue;
        if constexpr (EV) {
            // EVENTS: the chain's events, canonical order, at the slot's end;
            // 32 at a time: each lane reads its event's output summary, a warp
            // scan places the records, and the warp writes them 32 consecutive
            // records per round (full 32-byte sectors) -- each record's owner
            // is the last event starting at or before it
            const uint32_t ne = ev.events[c];
            if (ne > q) {
                if (lane == 0) list[atomicAdd(list_n, 1u)] = c;
                continue;
            }
            const uint64_t *src = scratch + c * q + (q - ne);
            uint64_t run = end - cnt;  // index of the chain's first record
            uint32_t le;
            asm("mov.u32 %0, %%lanemask_le;" : "=r"(le));
            // a three-stage pipeline over chunks of 32 events: the events of
            // chunk i + 2 and the output summaries of chunk i + 1 (whose events
            // landed during chunk i - 1) are in flight while chunk i is written
            // (ncu: the one-stage prefetch left 32 % of the stalls on the event
            // load feeding the summary load)
            auto load_ev = [&](uint32_t i0) -> uint64_t {
                return i0 + lane < ne ? __ldg(src + i0 + lane) : ~0ull;
            };
            auto summary = [&](uint64_t e, uint32_t &p, uint32_t &cx) {
                p = cx = 0;
                if (e != ~0ull) {
                    const uint32_t x = (uint32_t)e & 0xFFFFFFu;
                    if (ev.entry_bytes == 4) {
                        const uint32_t *row = static_cast<const uint32_t *>(ev.stt) + (uint64_t)x * ev.stride + ev.info_col;
                        p = __ldg(row);
                        cx = __ldg(row + 1);
                    } else {
                        const uint16_t *row = static_cast<const uint16_t *>(ev.stt) + (uint64_t)x * ev.stride + ev.info_col;
                        p = __ldg(reinterpret_cast<const uint32_t *>(row));
                        cx = __ldg(row + 2);
                        if (cx == 0xFFFFu) cx = __ldg(ev.out_off + x + 1) - __ldg(ev.out_off + x);
                    }
                }
            };
            uint64_t e_n = load_ev(0), e_nn = load_ev(32);
            uint32_t p_n, cx_n;
            summary(e_n, p_n, cx_n);
            for (uint32_t i0 = 0; i0 < ne; i0 += 32) {
                const uint64_t e = e_n;
                const uint32_t p = p_n, cx = cx_n;
                e_n = e_nn;
                if (i0 + 32 < ne) {
                    e_nn = load_ev(i0 + 64);
                    summary(e_n, p_n, cx_n);
                }
                uint32_t incl = cx;
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    const uint32_t t = __shfl_up_sync(0xffffffffu, incl, o);
                    if (lane >= o) incl += t;
                }
                const uint32_t excl = incl - cx, T = __shfl_sync(0xffffffffu, incl, 31);
                const uint32_t khi = (uint32_t)(e >> 32), klo = (uint32_t)e & 0xFF000000u;
                // rounds of 32 records, four at a time: every id load of the
                // batch is issued before its stores
                constexpr int RB = 4;
                for (uint32_t R0 = 0; R0 < T; R0 += 32 * RB) {
                    uint32_t id[RB], kh[RB], kl[RB];
#pragma unroll
                    for (int u = 0; u < RB; u++) {
                        const uint32_t R = R0 + 32u * u;
                        // record positions in (R, R + 32) where an event's records start
                        const uint32_t starts = __reduce_or_sync(
                            0xffffffffu, (cx && excl > R && excl < R + 32) ? 1u << (excl - R) : 0u);
                        const int o0 = __popc(__ballot_sync(0xffffffffu, cx && excl <= R)) - 1;  // owner of R
                        const int own = o0 + __popc(starts & le);
                        const uint32_t po = __shfl_sync(0xffffffffu, p, own), co = __shfl_sync(0xffffffffu, cx, own);
                        const uint32_t eo = __shfl_sync(0xffffffffu, excl, own);
                        kh[u] = __shfl_sync(0xffffffffu, khi, own);
                        kl[u] = __shfl_sync(0xffffffffu, klo, own);
                        const uint32_t r = R + lane;
                        id[u] = po;
                        if (r < T && co != 1u) id[u] = __ldg(ev.out_ids + po + (r - eo));
                    }
#pragma unroll
                    for (int u = 0; u < RB; u++) {
                        const uint32_t r = R0 + 32u * u + lane;
                        if (r < T) out[run + r] = ((uint64_t)kh[u] << 32) | kl[u] | id[u];
                    }
                }
                run += T;
            }
            continue;
        }
        if (cnt > q) {
            if (lane == 0) list[atomicAdd(list_n, 1u)] = c;
            continue;
        }
        uint64_t *dst = out + end - cnt;
        // every load of a batch is issued before its stores (predicated, not
        // a remainder loop): a typical chain (~100 records) is one round trip
        constexpr int B = 8;
        if (nm.nbits && c - nm.c0 < nm.n) {
            // narrow records (offset << nbits | pid) packed at the slot's end
            const uint32_t *src = reinterpret_cast<const uint32_t *>(scratch + (c + 1) * q) - cnt;
            const uint64_t lo = nm.lo0 + (c - nm.c0) * nm.chain_len;  // chain's first byte
            const uint32_t nb = nm.nbits, pm = (1u << nb) - 1u;
            for (uint64_t i = lane; i < cnt; i += 32 * B) {
                uint32_t r[B];
#pragma unroll
                for (int u = 0; u < B; u++) r[u] = i + 32 * u < cnt ? __ldg(src + i + 32 * u) : 0u;
#pragma unroll
                for (int u = 0; u < B; u++)
                    if (i + 32 * u < cnt) dst[i + 32 * u] = ((lo + (r[u] >> nb)) << 24) | (r[u] & pm);
            }
            continue;
        }
        const uint64_t *src = scratch + c * q + (q - cnt);
        for (uint64_t i = lane; i < cnt; i += 32 * B) {
            uint64_t r[B];
#pragma unroll
            for (int u = 0; u < B; u++) r[u] = i + 32 * u < cnt ? __ldg(src + i + 32 * u) : 0ull;
#pragma unroll
            for (int u = 0; u < B; u++)
                if (i + 32 * u < cnt) dst[i + 32 * u] = r[u];
        }
    }
}

cudaError_t launch_gather(const uint64_t *counts, uint64_t *chain_end, uint64_t n_chains,
                          const uint64_t *scratch, uint32_t q, uint64_t *out, ac_result *res,
                          uint64_t *list, unsigned int *list_n, const TailPlace &tp, const NarrowMain &nm,
                          const EventExpand &ev, int num_sms, cudaStream_t stream) {
    if (n_chains == 0) return cudaSuccess;
    if (tp.tile_state && tp.tail_n > kMaxTail) return cudaErrorInvalidValue;
    const uint64_t want = (n_chains + 7) / 8;
    const unsigned grid = (unsigned)(want < (uint64_t)num_sms * 8 ? want : (uint64_t)num_sms * 8);
    if (ev.events)
        k_gather<true><<<grid, 256, 0, stream>>>(counts, chain_end, n_chains, scratch, q, out, res, list, list_n, tp, nm,
                                                 ev);
    else
        k_gather<false><<<grid, 256, 0, stream>>>(counts, chain_end, n_chains, scratch, q, out, res, list, list_n, tp,
                                                  nm, ev);
    return cudaGetLastError();
}

cudaError_t launch_segments(int mode, uint32_t eb, uint32_t tier, const uint8_t *text, const uint64_t *seg_off,
                            uint64_t n_seg, const SttView &st, const ScanOut &so, size_t smem_stt, cudaStream_t stream) {
    switch (tier) {
        case AC_TIER_SMEM: return launch_segments_tier<AC_TIER_SMEM>(mode, eb, text, seg_off, n_seg, st, so, smem_stt, stream);
        case AC_TIER_HYBRID: return launch_segments_tier<AC_TIER_HYBRID>(mode, eb, text, seg_off, n_seg, st, so, smem_stt, stream);
        case AC_TIER_COMPACT: return launch_segments_tier<AC_TIER_COMPACT>(mode, eb, text, seg_off, n_seg, st, so, smem_stt, stream);
        default: return launch_segments_tier<AC_TIER_GLOBAL>(mode, eb, text, seg_off, n_seg, st, so, smem_stt, stream);
    }
}

cudaError_t launch_rewalk(uint32_t eb, uint32_t tier, const uint8_t *text, uint64_t n_total, const SttView &st,
                          const Region &a, const Region &b, const StagedGeom &g, const ScanOut &so,
                          const uint64_t *list, const unsigned int *list_n, size_t smem_stt, int num_sms,
                          cudaStream_t stream) {
    switch (tier) {
        case AC_TIER_SMEM: return launch_rewalk_tier<AC_TIER_SMEM>(eb, text, n_total, st, a, b, g, so, list, list_n, smem_stt, num_sms, stream);
        case AC_TIER_HYBRID: return launch_rewalk_tier<AC_TIER_HYBRID>(eb, text, n_total, st, a, b, g, so, list, list_n, smem_stt, num_sms, stream);
        case AC_TIER_COMPACT: return launch_rewalk_tier<AC_TIER_COMPACT>(eb, text, n_total, st, a, b, g, so, list, list_n, smem_stt, num_sms, stream);
        default: return launch_rewalk_tier<AC_TIER_GLOBAL>(eb, text, n_total, st, a, b, g, so, list, list_n, smem_stt, num_sms, stream);
    }
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
