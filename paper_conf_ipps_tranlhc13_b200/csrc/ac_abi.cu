// ac_abi.cu -- the C ABI of libac (include/ac.h): validation, STT upload and
// residency planning, scan planning and launch sequencing.
//
// Phase split follows the paper: the STT is built once on the host and
// copied to the device; the text is device resident before the scan
// (P:148); build and copies are outside the timed scan.
#include <algorithm>
#include <cstring>
#include <mutex>
#include <new>
#include <string>

#include <cudaTypedefs.h>
#include <nvtx3/nvToolsExt.h>

#include "ac_internal.h"
#include "ac_scan.cuh"

namespace acx {

static thread_local std::string g_err;
static thread_local uint32_t g_launches = 0;
static thread_local uint32_t g_scratch_rec = 0;  // bytes per scratch record of the last list-mode call
static thread_local const char *g_names[16];
static thread_local uint64_t g_bytes[16];  // text bytes each scan launch walks (owned + halo), 0 otherwise

void set_error(const std::string &msg) { g_err = msg; }

static ac_status cuda_fail(cudaError_t e, const char *what) {
    set_error(std::string(what) + ": " + cudaGetErrorName(e) + " (" + cudaGetErrorString(e) + ")");
    return AC_ERR_CUDA;
}

#define AC_CUDA(call, what)                          \
    do {                                             \
        cudaError_t e_ = (call);                     \
        if (e_ != cudaSuccess) return cuda_fail(e_, what); \
    } while (0)

static const uint64_t kGlobalTailChain = 64;  // head/tail chains of the staged path
static const int kAutoVariant = 4;  // 32 warps x 1 chain, 16-byte tiles, 3 slots (48 KB ring)
static const int kLeanVariant = 7;  // 32 warps x 1 chain, 16-byte tiles, 2 slots (32 KB ring): sizes COMPACT
// COMPACT automata run variant 11 (32 warps x 1 chain, one unswizzled 32-byte
// slot copied to registers and refilled at once): C2 list 0.548 -> 0.517 ms
// per 256 MiB (half the per-chunk ring bookkeeping per byte); its ring and
// barriers take no more shared memory than variant 7's, so COMPACT tables
// sized for variant 7 fit
static const int kCompactVariant = 11;
// SPLIT automata run variant 10 (32 warps x 1 chain, 32-byte tiles, 1 slot
// refilled as soon as it is copied to registers: 32 KB ring + 1 KB swizzle
// alignment; every text sector is fetched once -- C3 list 1.44 vs 3.3 GB of
// DRAM reads per GiB with variant 7's 16-byte boxes -- and the list step is
// 2.5 % faster: 0.628 vs 0.644 ms per 256 MiB); they are sized so that the
// lean variant 7 can stage them too
static const int kSplitVariant = 10;
// COMPACT budget used by ac_compile (no device): B200's 227 KB opt-in shared
// memory minus the lean staged variant's ring and bookkeeping (= stt_budget)
#define kDefaultCompactBudget (232448 - staged_smem_bytes(staged_variant(kLeanVariant), 0) - 128)
#define kDefaultSplitBudget (232448 - staged_smem_bytes(staged_variant(kSplitVariant), 0) - 128)
// Below ~32 MiB the staged kernel cannot fill 148 SMs x 1024 chains with
// chains of >= 256 B; the global kernel's shorter chains win (C1: 1 MiB list
// 0.037 ms global vs 0.052 ms staged).
static const uint64_t kStagedMinBytes = 32ull << 20;
static const uint64_t kMaxSlots = 4096;  // scratch records per chain in the single emitting pass
static const uint64_t kStagedMinChain = 256;

// cuTensorMapEncodeTiled through the runtime's driver entry point (no -lcuda).
static PFN_cuTensorMapEncodeTiled_v12000 encode_fn() {
    static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
        void *p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
    });
    return fn;
}

// NVTX range for the scope of a host call (header-only NVTX3: a no-op unless
// a profiler injects itself), so ncu/nsys timelines show build, scan,
// gather and host-pipeline phases by name.
struct NvtxRange {
    explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
};

// Makes `device` current for the scope of a call and restores the caller's.
struct DeviceGuard {
    int prev = -1;
    explicit DeviceGuard(int device) {
        if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
        if (prev != device) cudaSetDevice(device);
        else prev = -1;
    }
    ~DeviceGuard() {
        if (prev >= 0) cudaSetDevice(prev);
    }
};

// Per-thread, per-device side stream + fork/join events (created lazily,
// kept for the thread's lifetime).
struct SideStream {
    cudaStream_t stream = nullptr;
    cudaEvent_t fork = nullptr, join = nullptr;
};

static ac_status side_stream(int device, SideStream **out) {
    static thread_local SideStream per_dev[64];
    if (device < 0 || device >= 64) {
        set_error("device index out of range");
        return AC_ERR_INVALID_ARG;
    }
    SideStream &s = per_dev[device];
    if (!s.stream) {
        int prev = -1;
        cudaGetDevice(&prev);
        AC_CUDA(cudaSetDevice(device), "cudaSetDevice");
        cudaError_t e = cudaStreamCreateWithFlags(&s.stream, cudaStreamNonBlocking);
        if (e == cudaSuccess) e = cudaEventCreateWithFlags(&s.fork, cudaEventDisableTiming);
        if (e == cudaSuccess) e = cudaEventCreateWithFlags(&s.join, cudaEventDisableTiming);
        if (prev >= 0) cudaSetDevice(prev);
        if (e != cudaSuccess) return cuda_fail(e, "side stream setup");
    }
    *out = &s;
    return AC_OK;
}

// libac's own stream-ordered memory pool per device: workspace and scratch
// are reused from call to call (a list-mode call allocates ~GBs of scratch)
// without touching the device's default pool, which the host application's
// allocator may rely on; memory above the release threshold goes back to the
// device at the next synchronisation.
static const uint64_t kPoolKeepBytes = 16ull << 30;
static cudaMemPool_t lib_pool(int device) {
    static std::mutex mu;
    static cudaMemPool_t pools[64] = {};
    if (device < 0 || device >= 64) return nullptr;
    std::lock_guard<std::mutex> lk(mu);
    if (!pools[device]) {
        cudaMemPoolProps props = {};
        props.allocType = cudaMemAllocationTypePinned;
        props.location.type = cudaMemLocationTypeDevice;
        props.location.id = device;
        cudaMemPool_t p = nullptr;
        if (cudaMemPoolCreate(&p, &props) != cudaSuccess) {
            cudaGetLastError();
            return nullptr;
        }
        uint64_t thr = kPoolKeepBytes;
        cudaMemPoolSetAttribute(p, cudaMemPoolAttrReleaseThreshold, &thr);
        pools[device] = p;
    }
    return pools[device];
}

// Stream-ordered allocation from libac's pool (the default pool if the
// private one could not be created); freed with cudaFreeAsync.
static cudaError_t ws_alloc(void **p, size_t bytes, cudaStream_t s, int device) {
    cudaMemPool_t pool = lib_pool(device);
    return pool ? cudaMallocFromPoolAsync(p, bytes, pool, s) : cudaMallocAsync(p, bytes, s);
}

static ac_status check_device(int device, cudaDeviceProp *prop) {
    int count = 0;
    cudaError_t e = cudaGetDeviceCount(&count);
    if (e != cudaSuccess || count == 0) {
        set_error(std::string("no CUDA device: ") + cudaGetErrorString(e));
        cudaGetLastError();
        return AC_ERR_NO_DEVICE;
    }
    if (device < 0 || device >= count) {
        set_error("device index out of range");
        return AC_ERR_INVALID_ARG;
    }
    AC_CUDA(cudaGetDeviceProperties(prop, device), "cudaGetDeviceProperties");
    if (prop->major != 10) {
        set_error("libac is built for sm_100a only; device is sm_" + std::to_string(prop->major) +
                  std::to_string(prop->minor));
        return AC_ERR_NO_DEVICE;
    }
    return AC_OK;
}

// Shared memory left for STT rows by a staged variant (v >= 1) or by the
// global-only kernel (v == 0).
static size_t stt_budget(const ac_stt *h, int v) {
    const size_t fixed = (v ? staged_smem_bytes(staged_variant(v), 0) : 256) + 128;  // + static smem (k_rewalk: 64 B)
    return h->smem_optin > fixed ? h->smem_optin - fixed : 0;
}

static size_t row_bytes(const ac_stt *h) { return (size_t)h->host.row_stride * h->host.entry_bytes; }

// STT view for one launch: the rows a kernel stages are capped by its budget.
static SttView view_of(const ac_stt *h, int v) {
    SttView s;
    s.stt = h->d_stt;
    s.cmap = h->d_class_map;
    s.out_off = h->d_out_off;
    s.out_ids = h->d_out_ids;
    s.stride = h->host.row_stride;
    s.n_states = h->host.n_states;
    s.halo = h->host.maxlen ? h->host.maxlen - 1 : 0;
    s.info_col = h->host.info_col;
    s.c_dense = h->host.c_dense;
    s.c_row_bytes = 2 * h->host.c_dstride;
    s.c_sparse_x0 = h->host.c_sparse_off - 8u * h->host.c_dense;
    s.c_out_x0 = h->host.c_out_off - 8u * (h->host.c_dense - h->host.c_od);
    s.c_rec_bytes = 8;
    s.c_two = 2;
    s.c_mtwo = 0xFFFFFFFEu;
    s.c_half = 0x80000000u;
    s.c_k16 = 0x10000u;
    s.c_rep = 0x0101u;
    s.stt2 = v ? h->d_stt2 : nullptr;  // only the staged kernel walks two bytes per lookup
    s.stride2 = h->host.stride2;
    s.n_classes = h->host.n_classes;
    s.sblob = nullptr;
    s.cnt8 = 0;
    s.s_dense = s.s_rec = s.s_row_bytes = s.s_rec_x0 = 0;
    s.cmap_ident = 1;
    for (int b = 0; b < 256; b++) s.cmap_ident &= h->host.class_map[b] == b ? 1u : 0u;
    if (h->tier == AC_TIER_SPLIT) {
        // the staged kernel stages the split blob; the global-only kernel
        // (head/tail chains, short texts, re-walks) reads the global table
        s.smem_rows = 0;
        s.smem_bytes = 0;
        if (v && h->host.split.size() <= stt_budget(h, v)) {
            s.sblob = h->d_split;
            s.smem_bytes = (uint32_t)h->host.split.size();
            s.s_dense = h->host.s_dense;
            s.s_rec = h->host.s_rec;
            s.s_row_bytes = 2 * h->host.s_dstride;
            // records follow the dense rows + escape row; record of id s at s_rec_x0 + 8 s
            s.s_rec_x0 = (s.s_dense + 1) * s.s_row_bytes - 8u * s.s_dense;
        }
        return s;
    }
    if (h->tier == AC_TIER_COMPACT) {
        s.smem_rows = h->host.n_states;
        s.smem_bytes = (uint32_t)h->host.compact.size();
        return s;
    }
    uint64_t rows = h->tier == AC_TIER_GLOBAL ? 0 : h->hot_rows;
    const uint64_t cap = stt_budget(h, v) / row_bytes(h);
    s.smem_rows = (uint32_t)(rows < cap ? rows : cap);
    s.smem_bytes = (uint32_t)(s.smem_rows * row_bytes(h));
    if (h->tier == AC_TIER_GLOBAL && h->d_cnt8 && v && h->host.n_states <= stt_budget(h, v)) {
        // the staged kernel keeps every state's output count in shared memory
        s.sblob = h->d_cnt8;
        s.smem_bytes = h->host.n_states;
        s.cnt8 = 1;
    }
    return s;
}

static size_t smem_of(const ac_stt *, const SttView &v) { return ((size_t)v.smem_bytes + 15) / 16 * 16; }

// The kernel's tier: SMEM only when every row is resident, GLOBAL when none.
static uint32_t tier_of(const ac_stt *h, const SttView &v) {
    if (h->tier == AC_TIER_COMPACT) return AC_TIER_COMPACT;
    if (h->tier == AC_TIER_SPLIT) return v.sblob ? AC_TIER_SPLIT : AC_TIER_GLOBAL;
    if (v.smem_rows == 0) return AC_TIER_GLOBAL;
    if (v.smem_rows >= h->host.n_states) return AC_TIER_SMEM;
    return AC_TIER_HYBRID;
}

static void free_device(ac_stt *h) {
    cudaFree(h->d_stt);
    cudaFree(h->d_stt2);
    h->d_stt2 = nullptr;
    cudaFree(h->d_split);
    h->d_split = nullptr;
    cudaFree(h->d_cnt8);
    h->d_cnt8 = nullptr;
    cudaFree(h->d_class_map);
    cudaFree(h->d_out_off);
    cudaFree(h->d_out_ids);
    cudaFree(h->d_lens);
    h->d_stt = nullptr;
    h->d_class_map = nullptr;
    h->d_out_off = h->d_out_ids = h->d_lens = nullptr;
}

// ------------------------------------------------------------- the scan
static ac_status match_async(const ac_stt *h, const uint8_t *d_text, uint64_t n_owned, uint64_t n_halo,
                             uint64_t base, ac_match_t *d_out, uint64_t cap, ac_result *d_res, cudaStream_t stream,
                             const ac_match_opts *opts) {
    NvtxRange range(d_out ? "ac_match(list)" : "ac_match(count)");
    g_launches = 0;
    g_scratch_rec = 0;
    if (!h || !d_res || (!d_text && n_owned + n_halo > 0)) {
        set_error("NULL stt, result or text");
        return AC_ERR_INVALID_ARG;
    }
    if (opts && opts->struct_size != sizeof(ac_match_opts)) {
        set_error("ac_match_opts.struct_size mismatch");
        return AC_ERR_INVALID_ARG;
    }
    const uint64_t n_total = n_owned + n_halo;
    if (n_total < n_owned || n_total >= AC_MAX_TEXT || base + n_total >= AC_MAX_TEXT) {
        set_error("text too large (n >= 2^40)");
        return AC_ERR_TOO_LARGE;
    }
    uint32_t kernel = opts ? opts->kernel : AC_KERNEL_AUTO;
    if (opts && (opts->text_policy > 3 || opts->text_promotion > 4)) {
        set_error("text_policy must be 0..3 and text_promotion 0..4");
        return AC_ERR_INVALID_ARG;
    }
    if (kernel > AC_KERNEL_GLOBAL) {
        set_error("unknown kernel");
        return AC_ERR_INVALID_ARG;
    }
    const bool emit = d_out != nullptr;
    void **ev = opts ? opts->events : nullptr;
    const uint32_t nev = opts ? opts->n_events : 0;
    // per-launch timing events go on the stream the kernel runs on
    auto pre = [&](cudaStream_t on) {
        if (ev && g_launches < nev) cudaEventRecord(static_cast<cudaEvent_t>(ev[2 * g_launches]), on);
    };
    auto post = [&](const char *name, cudaStream_t on, uint64_t text_bytes) {
        if (ev && g_launches < nev) cudaEventRecord(static_cast<cudaEvent_t>(ev[2 * g_launches + 1]), on);
        if (g_launches < 16) {
            g_names[g_launches] = name;
            g_bytes[g_launches] = text_bytes;
        }
        g_launches++;
    };
    AC_CUDA(cudaMemsetAsync(d_res, 0, sizeof(ac_result), stream), "memset result");
    if (n_owned == 0 || h->host.n_patterns == 0) return AC_OK;

    const uint32_t eb = h->host.entry_bytes;
    // chain counters are 32-bit in the kernels: chain bytes x max|output| < 2^31
    const uint64_t count_lim = h->host.max_out ? (1ull << 31) / h->host.max_out : UINT64_MAX;
    const uint64_t req_chain = opts ? opts->chain_bytes : 0;
    if (kernel == AC_KERNEL_AUTO) kernel = n_owned >= kStagedMinBytes ? AC_KERNEL_STAGED : AC_KERNEL_GLOBAL;
    int variant = opts ? (int)opts->variant : 0;
    if (variant < 0 || variant > staged_variant_count()) {
        set_error("unknown staged variant");
        return AC_ERR_INVALID_ARG;
    }
    if (variant == 0) {
        variant = kAutoVariant;
        if (h->tier == AC_TIER_COMPACT) variant = kCompactVariant;
        if (h->tier == AC_TIER_SPLIT) variant = kSplitVariant;
    }
    if (h->tier == AC_TIER_COMPACT && h->host.compact.size() > stt_budget(h, variant)) {
        set_error("staged variant " + std::to_string(variant) + " has no room for the COMPACT table");
        return AC_ERR_INVALID_ARG;
    }
    SttView sg = view_of(h, 0), ss = view_of(h, variant);
    // the two-byte walk exists for the two 32-warp x 16-byte shapes only
    if ((opts && opts->stride == 1) || (variant != 4 && variant != 7)) ss.stt2 = nullptr;
    const uint32_t tier_g = tier_of(h, sg), tier_s = tier_of(h, ss);
    // l2_window_mib > 0: persisting L2 window over that many MiB of the
    // global table (tiers that read it: GLOBAL, HYBRID, SPLIT), capped by the
    // device's persisting L2 limit, which the first such call raises
    size_t win_bytes = 0;
    if (opts && opts->l2_window_mib && tier_s != AC_TIER_SMEM && tier_s != AC_TIER_COMPACT) {
        size_t lim = 0;
        if (cudaDeviceGetLimit(&lim, cudaLimitPersistingL2CacheSize) == cudaSuccess && lim == 0) {
            cudaDeviceProp pr;
            if (cudaGetDeviceProperties(&pr, h->device) == cudaSuccess)
                cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, (size_t)pr.persistingL2CacheMaxSize);
            cudaDeviceGetLimit(&lim, cudaLimitPersistingL2CacheSize);
        }
        cudaGetLastError();
        const size_t tbl = (size_t)h->host.n_states * row_bytes(h);
        win_bytes = std::min<size_t>({(size_t)opts->l2_window_mib << 20, tbl, lim});
    }
    const size_t smem_g = smem_of(h, sg), smem_s = smem_of(h, ss);
    const StagedConfig cfg = staged_variant(variant);

    // --- geometry: [head | main (staged) | tail] or a single global region
    Region ra{0, 0, kGlobalTailChain, 0, 0}, rb{0, 0, kGlobalTailChain, 0, 0};
    StagedGeom g{0, 0, 0, 0, 0, 0};
    CUtensorMap tmap;
    if (kernel == AC_KERNEL_STAGED) {
        const uint64_t W = (uint64_t)cfg.width, R = (uint64_t)cfg.warps * 32 * cfg.k;
        uint64_t head = (16 - (reinterpret_cast<uintptr_t>(d_text) & 15)) & 15;
        if (head > n_owned) head = n_owned;
        const uint64_t avail = n_owned - head;
        uint64_t L;
        if (req_chain) {
            L = (req_chain + W - 1) / W * W;
        } else {
            const uint64_t target = (uint64_t)h->num_sms * R;
            L = (avail + target - 1) / target;
            // list mode, single pass: keep the expected records per chain
            // (the capacity read as a density bound) within half a scratch
            // slot -- on long texts one chain per lane would overflow every
            // slot into k_rewalk (C5 English 1K at 16 GiB: 32K records per
            // chain); shorter chains just take more CTA waves (ticketed tiles)
            // (whole waves: L is re-divided so every wave is full)
            if (emit && cap > 0 && cap <= n_owned) {
                const uint64_t lmax = (kMaxSlots / 2) * (n_owned / cap);
                if (L > lmax) {
                    const uint64_t waves = (L + lmax - 1) / lmax;
                    L = (avail + waves * target - 1) / (waves * target);
                }
            }
            L = (L + W - 1) / W * W;
            if (L < kStagedMinChain) L = kStagedMinChain;
        }
        if (L > (1ull << 30)) L = (1ull << 30) / W * W;
        if (L > count_lim) L = std::max<uint64_t>(W, count_lim / W * W);
        uint64_t n_main = avail / L;
        if (n_main > (1ull << 31) - R) n_main = ((1ull << 31) - R);
        ra = Region{0, head, kGlobalTailChain, (head + kGlobalTailChain - 1) / kGlobalTailChain, 0};
        if (n_main > 0) {
            g.m0 = head;
            g.chain_len = L;
            g.n_chains = n_main;
            g.chain0 = ra.n_chains;
            g.n_readable = n_total - head;
            const uint32_t tp = opts ? opts->text_policy : 0;
            g.text_evict_first =
                tp ? tp - 1u
                   : (tier_s == AC_TIER_GLOBAL || tier_s == AC_TIER_HYBRID || tier_s == AC_TIER_SPLIT) ? 1u : 0u;
            PFN_cuTensorMapEncodeTiled_v12000 enc = encode_fn();
            if (!enc) {
                set_error("cuTensorMapEncodeTiled unavailable from the driver");
                return AC_ERR_CUDA;
            }
            cuuint64_t dims[2] = {(cuuint64_t)L, (cuuint64_t)n_main};
            cuuint64_t strides[1] = {(cuuint64_t)L};
            cuuint32_t box[2] = {(cuuint32_t)W, (cuuint32_t)(32 * cfg.k)};
            cuuint32_t estr[2] = {1, 1};
            const CUtensorMapSwizzle swz = !cfg.swizzle ? CU_TENSOR_MAP_SWIZZLE_NONE
                                           : W == 128 ? CU_TENSOR_MAP_SWIZZLE_128B
                                           : W == 64 ? CU_TENSOR_MAP_SWIZZLE_64B
                                           : W == 32 ? CU_TENSOR_MAP_SWIZZLE_32B
                                                     : CU_TENSOR_MAP_SWIZZLE_NONE;
            const uint32_t pr = opts ? opts->text_promotion : 0;
            const CUtensorMapL2promotion promo = pr == 1   ? CU_TENSOR_MAP_L2_PROMOTION_NONE
                                                 : pr == 2 ? CU_TENSOR_MAP_L2_PROMOTION_L2_64B
                                                 : pr == 3 ? CU_TENSOR_MAP_L2_PROMOTION_L2_128B
                                                           : CU_TENSOR_MAP_L2_PROMOTION_L2_256B;
            CUresult cr = enc(&tmap, CU_TENSOR_MAP_DATA_TYPE_UINT8, 2, (void *)(d_text + head), dims, strides, box,
                              estr, CU_TENSOR_MAP_INTERLEAVE_NONE, swz, promo, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
            if (cr != CUDA_SUCCESS) {
                set_error("cuTensorMapEncodeTiled failed with CUresult " + std::to_string((int)cr));
                return AC_ERR_CUDA;
            }
        }
        const uint64_t tail_lo = head + n_main * L;
        rb = Region{tail_lo, n_owned, kGlobalTailChain,
                    (n_owned - tail_lo + kGlobalTailChain - 1) / kGlobalTailChain, ra.n_chains + n_main};
    } else {
        uint64_t L = req_chain;
        if (!L) {
            L = (n_owned + (uint64_t)h->num_sms * 1024 - 1) / ((uint64_t)h->num_sms * 1024);
            L = (L + 15) / 16 * 16;
            if (L < 64) L = 64;
        }
        if (L > count_lim) {
            L = std::max<uint64_t>(1, count_lim);
        }
        ra = Region{0, n_owned, L, (n_owned + L - 1) / L, 0};
    }
    const uint64_t n_chains = ra.n_chains + g.n_chains + rb.n_chains;
    const bool any_global = ra.n_chains + rb.n_chains > 0;

    ScanOut so{};
    so.base = base;
    so.res = d_res;
    so.out = reinterpret_cast<uint64_t *>(d_out);
    // The few head/tail chains (global kernel) are latency bound: when a
    // staged main region exists they run concurrently on a side stream
    // (event fork/join, capturable in a CUDA graph).
    SideStream *side = nullptr;
    if (any_global && g.n_chains) {
        ac_status rc = side_stream(h->device, &side);
        if (rc != AC_OK) return rc;
    }
    uint32_t nm_bits = 0;  // narrow scratch records in the staged kernel (list mode, set below)
    auto scan = [&](int mode, const char *gname, const char *sname) -> ac_status {
        if (any_global) {
            cudaStream_t gs = stream;
            if (side) {
                AC_CUDA(cudaEventRecord(side->fork, stream), "cudaEventRecord(fork)");
                AC_CUDA(cudaStreamWaitEvent(side->stream, side->fork, 0), "cudaStreamWaitEvent(fork)");
                gs = side->stream;
            }
            pre(gs);
            AC_CUDA(launch_scan_global(mode, eb, tier_g, d_text, n_total, sg, ra, rb, so, smem_g, gs), gname);
            post(gname, gs, (ra.hi - ra.lo) + (rb.hi - rb.lo));
            if (side) AC_CUDA(cudaEventRecord(side->join, side->stream), "cudaEventRecord(join)");
        }
        if (g.n_chains) {
            pre(stream);
            ScanOut sso = so;
            if (mode == MODE_EMIT_OPT) sso.nbits = nm_bits;
            // optional L2 access-policy window (SURVEY 8(a)-a5 tier (iii)) over
            // the hottest rows of the global table (BFS order: shallow rows
            // first), set on the stream for this launch only
            const bool apw = win_bytes > 0;
            if (apw) {
                cudaStreamAttrValue v = {};
                v.accessPolicyWindow.base_ptr = h->d_stt;
                v.accessPolicyWindow.num_bytes = win_bytes;
                v.accessPolicyWindow.hitRatio = 1.0f;
                v.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
                v.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
                AC_CUDA(cudaStreamSetAttribute(stream, cudaStreamAttributeAccessPolicyWindow, &v),
                        "cudaStreamSetAttribute(access policy window)");
            }
            const cudaError_t le =
                launch_scan_staged(mode, eb, tier_s, variant, tmap, d_text + g.m0, ss, g, sso, smem_s, stream);
            if (apw) {
                cudaStreamAttrValue v = {};  // num_bytes = 0: the caller's later launches are unaffected
                cudaStreamSetAttribute(stream, cudaStreamAttributeAccessPolicyWindow, &v);
            }
            AC_CUDA(le, sname);
            post(sname, stream, g.n_chains * g.chain_len);
        }
        if (side) AC_CUDA(cudaStreamWaitEvent(stream, side->join, 0), "cudaStreamWaitEvent(join)");
        return AC_OK;
    };
    if (!emit) {
        so.total = reinterpret_cast<unsigned long long *>(&d_res->count);
        return scan(MODE_COUNT_TOTAL, "k_scan_global(count)", "k_scan_staged(count)");
    }
    // --- list mode workspace: counts | chain_end | list | tile_state | counters
    // Two passes (count, offsets, emit in place) for dense outputs (several
    // matches per byte), where every chain would overflow its scratch slot
    // into k_rewalk.  Measured (C5 English, 256 MiB): 20K patterns (2 per
    // byte) 13.6 -> 5.9 ms, 50K 70 -> 12 ms; the single pass stays better up
    // to ~1K records per chain (C2, 0.06 per byte: 0.51 vs 0.78 ms; 5K
    // patterns, 0.5 per byte: 2.96 vs 3.10 ms).  The capacity is read as the
    // caller's density bound: room for more than one record per owned text
    // byte selects the two-pass emission (no count pass is needed to plan).
    const bool dense_out = (!opts || (opts->two_pass == 0 && opts->scratch_slots == 0)) && cap > n_owned;
    // EVENTS (dense outputs): a single emitting pass that parks one event per
    // output state reached (an event per flagged byte, not a record per
    // match), so a slot of chain-length entries never overflows; k_gather
    // expands the events into records with coalesced, full-sector writes.
    // Needs a dense table whose rows carry the output summary k_gather reads
    // (every tier but COMPACT, whose states are renumbered) and state ids
    // below 2^24 (an event is start << 24 | state).
    // Measured (C5 English, 256 MiB, list): see DESIGN.md section 7.
    const uint64_t max_len = std::max<uint64_t>(g.n_chains ? g.chain_len : 0,
                                                std::max(ra.n_chains ? ra.chain_len : 0, rb.n_chains ? rb.chain_len : 0));
    const uint64_t max_ev_scratch = 32ull << 30;
    const bool ev_ok = (eb == 4 || h->tier != AC_TIER_COMPACT) && h->host.n_states < (1u << 24) && max_len > 0 &&
                       n_chains * max_len * 8 <= max_ev_scratch;
    bool events = ev_ok && ((opts && opts->two_pass == 4) || dense_out);
    bool two_pass = (opts && opts->two_pass == 1) || (dense_out && !events);
    // single pass: each chain keeps its first q records (or all its events)
    // in a scratch slot; if the slots cannot be allocated the call falls back
    // to two passes
    uint64_t q = opts && opts->scratch_slots ? opts->scratch_slots : 4 * (cap / n_chains) + 64;
    if (q > kMaxSlots) q = kMaxSlots;
    const uint64_t max_scratch = 8ull << 30;
    if (n_chains * q * 8 > max_scratch) q = max_scratch / (n_chains * 8);
    // a scratch budget too small for twice the expected records per chain
    // would send most chains to k_rewalk (C5 English 1K at 16 GiB, 4.8 G
    // records: 380 slots for ~1.7 K records per chain): two passes instead
    if (!events && !two_pass && (!opts || (opts->two_pass == 0 && opts->scratch_slots == 0)) &&
        q < 2 * (cap / n_chains))
        two_pass = true;
    if (events) q = max_len;
    if (q == 0) q = 1;
    void *scratch = nullptr;
    if (!two_pass) {
        cudaError_t e = ws_alloc(&scratch, n_chains * q * 8, stream, h->device);
        if (e != cudaSuccess) {
            cudaGetLastError();
            scratch = nullptr;
            two_pass = true;
            events = false;
        }
    }
    // in-kernel offsets: the staged kernel places its chains (decoupled
    // look-back per CTA) when the main region starts the list and the tail
    // is short; k_gather places the tail.  two_pass = 2 forces k_offsets.
    const bool place = !two_pass && !(opts && opts->two_pass == 2) && g.n_chains > 0 && ra.n_chains == 0 &&
                       rb.n_chains <= 256;
    const uint64_t R = (uint64_t)cfg.warps * 32 * cfg.k;
    const uint64_t n_lb = place ? (g.n_chains + R - 1) / R : 0;  // staged CTAs
    const size_t tiles = offsets_tiles(n_chains);
    const size_t bytes = n_chains * 8 * 3 + tiles * 8 + 16 + n_lb * 8 + (events ? n_chains * 4 : 0);
    void *ws = nullptr;
    {
        cudaError_t e = ws_alloc(&ws, bytes, stream, h->device);
        if (e != cudaSuccess) {
            if (scratch) cudaFreeAsync(scratch, stream);
            return cuda_fail(e, "cudaMallocAsync(workspace)");
        }
    }
    uint64_t *counts = static_cast<uint64_t *>(ws);
    uint64_t *chain_end = counts + n_chains;
    uint64_t *list = chain_end + n_chains;
    uint64_t *tile_state = list + n_chains;
    unsigned int *counter = reinterpret_cast<unsigned int *>(tile_state + tiles);
    unsigned int *list_n = counter + 1;
    unsigned long long *lb = place ? reinterpret_cast<unsigned long long *>(counter + 4) : nullptr;
    uint32_t *chain_events = events ? reinterpret_cast<uint32_t *>(counter + 4 + 2 * n_lb) : nullptr;
    so.chain_events = chain_events;
    so.tile_state = lb;
    so.ticket = place ? counter + 2 : nullptr;
    so.chain_end_w = chain_end;
    TailPlace tp{lb, n_lb, rb.chain0, rb.n_chains, cap};
    // narrow scratch records for the staged kernel's deferred emission (one
    // chain per lane, 16-bit table, one byte per lookup): offset in chain and
    // pattern id must share 32 bits.  Off for the two-pass ablation.
    NarrowMain nm{0, g.chain0, g.n_chains, base + g.m0, g.chain_len};
    if (!two_pass && !events && g.n_chains && cfg.k == 1 && eb == 2 && !ss.stt2 && !(opts && opts->two_pass == 3)) {
        uint32_t pid_bits = 1, off_bits = 1;
        while ((1ull << pid_bits) < h->host.n_patterns) pid_bits++;
        while ((1ull << off_bits) < g.chain_len) off_bits++;
        if (pid_bits + off_bits <= 32) nm.nbits = pid_bits;
    }
    nm_bits = nm.nbits;
    g_scratch_rec = two_pass ? 0u : nm.nbits ? 4u : 8u;
    const EventExpand evx{chain_events, h->d_stt,       h->host.row_stride, h->host.info_col,
                          eb,           h->d_out_off, h->d_out_ids};
    so.chain_counts = counts;
    so.chain_end = chain_end;
    if (scratch) {
        so.scratch = static_cast<uint64_t *>(scratch);
        so.q = (uint32_t)q;
    }
    auto run = [&]() -> ac_status {
        AC_CUDA(cudaMemsetAsync(tile_state, 0, tiles * 8 + 16 + n_lb * 8, stream), "memset workspace");
        if (two_pass) {
            ac_status rc = scan(MODE_COUNT_CHAINS, "k_scan_global(count)", "k_scan_staged(count)");
            if (rc != AC_OK) return rc;
            pre(stream);
            AC_CUDA(launch_offsets(counts, n_chains, chain_end, tile_state, counter, d_res, cap, 1, stream),
                    "k_offsets");
            post("k_offsets", stream, 0);
            return scan(MODE_EMIT, "k_scan_global(emit)", "k_scan_staged(emit)");
        }
        ac_status rc = scan(MODE_EMIT_OPT, "k_scan_global(emit1)", "k_scan_staged(emit1)");
        if (rc != AC_OK) return rc;
        if (!place) {
            pre(stream);
            AC_CUDA(launch_offsets(counts, n_chains, chain_end, tile_state, counter, d_res, cap, 1, stream),
                    "k_offsets");
            post("k_offsets", stream, 0);
        }
        pre(stream);
        AC_CUDA(launch_gather(counts, chain_end, n_chains, so.scratch, so.q, so.out, d_res, list, list_n, tp, nm, evx,
                              h->num_sms, stream),
                "k_gather");
        post("k_gather", stream, 0);
        pre(stream);
        AC_CUDA(launch_rewalk(eb, tier_g, d_text, n_total, sg, ra, rb, g, so, list, list_n, smem_g, h->num_sms,
                              stream),
                "k_rewalk");
        post("k_rewalk", stream, 0);
        return AC_OK;
    };
    const ac_status rc = run();
    if (scratch) cudaFreeAsync(scratch, stream);
    cudaFreeAsync(ws, stream);
    return rc;
}

// Packet batches (NEXT-2): independent segments, two passes (count, offsets,
// emit) over one thread per segment.
static ac_status match_segments(const ac_stt *h, const uint8_t *d_text, const uint64_t *d_seg_off, uint64_t n_seg,
                                ac_match_t *d_out, uint64_t cap, ac_result *d_res, cudaStream_t stream) {
    g_launches = 0;
    if (!h || !d_res || (n_seg && (!d_seg_off || !d_text))) {
        set_error("NULL stt, result, text or segment offsets");
        return AC_ERR_INVALID_ARG;
    }
    AC_CUDA(cudaMemsetAsync(d_res, 0, sizeof(ac_result), stream), "memset result");
    if (n_seg == 0 || h->host.n_patterns == 0) return AC_OK;
    const SttView sg = view_of(h, 0);
    const uint32_t tier = tier_of(h, sg), eb = h->host.entry_bytes;
    const size_t smem = smem_of(h, sg);
    ScanOut so{};
    so.res = d_res;
    so.out = reinterpret_cast<uint64_t *>(d_out);
    auto note = [&](const char *name) {
        if (g_launches < 16) {
            g_names[g_launches] = name;
            g_bytes[g_launches] = 0;
        }
        g_launches++;
    };
    if (!d_out) {
        so.total = reinterpret_cast<unsigned long long *>(&d_res->count);
        AC_CUDA(launch_segments(MODE_COUNT_TOTAL, eb, tier, d_text, d_seg_off, n_seg, sg, so, smem, stream),
                "k_scan_segments(count)");
        note("k_scan_segments(count)");
        return AC_OK;
    }
    const size_t tiles = offsets_tiles(n_seg);
    void *ws = nullptr;
    AC_CUDA(ws_alloc(&ws, n_seg * 16 + tiles * 8 + 16, stream, h->device), "cudaMallocAsync(workspace)");
    uint64_t *counts = static_cast<uint64_t *>(ws);
    uint64_t *chain_end = counts + n_seg;
    uint64_t *tile_state = chain_end + n_seg;
    unsigned int *counter = reinterpret_cast<unsigned int *>(tile_state + tiles);
    so.chain_counts = counts;
    so.chain_end = chain_end;
    auto run = [&]() -> ac_status {
        AC_CUDA(cudaMemsetAsync(tile_state, 0, tiles * 8 + 16, stream), "memset workspace");
        AC_CUDA(launch_segments(MODE_COUNT_CHAINS, eb, tier, d_text, d_seg_off, n_seg, sg, so, smem, stream),
                "k_scan_segments(count)");
        note("k_scan_segments(count)");
        AC_CUDA(launch_offsets(counts, n_seg, chain_end, tile_state, counter, d_res, cap, 1, stream), "k_offsets");
        note("k_offsets");
        AC_CUDA(launch_segments(MODE_EMIT, eb, tier, d_text, d_seg_off, n_seg, sg, so, smem, stream),
                "k_scan_segments(emit)");
        note("k_scan_segments(emit)");
        return AC_OK;
    };
    const ac_status rc = run();
    cudaFreeAsync(ws, stream);
    return rc;
}

static ac_status finish_sync(ac_result *d_res, uint64_t *count, cudaStream_t stream) {
    ac_result hres;
    AC_CUDA(cudaMemcpyAsync(&hres, d_res, sizeof(hres), cudaMemcpyDeviceToHost, stream), "D2H result");
    AC_CUDA(cudaStreamSynchronize(stream), "cudaStreamSynchronize");
    if (count) *count = hres.count;
    if (hres.status != AC_OK) {
        set_error("match list longer than cap (" + std::to_string(hres.count) + " records needed)");
        return (ac_status)hres.status;
    }
    return AC_OK;
}

// ------------------------------------------------- host-buffer pipeline
// the text is cut into chunks (shards with halos, the
// same ownership rule as a1); H2D of chunk i+2 (copy stream) overlaps the
// scan of chunk i (caller stream) and the D2H of chunk i-1's records (second
// copy stream).  Each chunk's list lands at the running offset, so the host
// list is the global canonical list.
struct HostPipe {
    cudaStream_t h2d = nullptr, d2h = nullptr;
    cudaEvent_t loaded[2] = {nullptr, nullptr}, freed[2] = {nullptr, nullptr}, done[2] = {nullptr, nullptr};
    ac_result *pinned = nullptr;  // kMaxChunks results
};
static const uint64_t kMaxChunks = 4096, kChunk = 32ull << 20;

static ac_status host_pipe(int device, HostPipe **out) {
    static thread_local HostPipe per_dev[64];
    if (device < 0 || device >= 64) {
        set_error("device index out of range");
        return AC_ERR_INVALID_ARG;
    }
    HostPipe &p = per_dev[device];
    if (!p.h2d) {
        cudaError_t e = cudaStreamCreateWithFlags(&p.h2d, cudaStreamNonBlocking);
        if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&p.d2h, cudaStreamNonBlocking);
        for (int i = 0; i < 2 && e == cudaSuccess; i++) {
            e = cudaEventCreateWithFlags(&p.loaded[i], cudaEventDisableTiming);
            if (e == cudaSuccess) e = cudaEventCreateWithFlags(&p.freed[i], cudaEventDisableTiming);
            if (e == cudaSuccess) e = cudaEventCreateWithFlags(&p.done[i], cudaEventDisableTiming);
        }
        if (e == cudaSuccess) e = cudaHostAlloc(&p.pinned, kMaxChunks * sizeof(ac_result), cudaHostAllocDefault);
        if (e != cudaSuccess) {
            p.h2d = nullptr;
            return cuda_fail(e, "host pipeline setup");
        }
    }
    *out = &p;
    return AC_OK;
}

static ac_status match_host_pipelined(const ac_stt *stt, const uint8_t *h_text, uint64_t n, ac_match_t *h_out,
                                      uint64_t cap, uint64_t *count, cudaStream_t s) {
    NvtxRange range("ac_match_host");
    int prev = -1;
    cudaGetDevice(&prev);
    AC_CUDA(cudaSetDevice(stt->device), "cudaSetDevice");
    struct Restore {
        int d;
        ~Restore() {
            if (d >= 0) cudaSetDevice(d);
        }
    } restore{prev};
    HostPipe *P = nullptr;
    ac_status rc = host_pipe(stt->device, &P);
    if (rc != AC_OK) return rc;
    const uint64_t H = stt->host.maxlen ? stt->host.maxlen - 1 : 0;
    uint64_t CH = kChunk;
    if (n / CH + 1 > kMaxChunks) CH = (n / (kMaxChunks - 1) + 16) / 16 * 16;
    const uint64_t nch = n ? (n + CH - 1) / CH : 1;
    const bool emit = h_out != nullptr;
    uint8_t *tb[2] = {nullptr, nullptr};
    ac_match_t *d_out = nullptr;
    ac_result *d_res = nullptr;
    auto cleanup = [&]() {
        // the copy streams still read d_out / the text buffers: drain them
        // before the frees are enqueued (stream-ordered reuse is per stream)
        cudaStreamSynchronize(P->d2h);
        cudaStreamSynchronize(P->h2d);
        for (auto &b : tb)
            if (b) cudaFreeAsync(b, s);
        if (d_out) cudaFreeAsync(d_out, s);
        if (d_res) cudaFreeAsync(d_res, s);
        cudaStreamSynchronize(s);
    };
    cudaError_t e = ws_alloc(reinterpret_cast<void **>(&d_res), nch * sizeof(ac_result), s, stt->device);
    for (int b = 0; b < 2 && e == cudaSuccess && n; b++)
        e = ws_alloc(reinterpret_cast<void **>(&tb[b]), CH + H + 16, s, stt->device);
    if (e == cudaSuccess && emit)
        e = ws_alloc(reinterpret_cast<void **>(&d_out), (cap ? cap : 1) * sizeof(ac_match_t), s, stt->device);
    // the copy streams must see the allocations
    if (e == cudaSuccess) e = cudaEventRecord(P->freed[0], s);
    if (e == cudaSuccess) e = cudaEventRecord(P->freed[1], s);
    if (e != cudaSuccess) {
        cleanup();
        return cuda_fail(e, "host pipeline buffers");
    }
    auto lo_of = [&](uint64_t i) { return i * CH; };
    auto own_of = [&](uint64_t i) { return std::min(CH, n - lo_of(i)); };
    auto halo_of = [&](uint64_t i) { return std::min(H, n - lo_of(i) - own_of(i)); };
    auto issue_h2d = [&](uint64_t j) -> cudaError_t {
        const int b = (int)(j & 1);
        cudaError_t err = cudaStreamWaitEvent(P->h2d, P->freed[b], 0);
        if (err == cudaSuccess)
            err = cudaMemcpyAsync(tb[b], h_text + lo_of(j), own_of(j) + halo_of(j), cudaMemcpyHostToDevice, P->h2d);
        if (err == cudaSuccess) err = cudaEventRecord(P->loaded[b], P->h2d);
        return err;
    };
    uint64_t off = 0;
    bool over = false;
    auto collect = [&](uint64_t i) -> ac_status {  // chunk i's count is needed on the host
        AC_CUDA(cudaEventSynchronize(P->done[i & 1]), "cudaEventSynchronize");
        const ac_result r = P->pinned[i];
        if (r.status == AC_ERR_CAPACITY) over = true;
        if (emit && !over && r.count)
            AC_CUDA(cudaMemcpyAsync(h_out + off, d_out + off, r.count * sizeof(ac_match_t), cudaMemcpyDeviceToHost,
                                    P->d2h),
                    "D2H matches");
        off += r.count;
        if (emit && off > cap) over = true;
        return AC_OK;
    };
    if (n) {
        for (uint64_t j = 0; j < 2 && j < nch; j++) AC_CUDA(issue_h2d(j), "H2D text");
    }
    for (uint64_t i = 0; i < nch; i++) {
        if (i > 0) {
            rc = collect(i - 1);
            if (rc != AC_OK) break;
        }
        const int b = (int)(i & 1);
        if (n) AC_CUDA(cudaStreamWaitEvent(s, P->loaded[b], 0), "cudaStreamWaitEvent");
        ac_match_t *dst = (emit && !over) ? d_out + off : nullptr;
        rc = ac_match_async(stt, n ? tb[b] : nullptr, n ? own_of(i) : 0, n ? halo_of(i) : 0, lo_of(i), dst,
                            (emit && !over) ? cap - off : 0, d_res + i, s, nullptr);
        if (rc != AC_OK) break;
        AC_CUDA(cudaEventRecord(P->freed[b], s), "cudaEventRecord");
        AC_CUDA(cudaMemcpyAsync(&P->pinned[i], d_res + i, sizeof(ac_result), cudaMemcpyDeviceToHost, s), "D2H result");
        AC_CUDA(cudaEventRecord(P->done[b], s), "cudaEventRecord");
        if (n && i + 2 < nch) AC_CUDA(issue_h2d(i + 2), "H2D text");
    }
    if (rc == AC_OK) rc = collect(nch - 1);
    cleanup();
    if (rc != AC_OK) return rc;
    if (count) *count = off;
    if (emit && (over || off > cap)) {
        set_error("match list longer than cap (" + std::to_string(off) + " records needed)");
        return AC_ERR_CAPACITY;
    }
    return AC_OK;
}

}  // namespace acx

using namespace acx;

extern "C" {

const char *ac_status_string(ac_status s) {
    switch (s) {
        case AC_OK: return "AC_OK";
        case AC_ERR_INVALID_ARG: return "AC_ERR_INVALID_ARG";
        case AC_ERR_EMPTY_PATTERN: return "AC_ERR_EMPTY_PATTERN";
        case AC_ERR_TOO_LARGE: return "AC_ERR_TOO_LARGE";
        case AC_ERR_CAPACITY: return "AC_ERR_CAPACITY";
        case AC_ERR_NO_MEMORY: return "AC_ERR_NO_MEMORY";
        case AC_ERR_CUDA: return "AC_ERR_CUDA";
        case AC_ERR_NO_DEVICE: return "AC_ERR_NO_DEVICE";
    }
    return "AC_ERR_UNKNOWN";
}

const char *ac_last_error(void) { return g_err.c_str(); }
const char *ac_version(void) { return "libac 0.1 sm_100a (TMA-staged + global-only scans)"; }
uint32_t ac_last_launch_count(void) { return g_launches; }
uint32_t ac_last_scratch_record_bytes(void) { return g_scratch_rec; }
const char *ac_last_launch_name(uint32_t i) { return i < g_launches && i < 16 ? g_names[i] : nullptr; }
uint64_t ac_last_launch_text_bytes(uint32_t i) { return i < g_launches && i < 16 ? g_bytes[i] : 0; }

ac_status ac_compile(const uint8_t *const *patterns, const uint32_t *lens, uint32_t n, const ac_build_opts *opts,
                     ac_table **out) {
    if (!out) {
        set_error("out is NULL");
        return AC_ERR_INVALID_ARG;
    }
    *out = nullptr;
    if (opts && opts->struct_size != sizeof(ac_build_opts)) {
        set_error("ac_build_opts.struct_size mismatch");
        return AC_ERR_INVALID_ARG;
    }
    ac_table *t = new (std::nothrow) ac_table();
    if (!t) return AC_ERR_NO_MEMORY;
    ac_status rc;
    try {
        ac_build_opts o4;
        const bool split = opts && opts->tier == AC_TIER_SPLIT;
        if (split) {  // the SPLIT tier's global table has 32-bit entries
            o4 = *opts;
            o4.entry_bytes = 4;
        }
        rc = compile_table(patterns, lens, n, split ? &o4 : opts, *t);
        if (rc == AC_OK && split && !split_table(*t, kDefaultSplitBudget)) {
            set_error("the automaton has no SPLIT encoding for the default shared-memory budget");
            rc = AC_ERR_TOO_LARGE;
        }
        if (rc == AC_OK && opts && opts->tier == AC_TIER_COMPACT && !compact_table(*t, kDefaultCompactBudget)) {
            set_error("the automaton does not fit the COMPACT shared-memory encoding");
            rc = AC_ERR_TOO_LARGE;
        }
        if (rc == AC_OK && opts && opts->stride == 2 && !stride2_table(*t, 64ull << 20)) {
            set_error("stride 2 needs 32-bit entries and a two-byte table <= 64 MiB");
            rc = AC_ERR_INVALID_ARG;
        }
    } catch (...) {
        set_error("host allocation failed");
        rc = AC_ERR_NO_MEMORY;
    }
    if (rc != AC_OK) {
        delete t;
        return rc;
    }
    *out = t;
    return AC_OK;
}

static void fill_info(const ac_table &t, ac_stt_info *info) {
    std::memset(info, 0, sizeof(*info));
    info->n_patterns = t.n_patterns;
    info->n_states = t.n_states;
    info->n_classes = t.n_classes;
    info->row_stride = t.row_stride;
    info->entry_bytes = t.entry_bytes;
    info->maxlen = t.maxlen;
    info->forward = t.forward;
    info->info_col = t.info_col;
    info->stt_bytes = (uint64_t)t.n_states * t.row_stride * t.entry_bytes;
    info->out_entries = t.out_ids.size();
    info->compact_dense = t.c_dense;
    info->compact_od = t.c_od;
    info->compact_os = t.c_os;
    info->compact_dstride = t.c_dstride;
    info->compact_sparse_off = t.c_sparse_off;
    info->compact_out_off = t.c_out_off;
    info->compact_bytes = t.compact.size();
    info->stride = t.stride2 ? 2 : 1;
    info->stride2_cols = t.stride2;
    info->stt2_bytes = (uint64_t)t.stt2.size() * 4;
    info->split_dense = t.s_dense;
    info->split_records = t.s_rec;
    info->split_dstride = t.s_dstride;
    info->split_cold_records = t.s_cold_rec;
    info->split_bytes = t.split.size();
}

ac_status ac_table_export_split(const ac_table *t, void *blob) {
    if (!t || t->split.empty() || !blob) return AC_ERR_INVALID_ARG;
    std::memcpy(blob, t->split.data(), t->split.size());
    return AC_OK;
}

ac_status ac_table_export_stride2(const ac_table *t, uint32_t *tab) {
    if (!t || t->stt2.empty() || !tab) return AC_ERR_INVALID_ARG;
    std::memcpy(tab, t->stt2.data(), t->stt2.size() * 4);
    return AC_OK;
}

ac_status ac_table_export_compact(const ac_table *t, void *blob, uint32_t *perm) {
    if (!t || t->compact.empty()) return AC_ERR_INVALID_ARG;
    if (blob) std::memcpy(blob, t->compact.data(), t->compact.size());
    if (perm) std::memcpy(perm, t->c_perm.data(), t->c_perm.size() * 4);
    return AC_OK;
}

ac_status ac_table_query(const ac_table *t, ac_stt_info *info) {
    if (!t || !info) return AC_ERR_INVALID_ARG;
    fill_info(*t, info);
    return AC_OK;
}

ac_status ac_table_export(const ac_table *t, uint8_t *class_map, void *stt, uint32_t *out_off, uint32_t *out_ids) {
    if (!t) return AC_ERR_INVALID_ARG;
    if (class_map) std::memcpy(class_map, t->class_map, 256);
    if (stt && !t->stt.empty()) std::memcpy(stt, t->stt.data(), t->stt.size());
    if (out_off) std::memcpy(out_off, t->out_off.data(), t->out_off.size() * 4);
    if (out_ids && !t->out_ids.empty()) std::memcpy(out_ids, t->out_ids.data(), t->out_ids.size() * 4);
    return AC_OK;
}

void ac_table_free(ac_table *t) { delete t; }

ac_status ac_build(const uint8_t *const *patterns, const uint32_t *lens, uint32_t n, int device,
                   const ac_build_opts *opts, ac_stt **out) {
    if (!out) {
        set_error("out is NULL");
        return AC_ERR_INVALID_ARG;
    }
    *out = nullptr;
    if (opts && opts->struct_size != sizeof(ac_build_opts)) {
        set_error("ac_build_opts.struct_size mismatch");
        return AC_ERR_INVALID_ARG;
    }
    if (opts && opts->forward) {
        set_error("the device scan needs the reversed automaton (forward=0)");
        return AC_ERR_INVALID_ARG;
    }
    if (opts && opts->tier > AC_TIER_SPLIT) {
        set_error("unknown tier");
        return AC_ERR_INVALID_ARG;
    }
    NvtxRange range("ac_build");
    cudaDeviceProp prop;
    ac_status rc = check_device(device, &prop);
    if (rc != AC_OK) return rc;
    ac_stt *h = new (std::nothrow) ac_stt();
    if (!h) return AC_ERR_NO_MEMORY;
    ac_build_opts o4;
    if (opts && opts->tier == AC_TIER_SPLIT) {  // the SPLIT tier's global table has 32-bit entries
        o4 = *opts;
        o4.entry_bytes = 4;
        opts = &o4;
    }
    try {
        rc = compile_table(patterns, lens, n, opts, h->host);
    } catch (...) {
        rc = AC_ERR_NO_MEMORY;
    }
    if (rc != AC_OK) {
        delete h;
        return rc;
    }
    ac_table &t = h->host;
    if ((uint64_t)t.n_states * t.row_stride >= (1ull << 32)) {
        delete h;
        set_error("STT has >= 2^32 entries");
        return AC_ERR_TOO_LARGE;
    }
    h->device = device;
    h->num_sms = prop.multiProcessorCount;
    h->smem_optin = prop.sharedMemPerBlockOptin;
    // residency tier
    const size_t row_bytes = (size_t)t.row_stride * t.entry_bytes;
    const size_t stt_bytes = (size_t)t.n_states * row_bytes;
    const size_t budget = stt_budget(h, 1);  // a 48 KB-ring staged variant
    uint32_t tier = opts ? opts->tier : AC_TIER_AUTO;
    uint32_t hot = opts ? opts->hot_rows : 0;
    // measured (scripts/sweep.py): an L1-cached global table beats a shared-memory
    // prefix reached through generic loads, so AUTO never picks HYBRID
    const size_t cbudget = stt_budget(h, kLeanVariant);
    const uint32_t want_stride = opts ? opts->stride : 0;
    bool auto_split = false;
    if (tier == AC_TIER_AUTO) {
        if (stt_bytes <= budget) tier = AC_TIER_SMEM;
        else if (compact_table(h->host, cbudget)) tier = AC_TIER_COMPACT;
        // small alphabets (DNA): the L1/L2 table with two bytes per lookup
        else if (t.n_classes <= 8 && want_stride != 1 && t.entry_bytes == 4) tier = AC_TIER_GLOBAL;
        else tier = AC_TIER_SPLIT, auto_split = true;
    }
    if (tier == AC_TIER_SPLIT) {
        // the cold states need the 32-bit global table: build it if the
        // dictionary compiled to 16-bit entries
        ac_table t4;
        ac_table *ts = &h->host;
        if (t.entry_bytes != 4) {
            ac_build_opts o = opts ? *opts : ac_build_opts{sizeof(ac_build_opts), 0, 0, 0, 0, 0, 0};
            o.entry_bytes = 4;
            try {
                rc = compile_table(patterns, lens, n, &o, t4);
            } catch (...) {
                rc = AC_ERR_NO_MEMORY;
            }
            if (rc != AC_OK) {
                delete h;
                return rc;
            }
            ts = &t4;
        }
        const bool ok = split_table(*ts, stt_budget(h, kSplitVariant));
        // AUTO keeps SPLIT where the plain table would live in DRAM (> 32 MiB;
        // a table that fits L2 beside the streamed text is served well by
        // L1/L2: C5 Snort 1K, 15 MB: 0.43 ms GLOBAL vs 0.55 SPLIT per 256
        // MiB list) and the shared-memory part covers the hot automaton
        // (<= 30 % of the sparse hot states are cold records: Snort 50K, 46 %:
        // 1.12 GLOBAL vs 1.63 SPLIT; Snort 20K, 22 %: 1.00 vs 0.80; Snort 5K,
        // 4 %: 0.68 vs 0.59; C3, 7 %: 0.80 vs 0.66)
        const bool big = (uint64_t)ts->n_states * ts->row_stride * 4 > (32ull << 20);
        const bool good = ok && big && 10u * ts->s_cold_rec <= 3u * (ts->s_rec - ts->s_dense);
        if (auto_split && !good) {
            tier = AC_TIER_GLOBAL;
        } else if (!ok) {
            delete h;
            set_error("the automaton has no SPLIT encoding for the shared-memory budget");
            return AC_ERR_TOO_LARGE;
        } else {
            if (ts != &h->host) h->host = std::move(t4);
            hot = h->host.s_rec;
        }
    }
    if (tier == AC_TIER_COMPACT) {
        if (h->host.compact.empty() && !compact_table(h->host, cbudget)) {
            delete h;
            set_error("the automaton does not fit the COMPACT shared-memory encoding");
            return AC_ERR_TOO_LARGE;
        }
        hot = t.n_states;
    } else if (tier == AC_TIER_SMEM) {
        if (stt_bytes > budget) {
            delete h;
            set_error("STT (" + std::to_string(stt_bytes) + " B) does not fit shared memory (" +
                      std::to_string(budget) + " B)");
            return AC_ERR_TOO_LARGE;
        }
        hot = t.n_states;
    } else if (tier == AC_TIER_SPLIT) {
        // set above
    } else if (tier == AC_TIER_HYBRID) {
        uint32_t cap_rows = (uint32_t)(budget / row_bytes);
        if (hot == 0 || hot > cap_rows) hot = cap_rows;
        if (hot > t.n_states) hot = t.n_states;
        if (hot == 0) tier = AC_TIER_GLOBAL;
    } else {
        hot = 0;
    }
    h->tier = tier;
    h->hot_rows = hot;
    // NEXT-4: two bytes per lookup for small alphabets on the L1/L2 tier
    if (want_stride > 2) {
        delete h;
        set_error("stride must be 0, 1 or 2");
        return AC_ERR_INVALID_ARG;
    }
    if (want_stride == 2 || (want_stride == 0 && tier == AC_TIER_GLOBAL && t.n_classes <= 8)) {
        const bool ok = tier == AC_TIER_GLOBAL && stride2_table(h->host, 64ull << 20);
        if (!ok && want_stride == 2) {
            delete h;
            set_error("stride 2 needs the GLOBAL tier, 32-bit entries and a two-byte table <= 64 MiB");
            return AC_ERR_INVALID_ARG;
        }
    }

    int prev = -1;
    cudaGetDevice(&prev);
    auto fail = [&](cudaError_t e, const char *what) {
        free_device(h);
        delete h;
        if (prev >= 0) cudaSetDevice(prev);
        return e == cudaErrorMemoryAllocation ? (set_error(what), AC_ERR_NO_MEMORY) : cuda_fail(e, what);
    };
    cudaError_t e = cudaSetDevice(device);
    if (e != cudaSuccess) return fail(e, "cudaSetDevice");
    if (!t.split.empty() && tier == AC_TIER_SPLIT) {
        // staged in 16-byte words: the padding after the blob is zeroed too
        if ((e = cudaMalloc(&h->d_split, (t.split.size() + 15) / 16 * 16)) != cudaSuccess)
            return fail(e, "cudaMalloc(split)");
        if ((e = cudaMemset(h->d_split, 0, (t.split.size() + 15) / 16 * 16)) != cudaSuccess)
            return fail(e, "cudaMemset(split)");
        if ((e = cudaMemcpy(h->d_split, t.split.data(), t.split.size(), cudaMemcpyHostToDevice)) != cudaSuccess)
            return fail(e, "H2D split");
    }
    if (tier == AC_TIER_GLOBAL && t.entry_bytes == 4) {
        // per-state output counts for the staged GLOBAL scan (view_of)
        std::vector<uint8_t> c8((t.n_states + 15) / 16 * 16, 0);
        for (uint32_t x = 0; x < t.n_states; x++)
            c8[x] = (uint8_t)std::min<uint32_t>(t.out_off[x + 1] - t.out_off[x], 255u);
        if ((e = cudaMalloc(&h->d_cnt8, c8.size())) != cudaSuccess) return fail(e, "cudaMalloc(cnt8)");
        if ((e = cudaMemcpy(h->d_cnt8, c8.data(), c8.size(), cudaMemcpyHostToDevice)) != cudaSuccess)
            return fail(e, "H2D cnt8");
    }
    const std::vector<uint8_t> &blob = tier == AC_TIER_COMPACT ? t.compact : t.stt;
    const size_t stt_alloc = (blob.size() + 15) / 16 * 16 + 16;
    if ((e = cudaMalloc(&h->d_stt, stt_alloc)) != cudaSuccess) return fail(e, "cudaMalloc(stt)");
    if ((e = cudaMemset(h->d_stt, 0, stt_alloc)) != cudaSuccess) return fail(e, "cudaMemset(stt)");
    if ((e = cudaMemcpy(h->d_stt, blob.data(), blob.size(), cudaMemcpyHostToDevice)) != cudaSuccess)
        return fail(e, "H2D stt");
    if (!t.stt2.empty()) {
        if ((e = cudaMalloc(&h->d_stt2, t.stt2.size() * 4)) != cudaSuccess) return fail(e, "cudaMalloc(stt2)");
        if ((e = cudaMemcpy(h->d_stt2, t.stt2.data(), t.stt2.size() * 4, cudaMemcpyHostToDevice)) != cudaSuccess)
            return fail(e, "H2D stt2");
    }
    if ((e = cudaMalloc(&h->d_class_map, 256)) != cudaSuccess) return fail(e, "cudaMalloc(class map)");
    uint8_t cmap[256];  // COMPACT walks with doubled classes (column byte offsets)
    for (int b = 0; b < 256; b++) cmap[b] = tier == AC_TIER_COMPACT ? (uint8_t)(2 * t.class_map[b]) : t.class_map[b];
    if ((e = cudaMemcpy(h->d_class_map, cmap, 256, cudaMemcpyHostToDevice)) != cudaSuccess)
        return fail(e, "H2D class map");
    if ((e = cudaMalloc(&h->d_out_off, t.out_off.size() * 4)) != cudaSuccess) return fail(e, "cudaMalloc(out_off)");
    if ((e = cudaMemcpy(h->d_out_off, t.out_off.data(), t.out_off.size() * 4, cudaMemcpyHostToDevice)) != cudaSuccess)
        return fail(e, "H2D out_off");
    const size_t nid = t.out_ids.size() ? t.out_ids.size() : 1;
    if ((e = cudaMalloc(&h->d_out_ids, nid * 4)) != cudaSuccess) return fail(e, "cudaMalloc(out_ids)");
    if (!t.out_ids.empty() &&
        (e = cudaMemcpy(h->d_out_ids, t.out_ids.data(), t.out_ids.size() * 4, cudaMemcpyHostToDevice)) != cudaSuccess)
        return fail(e, "H2D out_ids");
    const size_t nl = t.lens.size() ? t.lens.size() : 1;
    if ((e = cudaMalloc(&h->d_lens, nl * 4)) != cudaSuccess) return fail(e, "cudaMalloc(lens)");
    if (!t.lens.empty() && (e = cudaMemcpy(h->d_lens, t.lens.data(), t.lens.size() * 4, cudaMemcpyHostToDevice)) != cudaSuccess)
        return fail(e, "H2D lens");
    if (prev >= 0 && prev != device) cudaSetDevice(prev);
    *out = h;
    return AC_OK;
}

void ac_free(ac_stt *h) {
    if (!h) return;
    int prev = -1;
    cudaGetDevice(&prev);
    cudaSetDevice(h->device);
    free_device(h);
    if (prev >= 0) cudaSetDevice(prev);
    delete h;
}

ac_status ac_stt_query(const ac_stt *h, ac_stt_info *info) {
    if (!h || !info) return AC_ERR_INVALID_ARG;
    fill_info(h->host, info);
    info->tier = h->tier;
    info->hot_rows = h->hot_rows;
    return AC_OK;
}

ac_status ac_stt_pattern_lengths(const ac_stt *h, uint32_t *lens) {
    if (!h || (!lens && h->host.n_patterns)) return AC_ERR_INVALID_ARG;
    if (h->host.n_patterns) std::memcpy(lens, h->host.lens.data(), h->host.lens.size() * 4);
    return AC_OK;
}

ac_status ac_match_async(const ac_stt *stt, const uint8_t *d_text, uint64_t n_owned, uint64_t n_halo, uint64_t base,
                         ac_match_t *d_out, uint64_t cap, ac_result *d_result, void *stream,
                         const ac_match_opts *opts) {
    if (!stt) {
        set_error("stt is NULL");
        return AC_ERR_INVALID_ARG;
    }
    DeviceGuard guard(stt->device);  // launches go to the STT's device
    try {
        return match_async(stt, d_text, n_owned, n_halo, base, d_out, cap, d_result,
                           static_cast<cudaStream_t>(stream), opts);
    } catch (...) {
        set_error("unexpected host exception");
        return AC_ERR_NO_MEMORY;
    }
}

ac_status ac_match_segments(const ac_stt *stt, const uint8_t *d_text, const uint64_t *d_seg_off, uint64_t n_seg,
                            ac_match_t *d_out, uint64_t cap, ac_result *d_result, void *stream) {
    if (!stt) {
        set_error("stt is NULL");
        return AC_ERR_INVALID_ARG;
    }
    DeviceGuard guard(stt->device);
    try {
        return match_segments(stt, d_text, d_seg_off, n_seg, d_out, cap, d_result, static_cast<cudaStream_t>(stream));
    } catch (...) {
        set_error("unexpected host exception");
        return AC_ERR_NO_MEMORY;
    }
}

ac_status ac_match_shard(const ac_stt *stt, const uint8_t *d_text, uint64_t n_owned, uint64_t n_halo, uint64_t base,
                         ac_match_t *d_out, uint64_t cap, uint64_t *count, void *stream) {
    if (!stt) {
        set_error("stt is NULL");
        return AC_ERR_INVALID_ARG;
    }
    if (n_halo > (stt->host.maxlen ? stt->host.maxlen - 1 : 0)) {
        set_error("n_halo exceeds maxlen - 1");
        return AC_ERR_INVALID_ARG;
    }
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    DeviceGuard guard(stt->device);  // the result word lives on the STT's device
    ac_result *d_res = nullptr;
    AC_CUDA(ws_alloc(reinterpret_cast<void **>(&d_res), sizeof(ac_result), s, stt->device), "cudaMallocAsync(result)");
    ac_status rc = ac_match_async(stt, d_text, n_owned, n_halo, base, d_out, cap, d_res, stream, nullptr);
    if (rc == AC_OK) rc = finish_sync(d_res, count, s);
    cudaFreeAsync(d_res, s);
    return rc;
}

ac_status ac_match(const ac_stt *stt, const uint8_t *d_text, uint64_t n, ac_match_t *d_out, uint64_t cap,
                   uint64_t *count, void *stream) {
    return ac_match_shard(stt, d_text, n, 0, 0, d_out, cap, count, stream);
}

ac_status ac_match_host(const ac_stt *stt, const uint8_t *h_text, uint64_t n, ac_match_t *h_out, uint64_t cap,
                        uint64_t *count, void *stream) {
    if (!stt || (!h_text && n)) {
        set_error("NULL stt or text");
        return AC_ERR_INVALID_ARG;
    }
    try {
        return match_host_pipelined(stt, h_text, n, h_out, cap, count, static_cast<cudaStream_t>(stream));
    } catch (...) {
        set_error("unexpected host exception");
        return AC_ERR_NO_MEMORY;
    }
}

}  // extern "C"
