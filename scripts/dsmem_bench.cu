// dsmem_bench.cu -- is a DSMEM cluster-distributed STT worth building?
// (DESIGN.md section 12.)  Development tool, not the product.
//
// Every thread walks a dependent chain of random table lookups -- the shape of
// the AC DFA walk (one dependent gather per byte) -- over a table of
// `cs` x 2^15 32-bit entries (128 KB per CTA; power-of-two sizes so the index
// arithmetic is masks, not divisions) held three ways:
//   local : each CTA's own shared-memory copy of a per_cta slice (the SMEM tier)
//   dsmem : the table split across the `cs` CTAs of a thread-block cluster,
//           each lookup a ld.shared::cluster to the CTA that owns the entry
//   global: the whole table in global memory, read with ld.global.nc (L1/L2,
//           the GLOBAL tier)
// and reports lookups per second for the whole GPU.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o dsmem_bench scripts/dsmem_bench.cu
//   ./dsmem_bench            # one JSON line per (mode, cluster size)
#include <cooperative_groups.h>
#include <cstdint>
#include <cstdio>
#include <vector>

namespace cg = cooperative_groups;

constexpr int kThreads = 1024;
constexpr int kSteps = 4096;

__device__ __forceinline__ uint32_t mix(uint32_t x) {
    x ^= x >> 16;
    x *= 0x7feb352dU;
    x ^= x >> 15;
    return x;
}

// table entries hold the next random index (the "next state")
__global__ void fill(uint32_t *t, uint64_t n, uint32_t seed) {
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
        t[i] = mix((uint32_t)i * 2654435761u + seed);
}

__global__ void __launch_bounds__(kThreads, 1) k_local(const uint32_t *g, uint32_t per_cta, uint32_t *sink) {
    extern __shared__ uint32_t s[];
    for (uint32_t i = threadIdx.x; i < per_cta; i += blockDim.x) s[i] = g[i];
    __syncthreads();
    uint32_t x = mix(blockIdx.x * kThreads + threadIdx.x);
    for (int k = 0; k < kSteps; k++) x = s[x & (per_cta - 1)];
    if (x == 0xFFFFFFFFu) sink[0] = x;
}

__global__ void __launch_bounds__(kThreads, 1) k_dsmem(const uint32_t *g, uint32_t per_cta, uint32_t *sink) {
    extern __shared__ uint32_t s[];
    cg::cluster_group cl = cg::this_cluster();
    const uint32_t cs = cl.num_blocks(), me = cl.block_rank();
    for (uint32_t i = threadIdx.x; i < per_cta; i += blockDim.x) s[i] = g[(uint64_t)me * per_cta + i];
    cl.sync();
    uint32_t x = mix(blockIdx.x * kThreads + threadIdx.x);
    const uint32_t n = cs * per_cta;
    const uint32_t base = (uint32_t)__cvta_generic_to_shared(s);
    for (int k = 0; k < kSteps; k++) {
        const uint32_t idx = x & (n - 1);
        uint32_t remote;
        asm("mapa.shared::cluster.u32 %0, %1, %2;"
            : "=r"(remote)
            : "r"(base + (idx & (per_cta - 1)) * 4), "r"(idx >> 15));
        asm volatile("ld.shared::cluster.u32 %0, [%1];" : "=r"(x) : "r"(remote));
    }
    cl.sync();  // keep every slice alive until all readers are done
    if (x == 0xFFFFFFFFu) sink[0] = x;
}

__global__ void __launch_bounds__(kThreads, 1) k_global(const uint32_t *g, uint32_t n, uint32_t *sink) {
    uint32_t x = mix(blockIdx.x * kThreads + threadIdx.x);
    for (int k = 0; k < kSteps; k++) x = __ldg(g + (x & (n - 1)));
    if (x == 0xFFFFFFFFu) sink[0] = x;
}

int main() {
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const uint32_t per_cta = 32 * 1024;  // 128 KB slice per CTA (2^15 entries: index arithmetic is masks)
    const size_t smem = per_cta * 4;
    uint32_t *g, *sink;
    const uint64_t max_n = 16ull * per_cta;
    cudaMalloc(&g, max_n * 4);
    cudaMalloc(&sink, 4);
    fill<<<1024, 256>>>(g, max_n, 7);
    cudaFuncSetAttribute(k_local, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    cudaFuncSetAttribute(k_dsmem, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    cudaFuncSetAttribute(k_dsmem, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    auto report = [&](const char *mode, int cs, uint64_t table_bytes, int grid, float ms) {
        const double lookups = (double)grid * kThreads * kSteps;
        printf("{\"mode\": \"%s\", \"cluster\": %d, \"table_bytes\": %llu, \"grid\": %d, \"ms\": %.3f, "
               "\"glookups_per_s\": %.1f}\n",
               mode, cs, (unsigned long long)table_bytes, grid, ms, lookups / ms / 1e6);
        fflush(stdout);
    };
    for (int rep = 0; rep < 2; rep++) {
        cudaEventRecord(a);
        k_local<<<sms, kThreads, smem>>>(g, per_cta, sink);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        if (rep) report("local", 1, smem, sms, ms);
    }
    for (int cs : {2, 4, 8, 16}) {
        const int grid = sms / cs * cs;
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3(grid);
        cfg.blockDim = dim3(kThreads);
        cfg.dynamicSmemBytes = smem;
        cudaLaunchAttribute attr[1];
        attr[0].id = cudaLaunchAttributeClusterDimension;
        attr[0].val.clusterDim.x = cs;
        attr[0].val.clusterDim.y = 1;
        attr[0].val.clusterDim.z = 1;
        cfg.attrs = attr;
        cfg.numAttrs = 1;
        int max_clusters = 0;
        if (cudaOccupancyMaxActiveClusters(&max_clusters, k_dsmem, &cfg) != cudaSuccess || max_clusters == 0) {
            cudaGetLastError();
            printf("{\"mode\": \"dsmem\", \"cluster\": %d, \"skipped\": \"no active cluster of this size\"}\n", cs);
            continue;
        }
        const int g2 = (max_clusters * cs < grid) ? max_clusters * cs : grid;
        cfg.gridDim = dim3(g2);
        for (int rep = 0; rep < 2; rep++) {
            cudaEventRecord(a);
            cudaError_t e = cudaLaunchKernelEx(&cfg, k_dsmem, (const uint32_t *)g, per_cta, sink);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            if (e != cudaSuccess) {
                printf("{\"mode\": \"dsmem\", \"cluster\": %d, \"error\": \"%s\"}\n", cs, cudaGetErrorString(e));
                break;
            }
            float ms;
            cudaEventElapsedTime(&ms, a, b);
            if (rep) report("dsmem", cs, (uint64_t)cs * smem, g2, ms);
        }
        for (int rep = 0; rep < 2; rep++) {
            cudaEventRecord(a);
            k_global<<<sms, kThreads>>>(g, cs * per_cta, sink);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float ms;
            cudaEventElapsedTime(&ms, a, b);
            if (rep) report("global", cs, (uint64_t)cs * smem, sms, ms);
        }
    }
    printf("{\"done\": \"%s\"}\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
