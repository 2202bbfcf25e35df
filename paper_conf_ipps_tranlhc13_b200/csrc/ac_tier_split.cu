// ac_tier_split.cu -- instantiates the staged scan for the SPLIT STT tier
// (hot part in shared memory, cold states in L1/L2; ac_split.cpp).  The
// global-only kernel, the re-walk and packet batches read a SPLIT automaton
// through its GLOBAL table (ac_tier_global.cu).
#include "ac_kernels.cuh"

namespace acx {
template cudaError_t launch_staged_tier<AC_TIER_SPLIT>(int, uint32_t, int, const CUtensorMap &, const uint8_t *,
                                                    const SttView &, const StagedGeom &, const ScanOut &, size_t,
                                                    cudaStream_t);
}  // namespace acx

#ifdef AC_DEBUG_TIMES
extern "C" int ac_debug_times(unsigned long long *host, unsigned n) {
    return (int)cudaMemcpyFromSymbol(host, acx::ac_dbg_times, n * sizeof(unsigned long long));
}
#endif
