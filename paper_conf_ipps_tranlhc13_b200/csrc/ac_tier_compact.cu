// ac_tier_compact.cu -- instantiates the scan kernels for the COMPACT STT tier.
#include "ac_kernels.cuh"

namespace acx {
template cudaError_t launch_global_tier<AC_TIER_COMPACT>(int, uint32_t, const uint8_t *, uint64_t, const SttView &,
                                                     const Region &, const Region &, const ScanOut &, size_t,
                                                     cudaStream_t);
template cudaError_t launch_staged_tier<AC_TIER_COMPACT>(int, uint32_t, int, const CUtensorMap &, const uint8_t *,
                                                     const SttView &, const StagedGeom &, const ScanOut &, size_t,
                                                     cudaStream_t);
}  // namespace acx

namespace acx {
template cudaError_t launch_rewalk_tier<AC_TIER_COMPACT>(uint32_t, const uint8_t *, uint64_t, const SttView &,
                                                     const Region &, const Region &, const StagedGeom &,
                                                     const ScanOut &, const uint64_t *, const unsigned int *, size_t,
                                                     int, cudaStream_t);
}  // namespace acx

namespace acx {
template cudaError_t launch_segments_tier<AC_TIER_COMPACT>(int, uint32_t, const uint8_t *, const uint64_t *, uint64_t,
                                                       const SttView &, const ScanOut &, size_t, cudaStream_t);
}  // namespace acx
