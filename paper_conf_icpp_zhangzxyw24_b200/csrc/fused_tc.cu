// Dispatch of the fused tcgen05 kernel over the alpha families (fused_tc_a*.cu).
#include "common.cuh"

namespace i2cw {
cudaError_t launch_fused_tc_a4(const CUtensorMap&, const CUtensorMap&, const Plan&, const float*, cudaStream_t);
cudaError_t launch_fused_tc_a8(const CUtensorMap&, const CUtensorMap&, const Plan&, const float*, cudaStream_t);
cudaError_t launch_fused_tc_a12(const CUtensorMap&, const CUtensorMap&, const Plan&, const float*, cudaStream_t);
cudaError_t launch_fused_tc_a16(const CUtensorMap&, const CUtensorMap&, const Plan&, const float*, cudaStream_t);

cudaError_t launch_fused_tc(const CUtensorMap& xmap, const CUtensorMap& ymap, const Plan& pl, const float* u,
                            cudaStream_t stream) {
  switch (pl.alpha) {
    case 4: return launch_fused_tc_a4(xmap, ymap, pl, u, stream);
    case 8: return launch_fused_tc_a8(xmap, ymap, pl, u, stream);
    case 12: return launch_fused_tc_a12(xmap, ymap, pl, u, stream);
    case 16: return launch_fused_tc_a16(xmap, ymap, pl, u, stream);
    default: return cudaErrorInvalidValue;
  }
}
}  // namespace i2cw
