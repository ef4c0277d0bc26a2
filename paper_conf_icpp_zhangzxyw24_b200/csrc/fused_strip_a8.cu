// Instantiations of the strip kernel (fused_strip.cuh) for the alpha = 8 family (r = 2..7).
#include "fused_strip.cuh"

namespace i2cw {

cudaError_t launch_fused_strip_a8(const CUtensorMap& xmap, const YMaps& ymap, const Plan& pl, const float* u,
                                  cudaStream_t stream) {
  switch (pl.S * 10 + pl.m) {
    case 27: return launch_strip_t<7, 2>(xmap, ymap, pl, u, stream);
    case 36: return launch_strip_t<6, 3>(xmap, ymap, pl, u, stream);
    case 45: return launch_strip_t<5, 4>(xmap, ymap, pl, u, stream);
    case 54: return launch_strip_t<4, 5>(xmap, ymap, pl, u, stream);
    case 63: return launch_strip_t<3, 6>(xmap, ymap, pl, u, stream);
    case 72: return launch_strip_t<2, 7>(xmap, ymap, pl, u, stream);
    default: return cudaErrorNotSupported;
  }
}

}  // namespace i2cw
