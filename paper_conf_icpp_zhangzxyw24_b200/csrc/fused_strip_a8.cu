// Instantiations of the strip kernel (fused_strip.cuh) for the alpha = 8 family (r = 2..7).
#include "fused_strip.cuh"

namespace i2cw {

cudaError_t launch_fused_strip_a8(const CUtensorMap& xmap, const YMaps& ymap, const Plan& pl, const float* u,
                                  cudaStream_t stream) {
  switch (pl.S * 10 + pl.m) {
    case 27: return pl.pair ? launch_strip_t2<7, 2, true>(xmap, ymap, pl, u, stream) : launch_strip_t2<7, 2, false>(xmap, ymap, pl, u, stream);
    case 36: return pl.pair ? launch_strip_t2<6, 3, true>(xmap, ymap, pl, u, stream) : launch_strip_t2<6, 3, false>(xmap, ymap, pl, u, stream);
    case 45: return pl.pair ? launch_strip_t2<5, 4, true>(xmap, ymap, pl, u, stream) : launch_strip_t2<5, 4, false>(xmap, ymap, pl, u, stream);
    case 54: return pl.pair ? launch_strip_t2<4, 5, true>(xmap, ymap, pl, u, stream) : launch_strip_t2<4, 5, false>(xmap, ymap, pl, u, stream);
    case 63: return pl.pair ? launch_strip_t2<3, 6, true>(xmap, ymap, pl, u, stream) : launch_strip_t2<3, 6, false>(xmap, ymap, pl, u, stream);
    case 72: return pl.pair ? launch_strip_t2<2, 7, true>(xmap, ymap, pl, u, stream) : launch_strip_t2<2, 7, false>(xmap, ymap, pl, u, stream);
    default: return cudaErrorNotSupported;
  }
}

}  // namespace i2cw
