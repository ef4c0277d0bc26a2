// Instantiations of the fused tcgen05 kernel (fused_tc.cuh) for the alpha family "a12"
// (one translation unit per family so the build compiles them in parallel); pl.vol selects the
// 3D (VOL) instantiation, single-CTA only.
#include "fused_tc.cuh"

namespace i2cw {

// returns cudaErrorNotSupported when (m, r) is not in this family
cudaError_t launch_fused_tc_a12(const CUtensorMap& xmap, const CUtensorMap& ymap, const Plan& pl, const float* u,
                                 cudaStream_t stream) {
  const int key = pl.S * 1000 + pl.m * 10 + (pl.NT == 128 ? 2 : (pl.NT == 64 ? 1 : 0));
  switch (key) {
#define I2CW_TC(MM, RR)                                                                               \
  case RR * 1000 + MM * 10 + 1:                                                                      \
    if (pl.vol) return launch_tc_t<MM, RR, 64, false, true>(xmap, ymap, pl, u, stream);               \
    if (pl.prec) return launch_tc_t<MM, RR, 64, false, false, true>(xmap, ymap, pl, u, stream);       \
    return pl.pair ? launch_tc_t<MM, RR, 64, true>(xmap, ymap, pl, u, stream)                       \
                   : launch_tc_t<MM, RR, 64, false>(xmap, ymap, pl, u, stream);                     \
  case RR * 1000 + MM * 10 + 2:                                                                      \
    return pl.pair ? launch_tc_t<MM, RR, 128, true>(xmap, ymap, pl, u, stream)                      \
                   : launch_tc_t<MM, RR, 128, false>(xmap, ymap, pl, u, stream);                    \
  case RR * 1000 + MM * 10 + 0:                                                                      \
    if (pl.vol) return launch_tc_t<MM, RR, 32, false, true>(xmap, ymap, pl, u, stream);               \
    if (pl.prec) return launch_tc_t<MM, RR, 32, false, false, true>(xmap, ymap, pl, u, stream);       \
    return pl.pair ? launch_tc_t<MM, RR, 32, true>(xmap, ymap, pl, u, stream)                       \
                   : launch_tc_t<MM, RR, 32, false>(xmap, ymap, pl, u, stream);
    I2CW_TC(5, 8) I2CW_TC(4, 9)
#undef I2CW_TC
    default: return cudaErrorNotSupported;
  }
}

}  // namespace i2cw
