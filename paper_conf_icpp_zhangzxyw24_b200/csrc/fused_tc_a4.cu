// Instantiations of the fused tcgen05 kernel (fused_tc.cuh) for the alpha family "a4" (Gamma4(3,2), Gamma4(2,3): PAPER.md:281-288, 309-313)
// (one translation unit per family so the build compiles them in parallel).
#include "fused_tc.cuh"

namespace i2cw {

// returns cudaErrorNotSupported when (m, r) is not in this family
cudaError_t launch_fused_tc_a4(const CUtensorMap& xmap, const CUtensorMap& ymap, const Plan& pl, const float* u,
                                 cudaStream_t stream) {
  const int key = pl.S * 1000 + pl.m * 10 + (pl.NT == 128 ? 2 : (pl.NT == 64 ? 1 : 0));
  switch (key) {
#define I2CW_TC(MM, RR)                                                                               \
  case RR * 1000 + MM * 10 + 1:                                                                      \
    return pl.pair ? launch_tc_t<MM, RR, 64, true>(xmap, ymap, pl, u, stream)                       \
                   : launch_tc_t<MM, RR, 64, false>(xmap, ymap, pl, u, stream);                     \
  case RR * 1000 + MM * 10 + 0:                                                                      \
    return pl.pair ? launch_tc_t<MM, RR, 32, true>(xmap, ymap, pl, u, stream)                       \
                   : launch_tc_t<MM, RR, 32, false>(xmap, ymap, pl, u, stream);
    I2CW_TC(3, 2) I2CW_TC(2, 3)
#undef I2CW_TC
    default: return cudaErrorNotSupported;
  }
}

}  // namespace i2cw
