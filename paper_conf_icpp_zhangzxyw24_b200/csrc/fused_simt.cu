// TEST-ONLY stepping stone: a plain SIMT fp32 fused
// Im2col-Winograd kernel over the same plan, U layout and generated tables as
// the tcgen05 kernel. It is NOT dispatched by i2cw_conv2d_nhwc; it is exported
// only as i2cw_debug_conv_simt (declared in csrc/debug_api.h, not in the public
// header) so GPU tests can localise a failure to the contraction vs. the
// transforms / indexing / boundary handling.
//
// Per thread = one Winograd tile (n, p, q0 = tw*m), §4.1 Stage 2:
//   V_t = sum_j BT[t][j] x[n][p-ph+fh][q0-pw+j][c]      (input transform)
//   M_t[k] += V_t * U_t[k][(fh,c)]                      (elem-mul, accumulated over fh, c)
//   y[n][p][q0+i][k] = sum_t AT[i][t] M_t[k]            (output transform, once)
#include "common.cuh"
#include "transforms_generated.h"

namespace i2cw {

template <int M, int RW>
__global__ void __launch_bounds__(128) fused_simt_kernel(const __grid_constant__ Plan pl, const float* __restrict__ x,
                                                         const float* __restrict__ u, float* __restrict__ y) {
  using T = Wino<M, RW>;
  constexpr int A = T::alpha;
  const int lane = threadIdx.x;
  const int b = blockIdx.x;
  const int nb = b % pl.NB;
  int tb = b / pl.NB;
  const int seg = tb % pl.SEGS;
  tb /= pl.SEGS;
  const int rb = tb % pl.PB;
  const int vrow = pl.lane_row[lane], tw_l = pl.lane_tw[lane];
  if (vrow == 0xFF) return;
  const int n = (tb / pl.PB) * pl.NI + vrow / pl.ROWS;
  const int p = rb * pl.ROWS + vrow % pl.ROWS, tw = seg * pl.TS + tw_l;
  if (n >= pl.N || p >= pl.P || tw >= pl.T_r) return;
  const int q0 = tw * M;
  for (int k8 = 0; k8 < pl.NT / 8; ++k8) {
    float acc[A][8];
#pragma unroll
    for (int t = 0; t < A; ++t)
#pragma unroll
      for (int kk = 0; kk < 8; ++kk) acc[t][kk] = 0.f;
    for (int ks = 0; ks < pl.NKS; ++ks) {
      const int cc = ks / pl.R, fh = ks % pl.R;
      const int ih = p - pl.pad_h + fh;
      for (int ci = 0; ci < 8; ++ci) {
        const int c = cc * 8 + ci;
        float d[A];
#pragma unroll
        for (int j = 0; j < A; ++j) {
          const int iw = q0 - pl.pad_w + j;
          d[j] = (ih >= 0 && ih < pl.H && iw >= 0 && iw < pl.W && c < pl.C)
                     ? x[(((size_t)n * pl.H + ih) * pl.W + iw) * pl.C + c]
                     : 0.f;
        }
#pragma unroll
        for (int idx = 0; idx < A; ++idx) {
          const int pt = point_of(idx, A);
          float v = 0.f;
#pragma unroll
          for (int j = 0; j < A; ++j) v = fmaf(T::BT(pt, j), d[j], v);
          const size_t uo = u_offset(pl.NT, A, nb, pl.NKS, ks, idx, 0) + (size_t)(ci / 4) * pl.NT * 4 + (ci % 4);
#pragma unroll
          for (int kk = 0; kk < 8; ++kk) {
            const int nn = k8 * 8 + kk;
            const float uv = u[uo + (size_t)nn * 4] + u[uo + (size_t)nn * 4 + (size_t)pl.NT * 8];
            acc[idx][kk] = fmaf(v, uv, acc[idx][kk]);
          }
        }
      }
    }
#pragma unroll
    for (int i = 0; i < M; ++i) {
      if (q0 + i >= pl.Q) break;
      float* yp = y + (((size_t)n * pl.P + p) * pl.Q + q0 + i) * pl.K;
#pragma unroll
      for (int kk = 0; kk < 8; ++kk) {
        const int k = nb * pl.NT + k8 * 8 + kk;
        float o = 0.f;
#pragma unroll
        for (int idx = 0; idx < A; ++idx) o = fmaf(T::AT(i, point_of(idx, A)), acc[idx][kk], o);
        if (k < pl.K) yp[k] = o;
      }
    }
  }
}

cudaError_t launch_fused_simt(const Plan& pl, const float* x, const float* u, float* y, cudaStream_t stream) {
  const dim3 grid(pl.tile_blocks * pl.NB), block(128);
  switch (pl.S * 100 + pl.m) {
#define I2CW_CASE(MM, RR) \
  case RR * 100 + MM: fused_simt_kernel<MM, RR><<<grid, block, 0, stream>>>(pl, x, u, y); break;
    I2CW_CASE(7, 2) I2CW_CASE(6, 3) I2CW_CASE(5, 4) I2CW_CASE(4, 5) I2CW_CASE(3, 6) I2CW_CASE(2, 7)
    I2CW_CASE(5, 8) I2CW_CASE(4, 9) I2CW_CASE(10, 7) I2CW_CASE(9, 8) I2CW_CASE(8, 9)
#undef I2CW_CASE
    default: return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

}  // namespace i2cw
