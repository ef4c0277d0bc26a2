/*
 * ORACLE — TEST INFRASTRUCTURE ONLY (same rules as direct_conv.c: only tests/,
 * __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may load it;
 * it shares no code with the CUDA path).
 *
 * Plain fp64 direct 3D NDHWC convolution / deconvolution: the ND extension of the 2D
 * definition ("Im2col-Winograd can be applied to ND convolution, by
 * expanding Stage1 Im2col to ND, while remaining Stage2 unchanged"; Stage 1 is the im2col
 * index map, so the method reaches exactly the direct ND convolution):
 *
 *   conv:   y[n][d][p][q][k] = sum_{t<T} sum_{r<R} sum_{s<S} sum_{c<C}
 *                              x[n][d-pd+t][p-ph+r][q-pw+s][c] * w[k][t][r][s][c]
 *           OD = D + 2pd - T + 1, P = H + 2ph - R + 1, Q = W + 2pw - S + 1, x = 0 outside.
 *   deconv: y[n][d][p][q][k] = sum_{c,t,r,s} x[n][d+pd-t][p+ph-r][q+pw-s][c] * w[c][t][r][s][k]
 *           OD = D + T - 1 - 2pd, P = H + R - 1 - 2ph, Q = W + S - 1 - 2pw.
 * Both also return B = sum |x|*|w| over the same terms.
 * Loops: (n, d, p) outer (OpenMP), then q, k, then t, r, s, c innermost.
 */
#include <math.h>
#include <stddef.h>

static void point3(int deconv, int D, int H, int W, int C, int K, int T, int R, int S, int pd, int ph, int pw,
                   const float* x, const float* w, int n, int d, int p, int q, int k, double* yo, double* bo) {
  double acc = 0.0, bnd = 0.0;
  for (int t = 0; t < T; ++t) {
    const int id = deconv ? d + pd - t : d - pd + t;
    if (id < 0 || id >= D) continue; /* zero padding */
    for (int r = 0; r < R; ++r) {
      const int ih = deconv ? p + ph - r : p - ph + r;
      if (ih < 0 || ih >= H) continue;
      for (int s = 0; s < S; ++s) {
        const int iw = deconv ? q + pw - s : q - pw + s;
        if (iw < 0 || iw >= W) continue;
        const float* xp = x + ((((size_t)n * D + id) * H + ih) * W + iw) * C;
        for (int c = 0; c < C; ++c) {
          const double a = (double)xp[c];
          const double b = deconv ? (double)w[((((size_t)c * T + t) * R + r) * S + s) * K + k]
                                  : (double)w[((((size_t)k * T + t) * R + r) * S + s) * C + c];
          acc += a * b;
          bnd += fabs(a) * fabs(b);
        }
      }
    }
  }
  *yo = acc;
  if (bo) *bo = bnd;
}

static int run3(int deconv, int N, int D, int H, int W, int C, int K, int T, int R, int S, int pd, int ph, int pw,
                const float* x, const float* w, double* y, double* b) {
  const int OD = deconv ? D + T - 1 - 2 * pd : D + 2 * pd - T + 1;
  const int P = deconv ? H + R - 1 - 2 * ph : H + 2 * ph - R + 1;
  const int Q = deconv ? W + S - 1 - 2 * pw : W + 2 * pw - S + 1;
  if (N <= 0 || D <= 0 || H <= 0 || W <= 0 || C <= 0 || K <= 0 || T <= 0 || R <= 0 || S <= 0 || pd < 0 ||
      ph < 0 || pw < 0 || OD < 1 || P < 1 || Q < 1)
    return -1;
#pragma omp parallel for collapse(3) schedule(static)
  for (int n = 0; n < N; ++n)
    for (int d = 0; d < OD; ++d)
      for (int p = 0; p < P; ++p)
        for (int q = 0; q < Q; ++q)
          for (int k = 0; k < K; ++k) {
            const size_t o = ((((size_t)n * OD + d) * P + p) * Q + q) * K + k;
            point3(deconv, D, H, W, C, K, T, R, S, pd, ph, pw, x, w, n, d, p, q, k, &y[o], b ? &b[o] : NULL);
          }
  return 0;
}

int oracle_conv3d_ndhwc_f64(int N, int D, int H, int W, int C, int K, int T, int R, int S, int pd, int ph, int pw,
                            const float* x, const float* w, double* y, double* b) {
  return run3(0, N, D, H, W, C, K, T, R, S, pd, ph, pw, x, w, y, b);
}

int oracle_deconv3d_ndhwc_f64(int N, int D, int H, int W, int C, int K, int T, int R, int S, int pd, int ph, int pw,
                              const float* x, const float* w, double* y, double* b) {
  return run3(1, N, D, H, W, C, K, T, R, S, pd, ph, pw, x, w, y, b);
}
