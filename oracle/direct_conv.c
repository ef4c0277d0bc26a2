/*
 * ORACLE — TEST INFRASTRUCTURE ONLY.
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
 * reference legs may load this library. The product path (include/i2cw.h,
 * paper_conf_icpp_zhangzxyw24_b200/) never links, imports or calls it, and it
 * shares no code with the CUDA path.
 *
 * Plain fp64 direct NHWC convolution / deconvolution, written from the
 * definition the Im2col-Winograd method reaches exactly (up to rounding):
 *
 *   Table 1: X in R^{N x IH x IW x IC}, W in R^{OC x FH x FW x IC},
 *   Y in R^{N x OH x OW x OC}; pH, pW zero padding (implicit);
 *   unit stride; the paper's own ground truth is an
 *   "FP64-CPU convolution ... FP64 accumulators".
 *   §4.1: the method equals the im2col GEMM with
 *   GM = N*OH*OW, GK = IC*FH*FW, GN = OC, i.e. the direct sum below.
 *
 * conv (cross-correlation, SURVEY.md §8(c) c3 reading 1):
 *   y[n][p][q][k] = sum_{r<R} sum_{s<S} sum_{c<C} x[n][p-ph+r][q-pw+s][c] * w[k][r][s][c]
 *   P = H + 2ph - R + 1, Q = W + 2pw - S + 1, x = 0 outside [0,H) x [0,W).
 * deconv (backward-data with the 180-degree-rotated filter):
 *   y[n][p][q][k] = sum_{c,r,s} x[n][p+ph-r][q+pw-s][c] * w[c][r][s][k]
 *   P = H + R - 1 - 2ph, Q = W + S - 1 - 2pw.
 * Both also return the error scale  B = sum |x|*|w|  over the same terms
 * (the per-element tolerance of BASELINE.json north_star is 1e-4 * B).
 *
 * Loops: (n, p) outer (OpenMP), then q, k, then r, s, c innermost. No blocking,
 * no reordering beyond that.
 */
#include <math.h>
#include <stdint.h>
#include <stddef.h>
#ifdef _OPENMP
#include <omp.h>
#endif

int oracle_num_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}

/* one output element of the conv: y[n][p][q][k] (and its bound) */
static void conv_point(int H, int W, int C, int R, int S, int ph, int pw,
                       const float* x, const float* w, int n, int p, int q, int k,
                       double* yo, double* bo) {
  double acc = 0.0, bnd = 0.0;
  for (int r = 0; r < R; ++r) {
    const int ih = p - ph + r;
    if (ih < 0 || ih >= H) continue; /* zero padding */
    for (int s = 0; s < S; ++s) {
      const int iw = q - pw + s;
      if (iw < 0 || iw >= W) continue;
      const float* xp = x + (((size_t)n * H + ih) * W + iw) * C;
      const float* wp = w + (((size_t)k * R + r) * S + s) * C;
      for (int c = 0; c < C; ++c) {
        const double a = (double)xp[c], b = (double)wp[c];
        acc += a * b;
        bnd += fabs(a) * fabs(b);
      }
    }
  }
  *yo = acc;
  if (bo) *bo = bnd;
}

/* one output element of the deconv; w is [C][R][S][K] (C = deconv input channels) */
static void deconv_point(int H, int W, int C, int K, int R, int S, int ph, int pw,
                         const float* x, const float* w, int n, int p, int q, int k,
                         double* yo, double* bo) {
  double acc = 0.0, bnd = 0.0;
  for (int r = 0; r < R; ++r) {
    const int ih = p + ph - r;
    if (ih < 0 || ih >= H) continue;
    for (int s = 0; s < S; ++s) {
      const int iw = q + pw - s;
      if (iw < 0 || iw >= W) continue;
      const float* xp = x + (((size_t)n * H + ih) * W + iw) * C;
      for (int c = 0; c < C; ++c) {
        const double a = (double)xp[c];
        const double b = (double)w[(((size_t)c * R + r) * S + s) * K + k];
        acc += a * b;
        bnd += fabs(a) * fabs(b);
      }
    }
  }
  *yo = acc;
  if (bo) *bo = bnd;
}

/* Full conv. y, b: [N][P][Q][K] fp64 (b may be NULL). Returns 0, or -1 on bad shape. */
int oracle_conv2d_nhwc_f64(int N, int H, int W, int C, int K, int R, int S, int ph, int pw,
                           const float* x, const float* w, double* y, double* b) {
  const int P = H + 2 * ph - R + 1, Q = W + 2 * pw - S + 1;
  if (N <= 0 || H <= 0 || W <= 0 || C <= 0 || K <= 0 || R <= 0 || S <= 0 || P <= 0 || Q <= 0)
    return -1;
#pragma omp parallel for collapse(2) schedule(static)
  for (int n = 0; n < N; ++n)
    for (int p = 0; p < P; ++p)
      for (int q = 0; q < Q; ++q)
        for (int k = 0; k < K; ++k) {
          const size_t o = (((size_t)n * P + p) * Q + q) * K + k;
          conv_point(H, W, C, R, S, ph, pw, x, w, n, p, q, k, y + o, b ? b + o : NULL);
        }
  return 0;
}

int oracle_deconv2d_nhwc_f64(int N, int H, int W, int C, int K, int R, int S, int ph, int pw,
                             const float* x, const float* w, double* y, double* b) {
  const int P = H + R - 1 - 2 * ph, Q = W + S - 1 - 2 * pw;
  if (N <= 0 || H <= 0 || W <= 0 || C <= 0 || K <= 0 || R <= 0 || S <= 0 || P <= 0 || Q <= 0)
    return -1;
#pragma omp parallel for collapse(2) schedule(static)
  for (int n = 0; n < N; ++n)
    for (int p = 0; p < P; ++p)
      for (int q = 0; q < Q; ++q)
        for (int k = 0; k < K; ++k) {
          const size_t o = (((size_t)n * P + p) * Q + q) * K + k;
          deconv_point(H, W, C, K, R, S, ph, pw, x, w, n, p, q, k, y + o, b ? b + o : NULL);
        }
  return 0;
}

/* Sampled outputs: idx is [npts][4] = (n, p, q, k); y[i], b[i] for each point.
 * Used at full BASELINE sizes where the whole oracle would take too long. */
int oracle_conv2d_nhwc_f64_points(int N, int H, int W, int C, int K, int R, int S, int ph, int pw,
                                  const float* x, const float* w, int64_t npts, const int32_t* idx,
                                  double* y, double* b) {
  const int P = H + 2 * ph - R + 1, Q = W + 2 * pw - S + 1;
  if (P <= 0 || Q <= 0) return -1;
  for (int64_t i = 0; i < npts; ++i) {
    const int32_t* t = idx + 4 * i;
    if (t[0] < 0 || t[0] >= N || t[1] < 0 || t[1] >= P || t[2] < 0 || t[2] >= Q || t[3] < 0 || t[3] >= K)
      return -1;
  }
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < npts; ++i) {
    const int32_t* t = idx + 4 * i;
    conv_point(H, W, C, R, S, ph, pw, x, w, t[0], t[1], t[2], t[3], y + i, b ? b + i : NULL);
  }
  return 0;
}

int oracle_deconv2d_nhwc_f64_points(int N, int H, int W, int C, int K, int R, int S, int ph, int pw,
                                    const float* x, const float* w, int64_t npts, const int32_t* idx,
                                    double* y, double* b) {
  const int P = H + R - 1 - 2 * ph, Q = W + S - 1 - 2 * pw;
  if (P <= 0 || Q <= 0) return -1;
  for (int64_t i = 0; i < npts; ++i) {
    const int32_t* t = idx + 4 * i;
    if (t[0] < 0 || t[0] >= N || t[1] < 0 || t[1] >= P || t[2] < 0 || t[2] >= Q || t[3] < 0 || t[3] >= K)
      return -1;
  }
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < npts; ++i) {
    const int32_t* t = idx + 4 * i;
    deconv_point(H, W, C, K, R, S, ph, pw, x, w, t[0], t[1], t[2], t[3], y + i, b ? b + i : NULL);
  }
  return 0;
}
