// Filter transform U = G w (row a1 of SURVEY.md §8(a)).
//
// PAPER.md Alg 1 loadTiles (lines 355-362): G_tile = G(alpha,r) W_tile; §5.1
// (534-541): forward filters are re-laid out for vector loads, and for the
// backward deconvolution "the 180-degree filter-rotation is integrated into
// filter-transformation" (no separate rearrangement pass).
//
// For every output-channel block nb, k-step ks = (cc, fh), internal point idx:
//   U[nb][ks][idx][hl][kc][n][e] = split_hl( sum_s G[point(idx)][s] * w'(k, fh, s, c) )
//   k = nb*NT + n, c = cc*8 + kc*4 + e (zero outside [0,K) x [0,C))
//   conv:   w'(k, fh, s, c) = w[k][fh][s][c]                      (w is [K][R][S][C])
//   deconv: w'(k, fh, s, c) = w[c][R-1-fh][S-1-s][k]              (w is [C][R][S][K])
// G is applied in fp64 and rounded once to fp32 (the filter
// transform's precision hardly matters); hi = tf32_rna(u), lo = tf32_rna(u - hi).
#include <algorithm>
#include <cstdint>

#include "common.cuh"

namespace i2cw {

struct GTable {
  double g[16 * 9];  // row = INTERNAL point index, col = tap s
};

__global__ void filter_transform_kernel(const float* __restrict__ w, float* __restrict__ u, int C, int K, int R,
                                        int S, int is_deconv, int alpha, int NT, int NB, int NCC, int halves, int npg,
                                        GTable gt, UTag tag, UTag* tag_dst) {
  const int NKS = NCC * R;
  // let a programmatically dependent fused kernel start its prologue now (it waits with
  // griddepcontrol.wait before reading U, which covers this grid's completion)
  asm volatile("griddepcontrol.launch_dependents;");
  // the 256-byte tag in front of U (checked by the _pretransformed calls), written here instead
  // of by a separate host-to-device copy
  if (tag_dst && blockIdx.x == 0 && threadIdx.x == 0) *tag_dst = tag;
  // One thread per (point group, filter row segment (nb, ks, kc, n, e)): its S taps are read
  // once and the alpha / npg points of its group are produced from registers (npg = 1 for
  // large filters; small filters split the points over more threads to fill the GPU). The
  // fastest thread index follows the filter's contiguous dimension (c for the KRSC conv
  // filter, k for the CRSK deconv filter).
  const size_t rows = (size_t)NB * NKS * 2 * NT * 4;
  const size_t total = rows * npg;
  const int ppg = alpha / npg;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < total; i += (size_t)gridDim.x * blockDim.x) {
    size_t t = i % rows;
    const int g = (int)(i / rows);
    int e, n;
    if (is_deconv) {
      n = (int)(t % NT); t /= NT;
      e = (int)(t % 4); t /= 4;
    } else {
      e = (int)(t % 4); t /= 4;
      n = (int)(t % NT); t /= NT;
    }
    const int kc = (int)(t % 2); t /= 2;
    const int ks = (int)(t % NKS); t /= NKS;
    const int nb = (int)t;
    const int cc = ks / R, fh = ks % R;
    const int k = nb * NT + n, c = cc * 8 + kc * 4 + e;
    const bool live = k < K && c < C;
    double wv[9];
#pragma unroll
    for (int s = 0; s < 9; ++s) {
      wv[s] = 0.0;
      if (live && s < S)
        wv[s] = (double)(is_deconv ? w[(((size_t)c * R + (R - 1 - fh)) * S + (S - 1 - s)) * K + k]
                                   : w[(((size_t)k * R + fh) * S + s) * C + c]);
    }
    for (int idx = g * ppg; idx < (g + 1) * ppg; ++idx) {
      double acc = 0.0;
#pragma unroll
      for (int s = 0; s < 9; ++s)
        if (s < S) acc += gt.g[idx * 9 + s] * wv[s];
      const float uv = (float)acc;
      const float hi = tf32_rna(uv);
      const float lo = tf32_rna(uv - hi);
      if (halves == 2) {  // CTA-pair layout: [h][idx][hl][kc][n'][e] per (nb, ks)
        const int hN = NT / 2, h = n / hN, n2 = n % hN;
        const size_t base =
            u_offset_pair(NT, alpha, nb, NKS, ks, h, idx) + (size_t)kc * hN * 4 + (size_t)n2 * 4 + e;
        u[base] = hi;
        u[base + (size_t)hN * 8] = lo;
      } else {
        const size_t base = u_offset(NT, alpha, nb, NKS, ks, idx, 0) + (size_t)kc * NT * 4 + (size_t)n * 4 + e;
        u[base] = hi;
        u[base + (size_t)NT * 8] = lo;  // hl = 1 image follows the hl = 0 image
      }
    }
  }
}

cudaError_t launch_filter_transform(const float* w, float* u, int C, int K, int R, int S, int is_deconv, int alpha,
                                    int NT, int NB, int NCC, int halves, const double* G /* alpha x S, internal order */,
                                    const UTag& tag, UTag* tag_dst, cudaStream_t stream) {
  GTable gt;
  for (int i = 0; i < 16 * 9; ++i) gt.g[i] = 0.0;
  for (int i = 0; i < alpha; ++i)
    for (int s = 0; s < S; ++s) gt.g[i * 9 + s] = G[i * S + s];
  const size_t rows = (size_t)NB * NCC * R * 2 * NT * 4;
  // point groups: split the alpha points over threads until ~148 x 1024 threads are live
  int npg = 1;
  while (npg < alpha && alpha % (2 * npg) == 0 && rows * npg < (size_t)148 * 1024) npg *= 2;
  const size_t total = rows * npg;
  int blocks = (int)((total + 255) / 256);
  if (blocks > 148 * 16) blocks = 148 * 16;
  if (blocks < 1) blocks = 1;
  filter_transform_kernel<<<blocks, 256, 0, stream>>>(w, u, C, K, R, S, is_deconv, alpha, NT, NB, NCC, halves, npg, gt,
                                                      tag, tag_dst);
  return cudaGetLastError();
}

// Split-tail pre-zeroing of y (DESIGN.md §6.2 "split tail"), as a kernel instead of a
// cudaMemsetAsync: a memset node between the filter transform and the fused kernel would end
// their programmatic-dependent-launch overlap. This kernel is itself launched as a programmatic
// dependent of the filter transform (it does not read U, so it may run concurrently with it),
// lets the fused kernel launch at once, and waits for the filter transform's grid before it
// exits, so the fused kernel's griddepcontrol.wait (on this grid) still covers U.
// wait_first: the previous kernel in the stream is not the library's own filter transform (the
// pre-transformed path: whatever the caller ran last), so no store may happen before that grid
// has completed -- the PDL rule that a dependent touches no memory before griddepcontrol.wait.
__global__ void zero_tail_kernel(float* __restrict__ y, size_t count, int wait_first) {
  asm volatile("griddepcontrol.launch_dependents;");
  if (wait_first) asm volatile("griddepcontrol.wait;" ::: "memory");
  const size_t tid = blockIdx.x * (size_t)blockDim.x + threadIdx.x, nth = (size_t)gridDim.x * blockDim.x;
  size_t head = 0;
  if ((reinterpret_cast<uintptr_t>(y) & 15) == 0) {
    float4* y4 = reinterpret_cast<float4*>(y);
    const size_t n4 = count / 4;
    for (size_t i = tid; i < n4; i += nth) y4[i] = make_float4(0.f, 0.f, 0.f, 0.f);
    head = n4 * 4;
  }
  for (size_t i = head + tid; i < count; i += nth) y[i] = 0.f;
  asm volatile("griddepcontrol.wait;" ::: "memory");
}

cudaError_t launch_zero_tail(float* y, size_t count, bool wait_first, cudaStream_t stream) {
  if (count == 0) return cudaSuccess;
  size_t want = (count / 4 + 255) / 256;
  const unsigned blocks = (unsigned)std::min<size_t>(std::max<size_t>(want, 1), 148 * 8);
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(blocks);
  cfg.blockDim = dim3(256);
  cfg.stream = stream;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  cudaError_t e = cudaLaunchKernelEx(&cfg, zero_tail_kernel, y, count, (int)wait_first);
  return e != cudaSuccess ? e : cudaGetLastError();
}

}  // namespace i2cw
