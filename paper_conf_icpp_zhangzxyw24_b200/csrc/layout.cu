// Layout adapters for the NCHW entry points (the paper's portability
// remark PAPER.md:4699-4703): batched 2D transposes through shared memory, so an NCHW / OIHW
// caller reaches the NHWC fused kernel. out[b][c][r] = in[b][r][c] for a [B][rows][cols] input;
// NCHW -> NHWC is [N][C][H*W] -> [N][H*W][C], NHWC -> NCHW is [N][P*Q][K] -> [N][K][P*Q], and
// the OIHW filter [K][C][R*S] -> KRSC [K][R*S][C]. HBM-bound copies: 32x32 tiles, coalesced
// reads and writes, padded shared rows (no bank conflicts). Also the K-slice combine (ksum).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>

namespace i2cw {

__global__ void transpose_kernel(const float* __restrict__ in, float* __restrict__ out, int rows, int cols) {
  __shared__ float tile[32][33];
  const size_t b = blockIdx.z;
  const float* src = in + b * (size_t)rows * cols;
  float* dst = out + b * (size_t)rows * cols;
  const int c0 = blockIdx.x * 32, r0 = blockIdx.y * 32;
#pragma unroll
  for (int j = 0; j < 32; j += 8) {
    const int r = r0 + threadIdx.y + j, c = c0 + threadIdx.x;
    if (r < rows && c < cols) tile[threadIdx.y + j][threadIdx.x] = src[(size_t)r * cols + c];
  }
  __syncthreads();
#pragma unroll
  for (int j = 0; j < 32; j += 8) {
    const int c = c0 + threadIdx.y + j, r = r0 + threadIdx.x;
    if (r < rows && c < cols) dst[(size_t)c * rows + r] = tile[threadIdx.x][threadIdx.y + j];
  }
}

// batched transpose of B [rows][cols] matrices (gridDim.z <= 65535 batches per launch)
cudaError_t launch_transpose(const float* in, float* out, int B, int rows, int cols, cudaStream_t stream) {
  const dim3 block(32, 8);
  for (int b0 = 0; b0 < B; b0 += 65535) {
    const int nb = std::min(65535, B - b0);
    const dim3 grid((cols + 31) / 32, (rows + 31) / 32, nb);
    transpose_kernel<<<grid, block, 0, stream>>>(in + (size_t)b0 * rows * cols, out + (size_t)b0 * rows * cols, rows,
                                                 cols);
    const cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

// K-slice combine (api.cu run_fused, small grids): y[i] = (((y[i] + s_0[i]) + s_1[i]) + ...), a
// fixed summation order (deterministic). HBM-bound, grid-stride; float4 when y is 16-byte
// aligned (slices are `stride` floats apart, stride a multiple of 64).
template <bool V4>
__global__ void ksum_kernel(float* __restrict__ y, const float* __restrict__ sl, int nsl, size_t count,
                            size_t stride) {
  const size_t tid = blockIdx.x * (size_t)blockDim.x + threadIdx.x, nth = (size_t)gridDim.x * blockDim.x;
  size_t done = 0;
  if (V4) {
    const size_t n4 = count / 4, st4 = stride / 4;
    float4* y4 = reinterpret_cast<float4*>(y);
    const float4* s4 = reinterpret_cast<const float4*>(sl);
    for (size_t i = tid; i < n4; i += nth) {
      float4 a = y4[i];
      for (int k = 0; k < nsl; ++k) {
        const float4 b = s4[(size_t)k * st4 + i];
        a.x += b.x; a.y += b.y; a.z += b.z; a.w += b.w;
      }
      y4[i] = a;
    }
    done = n4 * 4;
  }
  for (size_t i = done + tid; i < count; i += nth) {
    float a = y[i];
    for (int k = 0; k < nsl; ++k) a += sl[(size_t)k * stride + i];
    y[i] = a;
  }
}

cudaError_t launch_ksum(float* y, const float* slices, int nslices, size_t count, size_t stride, cudaStream_t stream) {
  if (nslices <= 0 || count == 0) return cudaSuccess;
  const bool v4 = (reinterpret_cast<uintptr_t>(y) & 15) == 0;
  const size_t want = ((v4 ? count / 4 : count) + 255) / 256;
  const unsigned blocks = (unsigned)std::min<size_t>(std::max<size_t>(want, 1), 148 * 8);
  if (v4) ksum_kernel<true><<<blocks, 256, 0, stream>>>(y, slices, nslices, count, stride);
  else ksum_kernel<false><<<blocks, 256, 0, stream>>>(y, slices, nslices, count, stride);
  return cudaGetLastError();
}

}  // namespace i2cw
