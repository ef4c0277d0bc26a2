// Layout adapters for the NCHW entry points (the paper's portability
// remark PAPER.md:4699-4703): batched 2D transposes through shared memory, so an NCHW / OIHW
// caller reaches the NHWC fused kernel. out[b][c][r] = in[b][r][c] for a [B][rows][cols] input;
// NCHW -> NHWC is [N][C][H*W] -> [N][H*W][C], NHWC -> NCHW is [N][P*Q][K] -> [N][K][P*Q], and
// the OIHW filter [K][C][R*S] -> KRSC [K][R*S][C]. HBM-bound copies: 32x32 tiles, coalesced
// reads and writes, padded shared rows (no bank conflicts).
#include <cuda_runtime.h>

#include <algorithm>

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

}  // namespace i2cw
