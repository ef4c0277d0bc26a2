// Tools only: checks the strip kernel's TMA views on the GPU -- x as (C, W, H, N) with a
// (8, 9, 32, 1) box and 32B swizzle (where does element (c, col, row) land in shared memory?
// A (C, H, W, N) view with non-monotonic strides encodes fine but faults on load),
// and the y store view (K, P, Q, N) with a (16, ROWS, 4 tiles at element stride m, 1) box and
// 64B swizzle, including boxes that start at a negative q (clipped).
// Build: nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -I paper_conf_icpp_zhangzxyw24_b200/csrc tools/tma_view_test.cu -o tools/tma_view_test -lcuda
#include <cuda.h>
#include <cstdio>
#include <cstring>
#include <vector>

#include "common.cuh"

using namespace i2cw;

__global__ void load_kernel(const __grid_constant__ CUtensorMap xmap, int c0, int h0, int w0, int n0, float* out) {
  __shared__ __align__(1024) uint8_t box[9216];
  __shared__ uint64_t bar;
  if (threadIdx.x == 0) { mbar_init(&bar, 1); fence_mbar_init(); }
  __syncthreads();
  if (threadIdx.x == 0) {
    mbar_expect_tx(&bar, 9216);
    tma_load_4d(box, &xmap, &bar, c0, w0, h0, n0);
  }
  mbar_wait(&bar, 0);
  for (int i = threadIdx.x; i < 2304; i += blockDim.x) out[i] = reinterpret_cast<float*>(box)[i];
}

__global__ void store_kernel(const __grid_constant__ CUtensorMap ymap, int rows, int k0, int p0, int q0, int n0) {
  __shared__ __align__(1024) float box[16 * 32 * 4];
  for (int i = threadIdx.x; i < 16 * rows * 4; i += blockDim.x) box[i] = 1000.f + i;
  fence_proxy_async_smem();
  __syncthreads();
  if (threadIdx.x == 0) {
    tma_store_4d(&ymap, box, k0, p0, q0, n0);
    bulk_commit_group();
    bulk_wait_group_all();
  }
}

typedef CUresult (*Enc)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                        const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                        CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int main() {
  const int N = 2, H = 40, W = 13, C = 16;
  std::vector<float> hx((size_t)N * H * W * C);
  for (int n = 0; n < N; ++n)
    for (int h = 0; h < H; ++h)
      for (int w = 0; w < W; ++w)
        for (int c = 0; c < C; ++c) hx[(((size_t)n * H + h) * W + w) * C + c] = n * 1e6f + h * 1e4f + w * 100.f + c;
  float *dx, *dout;
  cudaMalloc(&dx, hx.size() * 4);
  cudaMemcpy(dx, hx.data(), hx.size() * 4, cudaMemcpyHostToDevice);
  cudaMalloc(&dout, 2304 * 4);
  void* p = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q);
  Enc enc = (Enc)p;
  CUtensorMap xm;
  cuuint64_t dims[4] = {(cuuint64_t)C, (cuuint64_t)W, (cuuint64_t)H, (cuuint64_t)N};
  cuuint64_t strides[3] = {(cuuint64_t)C * 4, (cuuint64_t)W * C * 4, (cuuint64_t)H * W * C * 4};
  cuuint32_t box[4] = {8, 9, 32, 1};
  cuuint32_t es[4] = {1, 1, 1, 1};
  CUresult r = enc(&xm, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, dx, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   CU_TENSOR_MAP_SWIZZLE_32B, CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  printf("x map encode: %d\n", (int)r);
  load_kernel<<<1, 128>>>(xm, 8, -1, 2, 1, dout);
  cudaError_t e = cudaDeviceSynchronize();
  printf("load: %s\n", cudaGetErrorString(e));
  if (e != cudaSuccess) return 1;
  std::vector<float> ho(2304);
  cudaMemcpy(ho.data(), dout, 2304 * 4, cudaMemcpyDeviceToHost);
  // check: element (c, col, row) expected at physical offset of the [row][col][c] image with the
  // 16-byte chunk bit 4 XOR address bit 7
  int bad = 0;
  for (int col = 0; col < 9; ++col)
    for (int row = 0; row < 32; ++row)
      for (int c = 0; c < 8; ++c) {
        const int h = -1 + row, w = 2 + col, cc = 8 + c;
        const float want = (h < 0 || h >= H || w >= W) ? 0.f : 1e6f + h * 1e4f + w * 100.f + cc;
        const uint32_t off = (uint32_t)((row * 9 + col) * 32 + c * 4);
        const uint32_t phys = off ^ ((off >> 3) & 16u);
        if (ho[phys / 4] != want) {
          if (bad < 5) printf("  mismatch col %d row %d c %d: got %.0f want %.0f\n", col, row, c, ho[phys / 4], want);
          ++bad;
        }
      }
  printf("x box layout check: %d mismatches\n", bad);
  // y store view
  const int P = 40, Q = 13, K = 32, m = 6, ROWS = 20;
  float* dy;
  cudaMalloc(&dy, (size_t)N * P * Q * K * 4);
  cudaMemset(dy, 0, (size_t)N * P * Q * K * 4);
  CUtensorMap ym;
  cuuint64_t ydims[4] = {(cuuint64_t)K, (cuuint64_t)P, (cuuint64_t)Q, (cuuint64_t)N};
  cuuint64_t ystr[3] = {(cuuint64_t)Q * K * 4, (cuuint64_t)K * 4, (cuuint64_t)P * Q * K * 4};
  cuuint32_t ybox[4] = {16, (cuuint32_t)ROWS, (cuuint32_t)(4 * m), 1};
  cuuint32_t yes[4] = {1, 1, (cuuint32_t)m, 1};
  r = enc(&ym, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, dy, ydims, ystr, ybox, yes, CU_TENSOR_MAP_INTERLEAVE_NONE,
          CU_TENSOR_MAP_SWIZZLE_64B, CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  printf("y map encode: %d\n", (int)r);
  for (int q0 : {1, -17}) {
    store_kernel<<<1, 128>>>(ym, ROWS, 16, 20, q0, 1);
    e = cudaDeviceSynchronize();
    printf("store q0 = %d: %s\n", q0, cudaGetErrorString(e));
    if (e != cudaSuccess) return 1;
  }
  std::vector<float> hy((size_t)N * P * Q * K);
  cudaMemcpy(hy.data(), dy, hy.size() * 4, cudaMemcpyDeviceToHost);
  int written = 0;
  for (int pp = 0; pp < P; ++pp)
    for (int qq = 0; qq < Q; ++qq)
      for (int k = 0; k < K; ++k)
        if (hy[(((size_t)1 * P + pp) * Q + qq) * K + k] != 0.f) {
          if (written < 3 || (qq == 1 && pp == 20 && k == 16))
            printf("  y[1][%d][%d][%d] = %.0f\n", pp, qq, k, hy[(((size_t)1 * P + pp) * Q + qq) * K + k]);
          ++written;
        }
  printf("y elements written: %d (expect q in {1, 7} and {1, 7} again for the clipped box: %d)\n", written, 2 * 20 * 16);
  return 0;
}
