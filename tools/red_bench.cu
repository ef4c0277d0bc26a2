// Epilogue write-path microbenchmark (the reduce pass's TMA reduce-adds hold
// their staging buffers ~3K cycles): the cfg2 output pattern -- y as [rows][64] fp32, a work
// unit = 12 output rows x 10 tiles x 6 output columns (q = 6 t + i), 4 warpgroups x 16 channels -- written
// by (0) TMA tensor store, (1) TMA tensor reduce-add (both staged through shared memory, 3
// buffers per warpgroup, as the fused kernel), (2) st.global.v4 and (3) red.global.add.v4.f32
// straight from registers. Prints ms and GB/s of y written per launch.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o tools/red_bench tools/red_bench.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>
#include <vector>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e_)); exit(1); } } while (0)

constexpr int kQ = 56, kNP = 128 * 56;  // cfg2: Q, N*P
constexpr int kRows = kNP * kQ;
constexpr int kCh = 64;
constexpr int kM = 6, kTS = 10, kPR = 12, kNOB = 3;  // m, tiles per row, output rows per unit
constexpr int kTiles = kTS * kPR;                   // 120 lanes
constexpr int kUnits = (kNP + kPR - 1) / kPR;

__device__ __forceinline__ unsigned smem_u32(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }

template <int MODE>
__global__ void __launch_bounds__(512, 1) epi(const __grid_constant__ CUtensorMap ymap, float* y) {
  extern __shared__ __align__(1024) float stage[];  // [4 wg][kNOB][128 rows][16 ch]
  const int g = threadIdx.x / 128, l = threadIdx.x % 128;
  float* mine = stage + (size_t)g * kNOB * 128 * 16;
  int col = 0;
  for (int u = blockIdx.x; u < kUnits; u += gridDim.x) {
    const int p0 = u * kPR;
    for (int i = 0; i < kM; ++i, ++col) {
      float v[16];
#pragma unroll
      for (int c = 0; c < 16; ++c) v[c] = 1e-3f * (c + l + i);
      const int pr = p0 + l / kTS, q = (l % kTS) * kM + i;
      const int row = pr * kQ + q;
      if (MODE >= 2) {
        if (l < kTiles && pr < kNP && q < kQ) {
          float4* dst = reinterpret_cast<float4*>(y + (size_t)row * kCh + g * 16);
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            if (MODE == 2) dst[j] = make_float4(v[4 * j], v[4 * j + 1], v[4 * j + 2], v[4 * j + 3]);
            else
              asm volatile("red.relaxed.gpu.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(dst + j),
                           "f"(v[4 * j]), "f"(v[4 * j + 1]), "f"(v[4 * j + 2]), "f"(v[4 * j + 3])
                           : "memory");
          }
        }
        continue;
      }
      const int ob = col % kNOB;
      // the store that last read this buffer must be done
      if (l == 0) asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(kNOB - 1) : "memory");
      asm volatile("bar.sync %0, 128;" ::"r"(1 + g));
      float4* stg = reinterpret_cast<float4*>(mine + (size_t)ob * 128 * 16) + l * 4;
#pragma unroll
      for (int j = 0; j < 4; ++j) stg[j] = make_float4(v[4 * j], v[4 * j + 1], v[4 * j + 2], v[4 * j + 3]);
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      asm volatile("bar.sync %0, 128;" ::"r"(1 + g));
      if (l == 0) {
        const unsigned src = smem_u32(mine + (size_t)ob * 128 * 16);
        if (MODE == 0)
          asm volatile("cp.async.bulk.tensor.3d.global.shared::cta.bulk_group [%0, {%2, %3, %4}], [%1];" ::"l"(&ymap),
                       "r"(src), "r"(g * 16), "r"(i), "r"(p0) : "memory");
        else
          asm volatile("cp.reduce.async.bulk.tensor.3d.global.shared::cta.add.tile.bulk_group [%0, {%2, %3, %4}], [%1];" ::"l"(
                           &ymap), "r"(src), "r"(g * 16), "r"(i), "r"(p0) : "memory");
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      }
    }
  }
  if (MODE < 2 && l == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

// Latency of ONE bulk tensor op from one thread (single CTA): cycles until the staging buffer
// may be reused (wait_group.read) and until the writes are complete (wait_group).
template <int RED>
__global__ void lat(const __grid_constant__ CUtensorMap ymap, long long* out, int reps) {
  extern __shared__ __align__(1024) float stage[];
  for (int i = threadIdx.x; i < kTiles * 64; i += blockDim.x) stage[i] = 1e-3f * i;
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  __syncthreads();
  if (threadIdx.x != 0) return;
  long long tr = 0, tc = 0;
  for (int r = 0; r < reps; ++r) {
    const int row = (r * 7919) % (kNP - 64);
    const long long t0 = clock64();
    if (RED)
      asm volatile("cp.reduce.async.bulk.tensor.3d.global.shared::cta.add.tile.bulk_group [%0, {%2, %3, %4}], [%1];" ::"l"(
                       &ymap), "r"(smem_u32(stage)), "r"(0), "r"(0), "r"(row) : "memory");
    else
      asm volatile("cp.async.bulk.tensor.3d.global.shared::cta.bulk_group [%0, {%2, %3, %4}], [%1];" ::"l"(&ymap),
                   "r"(smem_u32(stage)), "r"(0), "r"(0), "r"(row) : "memory");
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
    const long long t1 = clock64();
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    const long long t2 = clock64();
    tr += t1 - t0;
    tc += t2 - t0;
  }
  out[0] = tr / reps;
  out[1] = tc / reps;
}

// Throughput of k back-to-back bulk tensor ops from one CTA: `nthr` issuing threads (one per
// warpgroup, as the fused kernel's epilogue), each issuing k/nthr ops from its own staging
// buffer, then waiting for all; cycles for the whole batch.
template <int RED>
__global__ void batch(const __grid_constant__ CUtensorMap ymap, long long* out, int k, int nthr) {
  extern __shared__ __align__(1024) float stage[];
  for (int i = threadIdx.x; i < 4 * kTiles * 16; i += blockDim.x) stage[i] = 1e-3f * i;
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  __syncthreads();
  const int g = threadIdx.x / 128;
  const bool issuer = (threadIdx.x % 128) == 0 && g < nthr;
  const long long t0 = clock64();
  if (issuer) {
    for (int j = g; j < k; j += nthr) {
      const unsigned src = smem_u32(stage + (size_t)g * kTiles * 16);
      const int row = (j * 37) % (kNP - 64);
      if (RED)
        asm volatile("cp.reduce.async.bulk.tensor.3d.global.shared::cta.add.tile.bulk_group [%0, {%2, %3, %4}], [%1];" ::"l"(
                         &ymap), "r"(src), "r"(g * 16), "r"(j % kM), "r"(row) : "memory");
      else
        asm volatile("cp.async.bulk.tensor.3d.global.shared::cta.bulk_group [%0, {%2, %3, %4}], [%1];" ::"l"(&ymap),
                     "r"(src), "r"(g * 16), "r"(j % kM), "r"(row) : "memory");
      asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    }
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
  }
  __syncthreads();
  if (threadIdx.x == 0) out[0] = clock64() - t0;
}

int main() {
  float* y;
  CK(cudaMalloc(&y, (size_t)kRows * kCh * 4));
  CK(cudaMemset(y, 0, (size_t)kRows * kCh * 4));
  float* flush;
  const size_t fb = 256ull << 20;
  CK(cudaMalloc(&flush, fb));
  // y map: dims {64 ch, Q, N*P}, box {16, TS*m, 12} with element stride {1, m, 1} (one output
  // column of a unit: 120 rows of 64 bytes), as the fused kernel's
  CUtensorMap map;
  cuuint64_t dims[3] = {kCh, kQ, kNP};
  cuuint64_t strides[2] = {kCh * 4, kCh * 4 * kQ};
  cuuint32_t box[3] = {16, kTS * kM, kPR};
  cuuint32_t es[3] = {1, kM, 1};
  CUresult r = cuTensorMapEncodeTiled(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, y, dims, strides, box, es,
                                      CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                                      CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) { printf("encode failed %d\n", (int)r); return 1; }
  const int smem = 4 * kNOB * 128 * 16 * 4;
  auto run = [&](auto kern, const char* name) {
    CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    std::vector<float> ts;
    for (int it = 0; it < 12; ++it) {
      CK(cudaMemsetAsync(flush, it, fb));
      cudaEventRecord(a);
      kern<<<148, 512, smem>>>(map, y);
      cudaEventRecord(b);
      CK(cudaEventSynchronize(b));
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      if (it >= 2) ts.push_back(ms);
    }
    float best = 1e9, sum = 0;
    for (float t : ts) { best = t < best ? t : best; sum += t; }
    const double gb = (double)kRows * kCh * 4 / 1e9;
    printf("%-28s min %.1f us  mean %.1f us  %.0f GB/s (y bytes / min time)\n", name, best * 1e3, sum / ts.size() * 1e3,
           gb / (best * 1e-3));
  };
  run(epi<0>, "TMA tensor store");
  run(epi<1>, "TMA tensor reduce-add");
  run(epi<2>, "st.global.v4 (registers)");
  run(epi<3>, "red.global.add.v4 (registers)");
  // single-op latencies for box shapes: 16 ch (the kernel's) or 64 ch, q stride m (the kernel's)
  // or contiguous q
  long long* dout;
  CK(cudaMalloc(&dout, 16));
  const int lsm = 128 * 64 * 4;
  CK(cudaFuncSetAttribute(lat<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, lsm));
  CK(cudaFuncSetAttribute(lat<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, lsm));
  for (int shape = 0; shape < 4; ++shape) {
    CUtensorMap m2;
    cuuint32_t bx[3] = {(cuuint32_t)(shape & 1 ? 64 : 16), (cuuint32_t)(shape & 2 ? kTS : kTS * kM), kPR};
    cuuint32_t e2[3] = {1, (cuuint32_t)(shape & 2 ? 1 : kM), 1};
    if (cuTensorMapEncodeTiled(&m2, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, y, dims, strides, bx, e2,
                               CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                               CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS) {
      printf("encode failed\n");
      return 1;
    }
    for (int red = 0; red < 2; ++red) {
      long long h[2];
      if (red) lat<1><<<1, 128, lsm>>>(m2, dout, 200);
      else lat<0><<<1, 128, lsm>>>(m2, dout, 200);
      CK(cudaMemcpy(h, dout, 16, cudaMemcpyDeviceToHost));
      printf("latency %-8s box %2d ch x 120 rows, q stride %d: read-done %lld cycles, complete %lld cycles (%d bytes)\n",
             red ? "reduce" : "store", (int)bx[0], (int)e2[1], h[0], h[1], (int)(bx[0] * kTiles * 4));
    }
  }
  CK(cudaFuncSetAttribute(batch<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, 4 * kTiles * 16 * 4));
  CK(cudaFuncSetAttribute(batch<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, 4 * kTiles * 16 * 4));
  for (int red = 0; red < 2; ++red)
    for (int nthr : {1, 4})
      for (int k : {1, 4, 8, 24, 48}) {
        long long h = 0;
        for (int rep = 0; rep < 3; ++rep) {  // last of 3 (warm)
          if (red) batch<1><<<1, 512, 4 * kTiles * 16 * 4>>>(map, dout, k, nthr);
          else batch<0><<<1, 512, 4 * kTiles * 16 * 4>>>(map, dout, k, nthr);
          CK(cudaMemcpy(&h, dout, 8, cudaMemcpyDeviceToHost));
        }
        printf("batch %-6s %d issuers, %2d ops of 7680 B: %6lld cycles, %.1f B/clk\n", red ? "reduce" : "store", nthr, k,
               h, 7680.0 * k / h);
      }
  CK(cudaGetLastError());
  return 0;
}
