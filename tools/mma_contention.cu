// Microbenchmark (tools only): tcgen05.mma kind::tf32 TS-mode 128x64x8 throughput (4 issuer
// warps, disjoint accumulators) while NL other warps stream LDS.128 from shared memory
// and/or STTM into TMEM. Question: does shared-memory / TMEM traffic slow the tensor pipe?
#include <cstdio>
#include "common.cuh"
using namespace i2cw;

template <int NL, int MODE>  // MODE 0: LDS stress, 1: STTM stress, 2: both
__global__ void __launch_bounds__(128 + NL * 32, 1) kern(int iters, unsigned long long* out, float* sink) {
  __shared__ __align__(1024) uint8_t smem[40 * 1024];
  __shared__ uint64_t bar[4];
  __shared__ uint32_t tslot;
  __shared__ volatile int stop;
  const int warp = threadIdx.x / 32;
  for (int i = threadIdx.x; i < 40 * 1024 / 4; i += blockDim.x) reinterpret_cast<float*>(smem)[i] = 0.f;
  if (threadIdx.x == 0) { for (int i = 0; i < 4; ++i) mbar_init(&bar[i], 1); stop = 0; fence_mbar_init(); }
  if (warp == 0) { tmem_alloc(&tslot, 512); tmem_relinquish(); }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  tc_fence_before(); __syncthreads(); tc_fence_after();
  const uint32_t tbase = tslot;
  if (warp < 4) {
    if ((threadIdx.x % 32) == 0) {
      constexpr uint32_t idesc = idesc_tf32(128, 64);
      const uint64_t bdesc = umma_desc_kmajor_noswizzle(smem_u32(smem), 64 * 16, 128);
      const unsigned long long t0 = clock64();
      for (int it = 0; it < iters; ++it)
#pragma unroll
        for (int j = 0; j < 8; ++j) mma_tf32_ts(tbase + warp * 64, tbase + 384 + (j % 4) * 8, bdesc, idesc, 1u);
      mma_commit(&bar[warp]);
      mbar_wait(&bar[warp], 0);
      if (warp == 0) { out[blockIdx.x] = clock64() - t0; stop = 1; }
    }
    __syncwarp();
  } else if (NL > 0) {
    float acc = 0.f;
    const float4* src = reinterpret_cast<const float4*>(smem + 16384);
    const int l = threadIdx.x % 32;
    int k = 0;
    while (!stop) {
      if (MODE == 0 || MODE == 2) {
#pragma unroll
        for (int j = 0; j < 16; ++j) { float4 v = src[((k + j) * 32 + l) & 1023]; acc += v.x + v.w; }
      }
      if (MODE == 1 || MODE == 2) {
        const uint32_t ta = tbase + (((warp % 4) * 32) << 16) + 448;
#pragma unroll
        for (int j = 0; j < 8; ++j) tmem_st_x4(ta + (j % 4) * 4, acc, acc, acc, acc);
        tmem_wait_st();
      }
      k += 16;
    }
    if (acc == 12345.f) sink[0] = acc;
  }
  tc_fence_before(); __syncthreads();
  if (warp == 0) { tc_fence_after(); tmem_dealloc(tbase, 512); }
}

template <int NL, int MODE>
void run(const char* name) {
  unsigned long long* d; float* s;
  cudaMalloc(&d, 148 * 8); cudaMalloc(&s, 4);
  kern<NL, MODE><<<148, 128 + NL * 32>>>(10, d, s);
  const int iters = 500;
  kern<NL, MODE><<<148, 128 + NL * 32>>>(iters, d, s);
  cudaError_t e = cudaDeviceSynchronize();
  unsigned long long h; cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost);
  printf("%-28s %6.1f cycles per MMA (4 issuers, 128x64x8 TS)  [%s]\n", name, (double)h / (iters * 8 * 4),
         cudaGetErrorString(e));
  cudaFree(d); cudaFree(s);
}
int main() {
  run<0, 0>("no stress");
  run<4, 0>("LDS stress 4 warps");
  run<8, 0>("LDS stress 8 warps");
  run<16, 0>("LDS stress 16 warps");
  run<8, 1>("STTM stress 8 warps");
  run<8, 2>("LDS+STTM stress 8 warps");
  return 0;
}
