// Microbenchmark (tools only): latencies of the synchronisation hops of the fused kernel.
//  A) ping-pong between two warps through two mbarriers (arrive -> try_wait wake), round trip
//  B) same with the waiter using try_wait + 64 ns suspend hint (mbar_wait_cluster)
//  C) tcgen05.commit (no MMA in flight) -> mbarrier completion seen by the issuing thread
//  D) 16 x tcgen05.st.32x32b.x4 + tcgen05.wait::st by one warp
//  E) ping-pong where the "reply" is a tcgen05.commit after 3 UMMAs 128x64x8 (TS)
#include <cstdio>
#include "common.cuh"
using namespace i2cw;

__global__ void __launch_bounds__(128, 1) kern(int iters, long long* out) {
  __shared__ __align__(1024) uint8_t smem[16 * 1024];
  __shared__ uint64_t bar[4];
  __shared__ uint32_t tslot;
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  for (int i = threadIdx.x; i < 16 * 1024 / 4; i += blockDim.x) reinterpret_cast<float*>(smem)[i] = 0.f;
  if (threadIdx.x == 0) { for (int i = 0; i < 4; ++i) mbar_init(&bar[i], 1); fence_mbar_init(); }
  if (warp == 0) { tmem_alloc(&tslot, 512); tmem_relinquish(); }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  tc_fence_before(); __syncthreads(); tc_fence_after();
  const uint32_t tbase = tslot;
  // A / B: warp 0 lane 0 pings bar[0], warp 1 lane 0 waits bar[0] and pongs bar[1]
  for (int mode = 0; mode < 2; ++mode) {
    __syncthreads();
    if (threadIdx.x == 0) { mbar_init(&bar[0], 1); mbar_init(&bar[1], 1); fence_mbar_init(); }
    __syncthreads();
    if (warp == 0 && lane == 0) {
      long long t0 = clock64();
      for (int i = 0; i < iters; ++i) {
        mbar_arrive(&bar[0]);
        if (mode == 0) mbar_wait(&bar[1], i & 1); else mbar_wait_cluster(&bar[1], i & 1);
      }
      out[mode] = (clock64() - t0) / iters;
    } else if (warp == 1 && lane == 0) {
      for (int i = 0; i < iters; ++i) {
        if (mode == 0) mbar_wait(&bar[0], i & 1); else mbar_wait_cluster(&bar[0], i & 1);
        mbar_arrive(&bar[1]);
      }
    }
    __syncthreads();
  }
  // C: commit -> wait by the same thread (nothing in flight)
  if (threadIdx.x == 0) {
    mbar_init(&bar[2], 1); fence_mbar_init();
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) { mma_commit(&bar[2]); mbar_wait_cluster(&bar[2], i & 1); }
    out[2] = (clock64() - t0) / iters;
  }
  __syncthreads();
  // D: 16 x STTM.x4 + wait::st (warp 0)
  if (warp == 0) {
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
#pragma unroll
      for (int c = 0; c < 16; ++c) tmem_st_x4(tbase + 256 + c * 4, 1.f, 2.f, 3.f, 4.f);
      tmem_wait_st();
    }
    if (lane == 0) out[3] = (clock64() - t0) / iters;
  }
  __syncthreads();
  // E: 3 UMMAs + commit -> wait (single thread)
  if (threadIdx.x == 0) {
    mbar_init(&bar[3], 1); fence_mbar_init();
    constexpr uint32_t idesc = idesc_tf32(128, 64);
    const uint64_t bdesc = umma_desc_kmajor_noswizzle(smem_u32(smem), 64 * 16, 128);
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
      for (int j = 0; j < 3; ++j) mma_tf32_ts(tbase, tbase + 384, bdesc, idesc, 1u);
      mma_commit(&bar[3]);
      mbar_wait_cluster(&bar[3], i & 1);
    }
    out[4] = (clock64() - t0) / iters;
  }
  tc_fence_before(); __syncthreads();
  if (warp == 0) { tc_fence_after(); tmem_dealloc(tbase, 512); }
}

int main() {
  long long* d; cudaMalloc(&d, 8 * 8);
  kern<<<1, 128>>>(10, d);
  kern<<<1, 128>>>(2000, d);
  cudaError_t e = cudaDeviceSynchronize();
  long long h[8]; cudaMemcpy(h, d, 8 * 8, cudaMemcpyDeviceToHost);
  printf("[%s]\n", cudaGetErrorString(e));
  printf("A mbarrier ping-pong round trip (try_wait default):      %lld cycles\n", h[0]);
  printf("B mbarrier ping-pong round trip (try_wait 64ns hint):    %lld cycles\n", h[1]);
  printf("C tcgen05.commit -> wait, nothing in flight:             %lld cycles\n", h[2]);
  printf("D 16 x tcgen05.st.32x32b.x4 + wait::st (one warp):       %lld cycles\n", h[3]);
  printf("E 3 x UMMA 128x64x8 + commit -> wait:                    %lld cycles\n", h[4]);
  return 0;
}
