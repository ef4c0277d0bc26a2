// Microbenchmark (tools only, not product): throughput of tcgen05.mma kind::tf32
// M=128, K=8 for several N, A from TMEM ("TS") or shared memory ("SS"), issued by
// NI warps (one elected lane each) into disjoint accumulators, one CTA per SM.
// Build: nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -I paper_conf_icpp_zhangzxyw24_b200/csrc tools/mma_bench.cu -o tools/mma_bench
#include <cstdio>
#include <cstdlib>

#include "common.cuh"

using namespace i2cw;

template <int N, bool TS, int NI, bool VARY_A, bool ROT, bool WARP>
__global__ void __launch_bounds__(128, 1) mma_kernel(int iters, unsigned long long* out) {
  __shared__ __align__(1024) uint8_t smem[40 * 1024];
  __shared__ uint64_t bar[4];
  __shared__ uint32_t tslot;
  const int warp = threadIdx.x / 32;
  for (int i = threadIdx.x; i < 40 * 1024 / 4; i += blockDim.x) reinterpret_cast<float*>(smem)[i] = 0.f;
  if (threadIdx.x == 0) { for (int i = 0; i < 4; ++i) mbar_init(&bar[i], 1); fence_mbar_init(); }
  if (warp == 0) { tmem_alloc(&tslot, 512); tmem_relinquish(); }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tbase = tslot;
  constexpr int PER = 8;
  if (warp < NI && (WARP || (threadIdx.x % 32) == 0)) {
    constexpr uint32_t idesc = idesc_tf32(128, N);
    const uint32_t sb = smem_u32(smem);
    const uint64_t bdesc = umma_desc_kmajor_noswizzle(sb, N * 16, 128);
    const uint64_t adesc = umma_desc_kmajor_noswizzle(sb + 32768, 128 * 16, 128);
    const uint32_t dcol0 = tbase + warp * N;
    const unsigned long long t0 = clock64();
    for (int it = 0; it < iters; ++it) {
#pragma unroll
      for (int j = 0; j < PER; ++j) {
        const uint32_t acol = tbase + 384 + (VARY_A ? (j % 4) * 8 : 0);
        const uint32_t dcol = ROT ? tbase + (j % 4) * N : dcol0;
        if constexpr (TS && WARP) mma_tf32_ts_warp(dcol, acol, bdesc, idesc, 1u);
        else if constexpr (TS) mma_tf32_ts(dcol, acol, bdesc, idesc, 1u);
        else mma_tf32_ss(dcol, adesc, bdesc, idesc, 1u);
      }
    }
    if constexpr (WARP) mma_commit_warp(&bar[warp]);
    else mma_commit(&bar[warp]);
    mbar_wait(&bar[warp], 0);
    const unsigned long long t1 = clock64();
    if (warp == 0 && (threadIdx.x % 32) == 0) out[blockIdx.x] = t1 - t0;
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) { tc_fence_after(); tmem_dealloc(tbase, 512); }
}

template <int N, bool TS, int NI, bool VARY_A = true, bool ROT = false, bool WARP = false>
void run(int nsm) {
  unsigned long long* d;
  cudaMalloc(&d, nsm * sizeof(unsigned long long));
  const int iters = 1000, per = 8;
  mma_kernel<N, TS, NI, VARY_A, ROT, WARP><<<nsm, 128>>>(10, d);
  cudaEvent_t a, b;
  cudaEventCreate(&a); cudaEventCreate(&b);
  cudaEventRecord(a);
  mma_kernel<N, TS, NI, VARY_A, ROT, WARP><<<nsm, 128>>>(iters, d);
  cudaEventRecord(b);
  cudaError_t e = cudaDeviceSynchronize();
  float ms = 0;
  cudaEventElapsedTime(&ms, a, b);
  unsigned long long h[148];
  cudaMemcpy(h, d, nsm * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
  const double total_mma = (double)iters * per * NI;
  double cyc = (double)h[0] / total_mma;
  double flops = 2.0 * 128 * N * 8 * total_mma * nsm;
  printf("%s%s N=%3d issuers=%d varyA=%d rotD=%d: %6.1f cycles/MMA (ideal %d)  %7.1f TFLOP/s tf32  [%s]\n", TS ? "TS" : "SS", WARP ? "(warp-uniform)" : "", N,
         NI, (int)VARY_A, (int)ROT, cyc, N / 2, flops / (ms * 1e-3) / 1e12, cudaGetErrorString(e));
  cudaFree(d);
}

int main() {
  const int nsm = 148;
  run<64, true, 1, true, true, true>(nsm); run<64, true, 2, true, true, true>(nsm);
  run<64, true, 1, true, false, true>(nsm); run<64, true, 2, true, false, true>(nsm);
  run<64, true, 1, true, true>(nsm); run<32, true, 1, true, true>(nsm); run<64, true, 1>(nsm); run<64, true, 1, false>(nsm); run<64, true, 2>(nsm); run<64, true, 4>(nsm);
  run<32, true, 1>(nsm); run<32, true, 4>(nsm);
  run<128, true, 1>(nsm); run<128, true, 2>(nsm);
  run<64, false, 1>(nsm); run<64, false, 4>(nsm);
  run<128, false, 1>(nsm); run<128, false, 2>(nsm);
  run<256, true, 1>(nsm);
  return 0;
}
