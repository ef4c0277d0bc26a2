// Tools only: tcgen05.shift.cta_group::2 semantics on a CTA pair (cluster of 2): does the leader's
// shift move the rows of BOTH CTAs' tensor memory, and in order after a cta_group::2 MMA?
// Build: nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -I paper_conf_icpp_zhangzxyw24_b200/csrc tools/shift2_bench.cu -o tools/shift2_bench
#include <cstdio>
#include "common.cuh"
using namespace i2cw;

__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(128, 1) pair_kernel(float* out, int nshift) {
  __shared__ __align__(1024) float bsm[64 * 8];
  __shared__ uint64_t bar;
  __shared__ uint32_t tslot;
  const int warp = threadIdx.x / 32, l = threadIdx.x;
  const uint32_t rank = cluster_ctarank();
  for (int i = threadIdx.x; i < 64 * 8; i += blockDim.x) bsm[i] = 1.f;
  if (threadIdx.x == 0) { mbar_init(&bar, 1); fence_mbar_init(); }
  if (warp == 0) { tmem_alloc2(&tslot, 512); tmem_relinquish2(); }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  tc_fence_before();
  cluster_sync_all();
  tc_fence_after();
  const uint32_t tbase = tslot;
  const uint32_t lane_addr = tbase + ((uint32_t)(l & ~31) << 16);
  // A (cols 64..71) = 1000*rank + lane, D (cols 0..15) from MMA(A) + MMA(shift(A))
  { float a8[8]; for (int e = 0; e < 8; ++e) a8[e] = 1000.f * rank + l; tmem_st_x8(lane_addr + 64, a8); }
  tmem_wait_st();
  tc_fence_before();
  cluster_sync_all();
  tc_fence_after();
  if (rank == 0 && threadIdx.x == 0) {
    constexpr uint32_t idesc = idesc_tf32(256, 32);  // M = 256 over the pair, N = 32 (16 per CTA)
    const uint64_t bdesc = umma_desc_kmajor_noswizzle(smem_u32(bsm), 16 * 16, 128);
    mma2_tf32_ts(tbase, tbase + 64, bdesc, idesc, 0u);
    for (int s = 0; s < nshift; ++s) asm volatile("tcgen05.shift.cta_group::2.down [%0];" ::"r"(tbase + 64) : "memory");
    mma2_tf32_ts(tbase, tbase + 64, bdesc, idesc, 1u);
    mma_commit2(&bar);
  }
  mbar_wait_cluster(&bar, 0);
  tc_fence_after();
  float v[8];
  tmem_ld_x8(lane_addr, v);
  tmem_wait_ld();
  out[rank * 256 + l] = v[0];
  tmem_ld_x8(lane_addr + 64, v);
  tmem_wait_ld();
  out[rank * 256 + 128 + l] = v[0];
  tc_fence_before();
  cluster_sync_all();
  if (warp == 0) { tc_fence_after(); tmem_dealloc2(tbase, 512); }
}

int main() {
  float* d;
  cudaMalloc(&d, 512 * 4);
  static float h[512];
  for (int ns = 0; ns <= 1; ++ns) {
    cudaMemset(d, 0, 512 * 4);
    pair_kernel<<<2, 128>>>(d, ns);
    cudaError_t e = cudaDeviceSynchronize();
    cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    printf("== %d shift(s) (%s)\n", ns, cudaGetErrorString(e));
    for (int r = 0; r < 2; ++r) {
      printf("  CTA %d D[l] (l=0,1,30,31,32,127): ", r);
      for (int l : {0, 1, 30, 31, 32, 127}) printf("%.0f ", h[r * 256 + l]);
      printf(" | A after: ");
      for (int l : {0, 1, 30, 31, 32, 127}) printf("%.0f ", h[r * 256 + 128 + l]);
      printf("\n");
    }
  }
  return 0;
}
