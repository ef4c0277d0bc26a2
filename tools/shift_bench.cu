// Microbenchmark (tools only, not product): semantics, ordering and cost of tcgen05.shift
// (TMEM rows shifted down by one lane), the primitive that lets one input-row transform serve
// all R filter rows of a chunk.
// Build: nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -I paper_conf_icpp_zhangzxyw24_b200/csrc tools/shift_bench.cu -o tools/shift_bench
#include <cstdio>
#include <cstdlib>

#include "common.cuh"

using namespace i2cw;

__device__ __forceinline__ void tmem_shift_down(uint32_t taddr) {
  asm volatile("tcgen05.shift.cta_group::1.down [%0];" ::"r"(taddr) : "memory");
}

// mode 0: semantics. Lane l stores l*1000 + c in columns c < 48; thread 0 shifts the 32-byte
// element at (lane_off, col); everyone reads columns < 48 back.
// mode 1: ordering. A (cols 64..71) = lane id, B (smem, N=16) = 1; MMA, shift A, MMA into D
// (cols 0..15): D = 8*(A_before + A_after).
// mode 2: cost. nshift shifts (cycling over 8 column blocks) then commit; cycles reported.
// mode 3: cost of MMAs (12 per step, N=64) with 8 shifts between every 12 MMAs vs none.
__global__ void __launch_bounds__(128, 1) shift_kernel(int mode, int lane_off, int col, int nshift, float* out,
                                                       unsigned long long* cyc) {
  __shared__ __align__(1024) float bsm[64 * 8];
  __shared__ uint64_t bar;
  __shared__ uint32_t tslot;
  const int warp = threadIdx.x / 32, l = threadIdx.x;
  for (int i = threadIdx.x; i < 64 * 8; i += blockDim.x) bsm[i] = 1.f;
  if (threadIdx.x == 0) { mbar_init(&bar, 1); fence_mbar_init(); }
  if (warp == 0) { tmem_alloc(&tslot, 512); tmem_relinquish(); }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tbase = tslot;
  const uint32_t lane_addr = tbase + ((uint32_t)(l & ~31) << 16);
  if (mode == 0) {
    for (int c = 0; c < 48; c += 4) tmem_st_x4(lane_addr + c, l * 1000.f + c, l * 1000.f + c + 1, l * 1000.f + c + 2, l * 1000.f + c + 3);
    tmem_wait_st();
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    if (threadIdx.x == 0) {
      tmem_shift_down(tbase + ((uint32_t)lane_off << 16) + (uint32_t)col);
      mma_commit(&bar);
    }
    mbar_wait(&bar, 0);
    tc_fence_after();
    for (int c = 0; c < 48; c += 8) {
      float v[8];
      tmem_ld_x8(lane_addr + c, v);
      tmem_wait_ld();
      for (int e = 0; e < 8; ++e) out[l * 48 + c + e] = v[e];
    }
  } else if (mode == 1) {
    { float a8[8]; for (int e = 0; e < 8; ++e) a8[e] = (float)l; tmem_st_x8(lane_addr + 64, a8); }
    tmem_wait_st();
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    if (threadIdx.x == 0) {
      constexpr uint32_t idesc = idesc_tf32(128, 16);
      const uint64_t bdesc = umma_desc_kmajor_noswizzle(smem_u32(bsm), 16 * 16, 128);
      mma_tf32_ts(tbase, tbase + 64, bdesc, idesc, 0u);
      for (int s = 0; s < nshift; ++s) tmem_shift_down(tbase + 64);
      mma_tf32_ts(tbase, tbase + 64, bdesc, idesc, 1u);
      mma_commit(&bar);
    }
    mbar_wait(&bar, 0);
    tc_fence_after();
    float v[8];
    tmem_ld_x8(lane_addr, v);
    tmem_wait_ld();
    out[l] = v[0];
    tmem_ld_x8(lane_addr + 64, v);
    tmem_wait_ld();
    out[128 + l] = v[0];
  } else if (mode == 2) {
    if (threadIdx.x == 0) {
      const unsigned long long t0 = clock64();
      for (int s = 0; s < nshift; ++s) tmem_shift_down(tbase + 256 + (uint32_t)(s & 7) * 8);
      const unsigned long long t1 = clock64();
      mma_commit(&bar);
      mbar_wait(&bar, 0);
      const unsigned long long t2 = clock64();
      cyc[0] = t1 - t0;
      cyc[1] = t2 - t0;
    }
  } else {
    // chunk pattern: per chunk R filter rows, each 12 MMAs (4 points x 3 products); between rows the
    // 8 V slices are shifted. lane_off: 0 no shifts, 1 all 8 shifts after the row's 12 MMAs,
    // 2 each point's 2 shifts right after its 3 MMAs, 3 = shifts only (no MMAs)
    if (warp == 0) {
      constexpr uint32_t idesc = idesc_tf32(128, 64);
      const uint64_t bdesc = umma_desc_kmajor_noswizzle(smem_u32(bsm), 64 * 16, 128);
      const int R = col > 0 ? col : 1;
      const unsigned long long t0 = clock64();
      for (int it = 0; it < nshift; ++it) {
        const uint32_t vs = tbase + 256 + (uint32_t)(it & 3) * 64;
        for (int fh = 0; fh < R; ++fh) {
#pragma unroll
          for (int p = 0; p < 2; ++p)
#pragma unroll
            for (int t = 0; t < 4; ++t)
              if (lane_off != 3) mma_tf32_ts_warp(tbase + t * 64, vs + t * 16 + (p == 0 ? 8 : 0), bdesc, idesc, 1u);
#pragma unroll
          for (int t = 0; t < 4; ++t) {
            if (lane_off != 3) mma_tf32_ts_warp(tbase + t * 64, vs + t * 16, bdesc, idesc, 1u);
            if ((lane_off == 2 || lane_off == 3) && fh + 1 < R) {
              asm volatile("{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\t@e tcgen05.shift.cta_group::1.down [%0];\n\t}" ::"r"(vs + t * 16) : "memory");
              asm volatile("{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\t@e tcgen05.shift.cta_group::1.down [%0];\n\t}" ::"r"(vs + t * 16 + 8) : "memory");
            }
          }
          if (lane_off == 1 && fh + 1 < R) {
#pragma unroll
            for (int j = 0; j < 8; ++j) {
              asm volatile("{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\t@e tcgen05.shift.cta_group::1.down [%0];\n\t}" ::"r"(vs + j * 8) : "memory");
            }
          }
        }
      }
      mma_commit_warp(&bar);
      mbar_wait(&bar, 0);
      const unsigned long long t1 = clock64();
      if (l == 0) cyc[0] = t1 - t0;
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) { tc_fence_after(); tmem_dealloc(tbase, 512); }
}

int main() {
  float* d;
  unsigned long long* dc;
  cudaMalloc(&d, 128 * 48 * 4);
  cudaMalloc(&dc, 16 * 8);
  static float h[128 * 48];
  const int offs[][2] = {{0, 8}, {32, 8}, {0, 0}, {64, 16}};
  for (auto& oc : offs) {
    cudaMemset(d, 0, 128 * 48 * 4);
    shift_kernel<<<1, 128>>>(0, oc[0], oc[1], 1, d, dc);
    cudaError_t e = cudaDeviceSynchronize();
    cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    printf("== semantics: shift at lane %d col %d: %s\n", oc[0], oc[1], cudaGetErrorString(e));
    // per column block: which lanes changed and where their value came from
    for (int cb = 0; cb < 48; cb += 8) {
      int changed = 0, first = -1, last = -1, src_delta = 0;
      bool uniform = true;
      for (int l = 0; l < 128; ++l) {
        for (int c = cb; c < cb + 8; ++c) {
          const float v = h[l * 48 + c], orig = l * 1000.f + c;
          if (v != orig) {
            ++changed;
            if (first < 0) first = l;
            last = l;
            const int sl = (int)(v / 1000.f + 0.5f);
            const int sc = (int)(v - sl * 1000.f + 0.5f);
            if (changed == 1) src_delta = sl - l;
            else if (sl - l != src_delta || sc != c) uniform = false;
          }
        }
      }
      printf("  cols %2d..%2d: %4d values changed, lanes %d..%d, src lane delta %d %s\n", cb, cb + 7, changed, first, last, src_delta,
             uniform ? "(uniform)" : "(NOT uniform)");
    }
    printf("  lane 0 col %d: %.0f, lane 1: %.0f, lane 31: %.0f, lane 32: %.0f, lane 127: %.0f\n", oc[1], h[0 * 48 + oc[1]], h[1 * 48 + oc[1]],
           h[31 * 48 + oc[1]], h[32 * 48 + oc[1]], h[127 * 48 + oc[1]]);
  }
  for (int ns = 0; ns <= 2; ++ns) {
    shift_kernel<<<1, 128>>>(1, 0, 0, ns, d, dc);
    cudaError_t e = cudaDeviceSynchronize();
    cudaMemcpy(h, d, 256 * 4, cudaMemcpyDeviceToHost);
    printf("== ordering, %d shift(s) between two MMAs (%s): D[l] for l = 0,1,2,31,32,33,127: ", ns, cudaGetErrorString(e));
    for (int l : {0, 1, 2, 31, 32, 33, 127}) printf("%.0f ", h[l]);
    printf(" | A after: ");
    for (int l : {0, 1, 2, 31, 32, 33, 127}) printf("%.0f ", h[128 + l]);
    printf("\n");
  }
  for (int ns : {1, 8, 64, 512}) {
    shift_kernel<<<1, 128>>>(2, 0, 0, ns, d, dc);
    cudaError_t e = cudaDeviceSynchronize();
    unsigned long long c[2];
    cudaMemcpy(c, dc, 16, cudaMemcpyDeviceToHost);
    printf("== cost: %3d shifts: issue %llu cycles, complete %llu cycles (%.1f cycles/shift) %s\n", ns, c[0], c[1], (double)c[1] / ns,
           cudaGetErrorString(e));
  }
  const char* names[] = {"no shifts", "8 shifts after each row", "2 shifts after each point", "shifts only"};
  for (int R : {1, 3, 5, 7}) {
    for (int mode3 : {0, 1, 2, 3}) {
      shift_kernel<<<1, 128>>>(3, mode3, R, 100, d, dc);
      cudaError_t e = cudaDeviceSynchronize();
      unsigned long long c[1];
      cudaMemcpy(c, dc, 8, cudaMemcpyDeviceToHost);
      printf("== chunk R=%d, %-26s: %.1f cycles per chunk (MMA ideal %d) %s\n", R, names[mode3], (double)c[0] / 100, 384 * R,
             cudaGetErrorString(e));
    }
  }
  return 0;
}
