// The fused Im2col-Winograd forward kernel for sm_100a (rows a2-a5 of
// SURVEY.md §8(a)); deconvolution runs through the same kernel with a
// rotated, channel-transposed U (filter_transform.cu).
//
// Method (§4.1, Fig 2): Stage 1 im2col is an index map;
// Stage 2 slides 1D windows of alpha = m + S - 1 input columns along W, runs
// F(m, S) on them and accumulates over filter rows fh and channels c:
//   V_t[tile][(fh,c)] = sum_j BT[t][j] x[n][p-ph+fh][q0-pw+j][c]          (a3)
//   M_t[tile][k]      = sum_{fh,c} V_t[tile][(fh,c)] U_t[k][(fh,c)]        (a4)
//   y[n][p][q0+i][k]  = sum_t AT[i][t] M_t[tile][k]   (q0+i < Q only)      (a5)
// A^T is applied once after the (fh, c) sum by linearity.
//
// B200 mapping:
//  * CTA = 128 Winograd tiles (UMMA M, one TMEM lane each) x NT output channels.
//    Tiles are ROWS output rows x TS tiles of one image; lane->tile is a host
//    permutation that spreads the 16-byte shared-memory reads over banks.
//  * a2: one TMA warp stages, per 8-channel chunk, the (ROWS+R-1) x WBOX input
//    rows of the block as two 16-byte channel planes (OOB zero fill = padding,
//    PAPER.md:337-338); the rows are reused across all fh (vertical overlap)
//    and by neighbouring windows (the (r-1) horizontal overlap, §5.4).
//    U k-step images arrive by 1D bulk copy into a ring.
//  * a3: NWG transform warpgroups (thread = tile) read the alpha-window from
//    shared memory, apply BT with zeros/±1 folded at compile time and the ±
//    pair trick, split 3xTF32 hi/lo and write V into TMEM
//    with tcgen05.st (V is the UMMA A operand, "TS" mode).
//  * a4: one thread issues, per k-step and point, 3 tcgen05.mma.kind::tf32
//    (lo*hi, hi*lo, hi*hi) into the point's fp32 accumulator in TMEM.
//  * a5: after the last k-step the same warpgroups tcgen05.ld the accumulators,
//    apply A^T in registers (pair trick) and store y with masked 16-byte stores.
//  * TMEM budget: GP points x NT columns of accumulators + NWG V stages of
//    GP x 16 columns <= 512; alpha/GP passes, pass > 0 adds into y (RMW).
#include <utility>

#include "common.cuh"
#include "transforms_generated.h"

namespace i2cw {

template <class F, int... I>
__device__ __forceinline__ void static_for_impl(F&& f, std::integer_sequence<int, I...>) {
  (f(std::integral_constant<int, I>{}), ...);
}
template <int N, class F>
__device__ __forceinline__ void static_for(F&& f) {
  static_for_impl(f, std::make_integer_sequence<int, N>{});
}

// sum_j c_j * d[j][e] with compile-time coefficients; zeros skipped, ±1 as add/sub.
// Only j with (j % JSTEP == JOFF) are included (the pair trick's even/odd halves).
template <class T, int PT, int JSTEP, int JOFF, int A>
__device__ __forceinline__ float bt_dot(const float (&d)[A][4], int e) {
  float acc = 0.f;
  static_for<A>([&](auto J) {
    constexpr int j = J;
    if constexpr (j % JSTEP == JOFF) {
      constexpr float c = T::BT(PT, j);
      if constexpr (c == 1.f) acc += d[j][e];
      else if constexpr (c == -1.f) acc -= d[j][e];
      else if constexpr (c != 0.f) acc = fmaf(c, d[j][e], acc);
    }
  });
  return acc;
}

template <int M, int RW, int NT, int GP, int NWG>
struct TcCfg {
  using T = Wino<M, RW>;
  static constexpr int A = T::alpha;
  static constexpr int NPASS = A / GP;
  static constexpr int NIS = 2;                       // input stages
  static constexpr int VCOL = GP * NT;                // first V column in TMEM
  static constexpr int TMEM_COLS = 512;
  static constexpr int UBYTES = GP * 2 * NT * 32;     // one k-step of U (GP points, hi+lo)
  static constexpr int NTHREADS = NWG * 128 + 64;     // + TMA warp + MMA warp
  static_assert(A % GP == 0 && GP % 2 == 0, "passes must hold whole ± pairs");
  static_assert(GP * NT + NWG * GP * 16 <= TMEM_COLS, "TMEM budget");
  static_assert(NT % 16 == 0 && NT >= 16 && NT <= 256, "UMMA N for M=128");
  static_assert((NT / NWG) % 8 == 0, "epilogue column split");
};

template <int M, int RW, int NT, int GP, int NWG>
__global__ void __launch_bounds__(TcCfg<M, RW, NT, GP, NWG>::NTHREADS, 1)
    fused_tc_kernel(const __grid_constant__ CUtensorMap xmap, const __grid_constant__ Plan pl,
                    const float* __restrict__ u, float* __restrict__ y) {
  using Cfg = TcCfg<M, RW, NT, GP, NWG>;
  using T = typename Cfg::T;
  constexpr int A = Cfg::A, NPASS = Cfg::NPASS, NIS = Cfg::NIS, VCOL = Cfg::VCOL;
  constexpr uint32_t UBYTES = Cfg::UBYTES;

  extern __shared__ __align__(1024) uint8_t smem[];
  const int NUS = pl.NUS;
  const uint32_t inplane = (uint32_t)pl.PLANE;  // plane stride (128-aligned)
  uint8_t* u_smem = smem;
  uint8_t* in_smem = smem + (size_t)NUS * UBYTES;
  uint64_t* bars = reinterpret_cast<uint64_t*>(in_smem + (size_t)NIS * 2 * inplane);
  uint64_t* in_full = bars;             // [NIS]
  uint64_t* in_empty = in_full + NIS;   // [NIS]
  uint64_t* v_full = in_empty + NIS;    // [NWG]
  uint64_t* v_empty = v_full + NWG;     // [NWG]
  uint64_t* d_full = v_empty + NWG;     // [1]
  uint64_t* d_empty = d_full + 1;       // [1]
  uint64_t* u_full = d_empty + 1;       // [NUS]
  uint64_t* u_empty = u_full + NUS;     // [NUS]
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(u_empty + NUS);

  const int warp = threadIdx.x / 32, lane32 = threadIdx.x % 32;
  const int b = blockIdx.x;
  const int nb = b % pl.NB;
  int tb = b / pl.NB;
  const int seg = tb % pl.SEGS;
  tb /= pl.SEGS;
  const int rb = tb % pl.PB;
  const int n = tb / pl.PB;
  const int p0 = rb * pl.ROWS;

  if (threadIdx.x == 0) {
    for (int i = 0; i < NIS; ++i) { mbar_init(&in_full[i], 1); mbar_init(&in_empty[i], NWG * 128); }
    for (int i = 0; i < NWG; ++i) { mbar_init(&v_full[i], 128); mbar_init(&v_empty[i], 1); }
    mbar_init(d_full, 1);
    mbar_init(d_empty, NWG * 128);
    for (int i = 0; i < NUS; ++i) { mbar_init(&u_full[i], 1); mbar_init(&u_empty[i], 1); }
    fence_mbar_init();
  }
  if (warp == NWG * 4 + 1) {  // MMA warp owns the TMEM allocation
    tmem_alloc(tmem_slot, Cfg::TMEM_COLS);
    tmem_relinquish();
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tbase = *tmem_slot;

  if (warp < NWG * 4) {
    // ===================== transform + epilogue warpgroups =====================
    const int g = warp / 4;
    const int l = threadIdx.x % 128;  // TMEM lane == tile slot
    const int row_l = pl.lane_row[l], tw_l = pl.lane_tw[l];
    const bool has_slot = row_l != 0xFF;
    const int p = p0 + (has_slot ? row_l : 0);
    const int tw = seg * pl.TS + (has_slot ? tw_l : 0);
    const bool valid = has_slot && p < pl.P && tw < pl.T_r;
    const int q0 = tw * M;
    const int col0 = has_slot ? tw_l * M : 0;
    const uint32_t lane_addr = tbase + ((uint32_t)(l & ~31) << 16);
    const uint32_t vbase = lane_addr + VCOL + g * GP * 16;
    int vuse = 0;

    static_for<NPASS>([&](auto PASS_) {
      constexpr int PASS = PASS_;
      for (int cc = 0; cc < pl.NCC; ++cc) {
        const int li = PASS * pl.NCC + cc, st = li % NIS;
        mbar_wait(&in_full[st], (li / NIS) & 1);
        const float4* planes = reinterpret_cast<const float4*>(in_smem + (size_t)st * 2 * inplane);
        for (int fh = 0; fh < pl.R; ++fh) {
          const int ks = cc * pl.R + fh;
          if (ks % NWG != g) continue;
          if (l == 0) trace_rec(pl.trace, 3 * g + 0, vuse);
          if (vuse > 0) mbar_wait(&v_empty[g], (vuse - 1) & 1);
          if (l == 0) trace_rec(pl.trace, 3 * g + 1, vuse);
          const int off = (has_slot ? (row_l + fh) : 0) * pl.WBOX + col0;
#pragma unroll
          for (int h = 0; h < 2; ++h) {
            const float4* src = planes + (size_t)h * (inplane / 16) + off;
            float d[A][4];
#pragma unroll
            for (int j = 0; j < A; ++j) {
              float4 v = has_slot ? src[j] : make_float4(0.f, 0.f, 0.f, 0.f);
              d[j][0] = v.x; d[j][1] = v.y; d[j][2] = v.z; d[j][3] = v.w;
            }
            static_for<GP / 2>([&](auto Q_) {
              constexpr int idx0 = PASS * GP + 2 * (int)Q_;  // internal index of this pair slot
              constexpr int tl0 = 2 * (int)Q_;
              float va[4], vb[4];
              if constexpr (idx0 == 0) {  // singles: point 0 and point alpha-1
#pragma unroll
                for (int e = 0; e < 4; ++e) {
                  va[e] = bt_dot<T, 0, 1, 0>(d, e);
                  vb[e] = bt_dot<T, A - 1, 1, 0>(d, e);
                }
              } else {  // ± pair (a, a+1): E over even j, O over odd j
                constexpr int pa = point_of(idx0, A);
#pragma unroll
                for (int e = 0; e < 4; ++e) {
                  const float E = bt_dot<T, pa, 2, 0>(d, e);
                  const float O = bt_dot<T, pa, 2, 1>(d, e);
                  va[e] = E + O;
                  vb[e] = E - O;
                }
              }
              float ha[4], la[4], hb[4], lb[4];
#pragma unroll
              for (int e = 0; e < 4; ++e) {
                ha[e] = tf32_rna(va[e]); la[e] = tf32_rna(va[e] - ha[e]);
                hb[e] = tf32_rna(vb[e]); lb[e] = tf32_rna(vb[e] - hb[e]);
              }
              const uint32_t ca = vbase + tl0 * 16 + h * 4, cb = ca + 16;
              tmem_st_x4(ca, ha[0], ha[1], ha[2], ha[3]);
              tmem_st_x4(ca + 8, la[0], la[1], la[2], la[3]);
              tmem_st_x4(cb, hb[0], hb[1], hb[2], hb[3]);
              tmem_st_x4(cb + 8, lb[0], lb[1], lb[2], lb[3]);
            });
          }
          tmem_wait_st();
          tc_fence_before();
          mbar_arrive(&v_full[g]);
          if (l == 0) trace_rec(pl.trace, 3 * g + 2, vuse);
          ++vuse;
        }
        mbar_arrive(&in_empty[st]);
      }
      // ---------------- epilogue of this pass: y (+)= A^T M ----------------
      if (l == 0) trace_rec(pl.trace, 8 + g, 2 * PASS);
      mbar_wait(d_full, PASS & 1);
      if (l == 0) trace_rec(pl.trace, 8 + g, 2 * PASS + 1);
      tc_fence_after();
      constexpr int CPW = NT / NWG;
#pragma unroll 1
      for (int c8 = 0; c8 < CPW / 8; ++c8) {
        const int col = g * CPW + c8 * 8;
        float Mt[GP][8];
#pragma unroll
        for (int tl = 0; tl < GP; ++tl) tmem_ld_x8(lane_addr + tl * NT + col, Mt[tl]);
        tmem_wait_ld();
        // pair sums / differences (internal slots 2q, 2q+1 hold points a, a+1)
        const int k0 = nb * NT + col;
        static_for<M>([&](auto I_) {
          constexpr int i = I_;
          float o[8];
#pragma unroll
          for (int e = 0; e < 8; ++e) o[e] = 0.f;
          static_for<GP / 2>([&](auto Q_) {
            constexpr int idx0 = PASS * GP + 2 * (int)Q_;
            constexpr int tl0 = 2 * (int)Q_;
            if constexpr (idx0 == 0) {
              constexpr float c0 = T::AT(i, 0), c1 = T::AT(i, A - 1);
#pragma unroll
              for (int e = 0; e < 8; ++e) {
                if constexpr (c0 != 0.f) o[e] = fmaf(c0, Mt[tl0][e], o[e]);
                if constexpr (c1 != 0.f) o[e] = fmaf(c1, Mt[tl0 + 1][e], o[e]);
              }
            } else {
              constexpr int pa = point_of(idx0, A);
              constexpr float ca = T::AT(i, pa);
#pragma unroll
              for (int e = 0; e < 8; ++e) {
                const float s = (i % 2 == 0) ? (Mt[tl0][e] + Mt[tl0 + 1][e]) : (Mt[tl0][e] - Mt[tl0 + 1][e]);
                if constexpr (ca == 1.f) o[e] += s;
                else if constexpr (ca != 0.f) o[e] = fmaf(ca, s, o[e]);
              }
            }
          });
          if (valid && q0 + i < pl.Q) {
            float* yp = y + (((size_t)n * pl.P + p) * pl.Q + q0 + i) * pl.K + k0;
#pragma unroll
            for (int hh = 0; hh < 2; ++hh) {
              if (k0 + hh * 4 + 4 <= pl.K) {
                float4 v = make_float4(o[hh * 4 + 0], o[hh * 4 + 1], o[hh * 4 + 2], o[hh * 4 + 3]);
                float4* dst = reinterpret_cast<float4*>(yp + hh * 4);
                if constexpr (PASS > 0) {
                  const float4 prev = *dst;
                  v.x += prev.x; v.y += prev.y; v.z += prev.z; v.w += prev.w;
                }
                *dst = v;
              }
            }
          }
        });
      }
      tc_fence_before();
      mbar_arrive(d_empty);
      if (l == 0) trace_rec(pl.trace, 10 + g, PASS);
    });
  } else if (warp == NWG * 4) {
    // ============================ TMA producer ============================
    if (lane32 == 0) {
      tma_prefetch_desc(&xmap);
      const int wstart = seg * pl.TS * M - pl.pad_w;
      const int hstart = p0 - pl.pad_h;
      int ui = 0;
      for (int pass = 0; pass < NPASS; ++pass) {
        for (int cc = 0; cc < pl.NCC; ++cc) {
          const int li = pass * pl.NCC + cc, st = li % NIS;
          if (li >= NIS) mbar_wait(&in_empty[st], ((li / NIS) - 1) & 1);
          uint8_t* dst = in_smem + (size_t)st * 2 * inplane;
          mbar_expect_tx(&in_full[st], 2u * (uint32_t)pl.BOXB);
          tma_load_4d(dst, &xmap, &in_full[st], cc * 8, wstart, hstart, n);
          tma_load_4d(dst + inplane, &xmap, &in_full[st], cc * 8 + 4, wstart, hstart, n);
          for (int fh = 0; fh < pl.R; ++fh, ++ui) {
            const int ks = cc * pl.R + fh, us = ui % NUS;
            if (ui >= NUS) mbar_wait(&u_empty[us], ((ui / NUS) - 1) & 1);
            mbar_expect_tx(&u_full[us], UBYTES);
            bulk_load(u_smem + (size_t)us * UBYTES, u + u_offset(NT, A, nb, pl.NKS, ks, pass * GP, 0), UBYTES,
                      &u_full[us]);
          }
        }
      }
    }
    __syncwarp();
  } else {
    // ============================= MMA issuer =============================
    if (lane32 == 0) {
      constexpr uint32_t idesc = idesc_tf32(128, NT);
      const uint32_t u_base = smem_u32(u_smem);
      int ui = 0;
      int vuse[NWG];
#pragma unroll
      for (int i = 0; i < NWG; ++i) vuse[i] = 0;
      for (int pass = 0; pass < NPASS; ++pass) {
        if (pass > 0) {
          mbar_wait(d_empty, (pass - 1) & 1);
          tc_fence_after();
        }
        for (int ks = 0; ks < pl.NKS; ++ks, ++ui) {
          const int g = ks % NWG;
          trace_rec(pl.trace, 12, ui);
          mbar_wait(&v_full[g], vuse[g] & 1);
          trace_rec(pl.trace, 13, ui);
          ++vuse[g];
          const int us = ui % NUS;
          mbar_wait(&u_full[us], (ui / NUS) & 1);
          tc_fence_after();
          trace_rec(pl.trace, 6, ui);
          const uint32_t ub = u_base + us * UBYTES;
#pragma unroll
          for (int tl = 0; tl < GP; ++tl) {
            const uint32_t a_hi = tbase + VCOL + g * GP * 16 + tl * 16, a_lo = a_hi + 8;
            const uint64_t b_hi = umma_desc_kmajor_noswizzle(ub + (tl * 2 + 0) * NT * 32, NT * 16, 128);
            const uint64_t b_lo = umma_desc_kmajor_noswizzle(ub + (tl * 2 + 1) * NT * 32, NT * 16, 128);
            const uint32_t dcol = tbase + tl * NT;
            mma_tf32_ts(dcol, a_lo, b_hi, idesc, ks > 0 ? 1u : 0u);
            mma_tf32_ts(dcol, a_hi, b_lo, idesc, 1u);
            mma_tf32_ts(dcol, a_hi, b_hi, idesc, 1u);
          }
          trace_rec(pl.trace, 7, ui);
          mma_commit(&v_empty[g]);
          mma_commit(&u_empty[us]);
          trace_rec(pl.trace, 14, ui);
        }
        mma_commit(d_full);
      }
    }
    __syncwarp();
  }

  tc_fence_before();
  __syncthreads();
  if (warp == NWG * 4 + 1) {
    tc_fence_after();
    tmem_dealloc(tbase, Cfg::TMEM_COLS);
  }
}

template <int M, int RW, int NT, int GP>
static cudaError_t launch_tc_t(const CUtensorMap& xmap, const Plan& pl, const float* u, float* y,
                               cudaStream_t stream) {
  constexpr int NWG = 2;
  using Cfg = TcCfg<M, RW, NT, GP, NWG>;
  auto kern = fused_tc_kernel<M, RW, NT, GP, NWG>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, pl.smem_bytes);
  if (e != cudaSuccess) return e;
  kern<<<pl.tile_blocks * pl.NB, Cfg::NTHREADS, pl.smem_bytes, stream>>>(xmap, pl, u, y);
  return cudaGetLastError();
}

// (m, r) -> kernel instantiation for the two N tiles; GP from the TMEM budget
// (NT=64: GP=4; NT=32: GP=8), see make_plan() in api.cu.
cudaError_t launch_fused_tc(const CUtensorMap& xmap, const Plan& pl, const float* u, float* y, cudaStream_t stream) {
  const int key = pl.S * 1000 + pl.m * 10 + (pl.NT == 64 ? 1 : 0);
  switch (key) {
#define I2CW_TC(MM, RR)                                                                               \
  case RR * 1000 + MM * 10 + 1: return launch_tc_t<MM, RR, 64, gp_for(MM + RR - 1, 64)>(xmap, pl, u, y, stream); \
  case RR * 1000 + MM * 10 + 0: return launch_tc_t<MM, RR, 32, gp_for(MM + RR - 1, 32)>(xmap, pl, u, y, stream);
    I2CW_TC(7, 2) I2CW_TC(6, 3) I2CW_TC(5, 4) I2CW_TC(4, 5) I2CW_TC(3, 6) I2CW_TC(2, 7)  // alpha 8
    I2CW_TC(5, 8) I2CW_TC(4, 9)                                                          // alpha 12
    I2CW_TC(10, 7) I2CW_TC(9, 8) I2CW_TC(8, 9)                                           // alpha 16 (ablation)
#undef I2CW_TC
    default: return cudaErrorInvalidValue;
  }
}

}  // namespace i2cw
