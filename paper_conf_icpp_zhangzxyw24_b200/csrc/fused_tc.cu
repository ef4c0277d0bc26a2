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
//  * a2: a TMA warp stages, per 8-channel chunk, the (ROWS+R-1) x WBOX input
//    rows of the block as two 16-byte channel planes (OOB zero fill = padding,
//    PAPER.md:337-338); the rows are reused across all fh (vertical overlap)
//    and by neighbouring windows (the (r-1) horizontal overlap, §5.4).
//    The same warp streams each k-step's U image (1D bulk copy) into a ring.
//  * a3: NWG transform warpgroups (thread = tile) read the alpha-window from
//    shared memory, apply BT with zeros/±1 folded at compile time and the ±
//    pair trick, split 3xTF32 hi/lo and write V into TMEM
//    with tcgen05.st (V is the UMMA A operand, "TS" mode: no SMEM read for A).
//  * a4: NISS issuer warps, each owning GP/NISS points' accumulators, issue per
//    k-step 3 tcgen05.mma.kind::tf32 per point (lo*hi, hi*lo, hi*hi). Several
//    issuers are needed: one warp issues at most one UMMA per ~45 cycles while
//    a 128x64x8 tf32 UMMA takes 32 (tools/mma_bench.cu). Each accumulator has
//    exactly one issuer, so results are bitwise deterministic.
//  * k-step stages: NS slots, each = V (TMEM) + U (SMEM); one "full" barrier
//    (128 transform arrivals + U tx bytes) and one "empty" barrier (NISS commits).
//  * a5: the warpgroups tcgen05.ld the accumulators, apply A^T in registers
//    (pair trick), stage 8-channel slices in shared memory and TMA-store them
//    (TMA clips q >= Q, p >= P, k >= K: the in-kernel boundary). Passes > 0 use a
//    TMA reduce-add into y (the accumulators hold GP of alpha points per pass).
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

template <int M, int RW, int NT>
struct TcCfg {
  using T = Wino<M, RW>;
  static constexpr int A = T::alpha;
  static constexpr int GP = gp_for(A, NT);
  static constexpr int NS = ns_for(A, NT);
  static constexpr int NISS = niss_for(GP);
  static constexpr int NWG = kNWG;
  static constexpr int NPASS = A / GP;
  static constexpr int NIS = 2;                       // input stages
  static constexpr int VCOL = GP * NT;                // first V column in TMEM
  static constexpr int TMEM_COLS = 512;
  static constexpr int UBYTES = GP * 2 * NT * 32;     // one k-step of U (GP points, hi+lo)
  static constexpr int NTHREADS = tc_threads(GP);
  static constexpr int PPI = GP / NISS;               // points per issuer
  static_assert(A % GP == 0 && GP % 2 == 0, "passes must hold whole ± pairs");
  static_assert(NS >= 2 && NS % NWG == 0, "stage ring");
  static_assert(GP * NT + NS * GP * 16 <= TMEM_COLS, "TMEM budget");
  static_assert(NT % 16 == 0 && NT >= 16 && NT <= 256, "UMMA N for M=128");
  static_assert((NT / NWG) % 8 == 0, "epilogue column split");
  static_assert(GP % NISS == 0, "issuer split");
};

template <int M, int RW, int NT>
__global__ void __launch_bounds__(TcCfg<M, RW, NT>::NTHREADS, 1)
    fused_tc_kernel(const __grid_constant__ CUtensorMap xmap, const __grid_constant__ CUtensorMap ymap,
                    const __grid_constant__ Plan pl, const float* __restrict__ u) {
  using Cfg = TcCfg<M, RW, NT>;
  using T = typename Cfg::T;
  constexpr int A = Cfg::A, GP = Cfg::GP, NS = Cfg::NS, NISS = Cfg::NISS, NWG = Cfg::NWG;
  constexpr int NPASS = Cfg::NPASS, NIS = Cfg::NIS, VCOL = Cfg::VCOL, PPI = Cfg::PPI;
  constexpr uint32_t UBYTES = Cfg::UBYTES;

  extern __shared__ __align__(1024) uint8_t smem[];
  const uint32_t inplane = (uint32_t)pl.PLANE;  // plane stride (128-aligned)
  uint8_t* u_smem = smem;                                        // [NS][UBYTES]
  uint8_t* in_smem = u_smem + (size_t)NS * UBYTES;               // [NIS][2 planes][PLANE]
  uint8_t* o_smem = in_smem + (size_t)NIS * 2 * inplane;         // [NWG][NOB][OSTRIDE]
  uint64_t* bars = reinterpret_cast<uint64_t*>(o_smem + (size_t)NWG * pl.NOB * pl.OSTRIDE);
  uint64_t* in_full = bars;             // [NIS]
  uint64_t* in_empty = in_full + NIS;   // [NIS]
  uint64_t* st_full = in_empty + NIS;   // [NS]
  uint64_t* st_empty = st_full + NS;    // [NS]
  uint64_t* d_full = st_empty + NS;     // [1]
  uint64_t* d_empty = d_full + 1;       // [1]
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(d_empty + 1);

  const int warp = threadIdx.x / 32, lane32 = threadIdx.x % 32;
  const int b = blockIdx.x;
  const int nb = b % pl.NB;
  int tb = b / pl.NB;
  const int seg = tb % pl.SEGS;
  tb /= pl.SEGS;
  const int rb = tb % pl.PB;
  const int n = tb / pl.PB;
  const int p0 = rb * pl.ROWS;
  constexpr int PROD_WARP = NWG * 4, ISS_WARP0 = NWG * 4 + 1;

  if (threadIdx.x == 0) {
    for (int i = 0; i < NIS; ++i) { mbar_init(&in_full[i], 1); mbar_init(&in_empty[i], NWG * 128); }
    for (int i = 0; i < NS; ++i) { mbar_init(&st_full[i], 128 + 1); mbar_init(&st_empty[i], NISS); }
    mbar_init(d_full, NISS);
    mbar_init(d_empty, NWG * 128);
    fence_mbar_init();
  }
  if (warp == ISS_WARP0) {  // the first issuer warp owns the TMEM allocation
    tmem_alloc(tmem_slot, Cfg::TMEM_COLS);
    tmem_relinquish();
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tbase = *tmem_slot;
  const int NKS = pl.NKS;

  if (warp < NWG * 4) {
    // ===================== transform + epilogue warpgroups =====================
    const int g = warp / 4;
    const int l = threadIdx.x % 128;  // TMEM lane == tile slot
    const int row_l = pl.lane_row[l], tw_l = pl.lane_tw[l];
    const bool has_slot = row_l != 0xFF;
    const int col0 = has_slot ? tw_l * M : 0;
    const uint32_t lane_addr = tbase + ((uint32_t)(l & ~31) << 16);
    const int TSM = pl.TS * M;  // output columns per CTA row segment
    float* ostage = reinterpret_cast<float*>(o_smem + (size_t)g * pl.NOB * pl.OSTRIDE);

    static_for<NPASS>([&](auto PASS_) {
      constexpr int PASS = PASS_;
      for (int cc = 0; cc < pl.NCC; ++cc) {
        const int li = PASS * pl.NCC + cc, ist = li % NIS;
        mbar_wait(&in_full[ist], (li / NIS) & 1);
        const float4* planes = reinterpret_cast<const float4*>(in_smem + (size_t)ist * 2 * inplane);
        for (int fh = 0; fh < pl.R; ++fh) {
          const int kg = PASS * NKS + cc * pl.R + fh;  // global k-step index
          if (kg % NWG != g) continue;
          const int s = kg % NS, use = kg / NS;
          if (l == 0) trace_rec(pl.trace, 3 * g + 0, kg / NWG);
          if (use > 0) mbar_wait(&st_empty[s], (use - 1) & 1);
          if (l == 0) trace_rec(pl.trace, 3 * g + 1, kg / NWG);
          const uint32_t vbase = lane_addr + VCOL + s * GP * 16;
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
                split_tf32(va[e], ha[e], la[e]);
                split_tf32(vb[e], hb[e], lb[e]);
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
          mbar_arrive(&st_full[s]);
          if (l == 0) trace_rec(pl.trace, 3 * g + 2, kg / NWG);
        }
        mbar_arrive(&in_empty[ist]);
      }
      // ---------- epilogue of this pass: y (+)= A^T M via shared memory + TMA ----------
      if (l == 0) trace_rec(pl.trace, 8 + g, 2 * PASS);
      mbar_wait(d_full, PASS & 1);
      tc_fence_after();
      if (l == 0) trace_rec(pl.trace, 8 + g, 2 * PASS + 1);
      constexpr int CPW = NT / NWG;
      const int qbase = seg * TSM;
#pragma unroll 1
      for (int c8 = 0; c8 < CPW / 8; ++c8) {
        const int col = g * CPW + c8 * 8;
        float Mt[GP][8];
#pragma unroll
        for (int tl = 0; tl < GP; ++tl) tmem_ld_x8(lane_addr + tl * NT + col, Mt[tl]);
        tmem_wait_ld();
        if (c8 == CPW / 8 - 1) {  // accumulators fully read: the issuers may start the next pass
          tc_fence_before();
          mbar_arrive(d_empty);
        }
        // staging buffer reuse: the TMA store that last read it must be done reading
        const int ob = pl.NOB == 2 ? (c8 & 1) : 0;
        if (l == 0) {
          if (pl.NOB == 2) bulk_wait_group_read<1>();
          else bulk_wait_group_read<0>();
        }
        named_bar_sync(1 + g, 128);
        float* stg = ostage + (size_t)ob * (pl.OSTRIDE / 4);
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
                const float sv = (i % 2 == 0) ? (Mt[tl0][e] + Mt[tl0 + 1][e]) : (Mt[tl0][e] - Mt[tl0 + 1][e]);
                if constexpr (ca == 1.f) o[e] += sv;
                else if constexpr (ca != 0.f) o[e] = fmaf(ca, sv, o[e]);
              }
            }
          });
          if (has_slot) {
            float4* dst = reinterpret_cast<float4*>(stg + ((size_t)row_l * TSM + tw_l * M + i) * 8);
            dst[0] = make_float4(o[0], o[1], o[2], o[3]);
            dst[1] = make_float4(o[4], o[5], o[6], o[7]);
          }
        });
        fence_proxy_async_smem();
        named_bar_sync(1 + g, 128);
        if (l == 0) {
          const int k0 = nb * NT + col;
          if constexpr (PASS == 0) tma_store_4d(&ymap, stg, k0, qbase, p0, n);
          else tma_reduce_add_4d(&ymap, stg, k0, qbase, p0, n);
          bulk_commit_group();
        }
      }
      // this pass's writes must be complete before the next pass's reduce-add
      if (l == 0) bulk_wait_group_all();
      if (l == 0) trace_rec(pl.trace, 10 + g, PASS);
    });
  } else if (warp == PROD_WARP) {
    // ====================== TMA / bulk-copy producer ======================
    if (lane32 == 0) {
      tma_prefetch_desc(&xmap);
      tma_prefetch_desc(&ymap);
      const int wstart = seg * pl.TS * M - pl.pad_w;
      const int hstart = p0 - pl.pad_h;
      for (int pass = 0; pass < NPASS; ++pass) {
        for (int cc = 0; cc < pl.NCC; ++cc) {
          const int li = pass * pl.NCC + cc, ist = li % NIS;
          if (li >= NIS) mbar_wait(&in_empty[ist], ((li / NIS) - 1) & 1);
          uint8_t* dst = in_smem + (size_t)ist * 2 * inplane;
          mbar_expect_tx(&in_full[ist], 2u * (uint32_t)pl.BOXB);
          tma_load_4d(dst, &xmap, &in_full[ist], cc * 8, wstart, hstart, n);
          tma_load_4d(dst + inplane, &xmap, &in_full[ist], cc * 8 + 4, wstart, hstart, n);
          for (int fh = 0; fh < pl.R; ++fh) {
            const int ks = cc * pl.R + fh, kg = pass * NKS + ks;
            const int s = kg % NS, use = kg / NS;
            if (use > 0) mbar_wait(&st_empty[s], (use - 1) & 1);
            mbar_expect_tx(&st_full[s], UBYTES);
            bulk_load(u_smem + (size_t)s * UBYTES, u + u_offset(NT, A, nb, NKS, ks, pass * GP, 0), UBYTES,
                      &st_full[s]);
          }
        }
      }
    }
    __syncwarp();
  } else {
    // ============================= MMA issuers =============================
    const int iss = warp - ISS_WARP0;  // owns points tl = iss * PPI .. iss * PPI + PPI - 1
    if (lane32 == 0) {
      constexpr uint32_t idesc = idesc_tf32(128, NT);
      const uint32_t u_base = smem_u32(u_smem);
      for (int pass = 0; pass < NPASS; ++pass) {
        if (pass > 0) {
          mbar_wait(d_empty, (pass - 1) & 1);
          tc_fence_after();
        }
        for (int ks = 0; ks < NKS; ++ks) {
          const int kg = pass * NKS + ks;
          const int s = kg % NS, use = kg / NS;
          if (iss == 0) trace_rec(pl.trace, 12, kg);
          mbar_wait(&st_full[s], use & 1);
          tc_fence_after();
          if (iss == 0) trace_rec(pl.trace, 6, kg);
          const uint32_t ub = u_base + s * UBYTES;
          const uint32_t va = tbase + VCOL + s * GP * 16;
          // product order lo*hi, hi*lo, hi*hi (small terms first), points innermost
#pragma unroll
          for (int prod = 0; prod < 3; ++prod) {
#pragma unroll
            for (int pi = 0; pi < PPI; ++pi) {
              const int tl = iss * PPI + pi;
              const uint32_t a = va + tl * 16 + (prod == 0 ? 8 : 0);
              const uint64_t bd = umma_desc_kmajor_noswizzle(ub + (tl * 2 + (prod == 1 ? 1 : 0)) * NT * 32, NT * 16, 128);
              mma_tf32_ts(tbase + tl * NT, a, bd, idesc, (ks > 0 || prod > 0) ? 1u : 0u);
            }
          }
          if (iss == 0) trace_rec(pl.trace, 7, kg);
          mma_commit(&st_empty[s]);
          if (iss == 0) trace_rec(pl.trace, 14, kg);
        }
        mma_commit(d_full);
      }
    }
    __syncwarp();
  }

  tc_fence_before();
  __syncthreads();
  if (warp == ISS_WARP0) {
    tc_fence_after();
    tmem_dealloc(tbase, Cfg::TMEM_COLS);
  }
}

template <int M, int RW, int NT>
static cudaError_t launch_tc_t(const CUtensorMap& xmap, const CUtensorMap& ymap, const Plan& pl, const float* u,
                               cudaStream_t stream) {
  using Cfg = TcCfg<M, RW, NT>;
  auto kern = fused_tc_kernel<M, RW, NT>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, pl.smem_bytes);
  if (e != cudaSuccess) return e;
  kern<<<pl.tile_blocks * pl.NB, Cfg::NTHREADS, pl.smem_bytes, stream>>>(xmap, ymap, pl, u);
  return cudaGetLastError();
}

// (m, r, NT) -> kernel instantiation (GP, NS, NISS derived; see common.cuh).
cudaError_t launch_fused_tc(const CUtensorMap& xmap, const CUtensorMap& ymap, const Plan& pl, const float* u,
                            cudaStream_t stream) {
  const int key = pl.S * 1000 + pl.m * 10 + (pl.NT == 64 ? 1 : 0);
  switch (key) {
#define I2CW_TC(MM, RR)                                                                          \
  case RR * 1000 + MM * 10 + 1: return launch_tc_t<MM, RR, 64>(xmap, ymap, pl, u, stream); \
  case RR * 1000 + MM * 10 + 0: return launch_tc_t<MM, RR, 32>(xmap, ymap, pl, u, stream);
    I2CW_TC(7, 2) I2CW_TC(6, 3) I2CW_TC(5, 4) I2CW_TC(4, 5) I2CW_TC(3, 6) I2CW_TC(2, 7)  // alpha 8
    I2CW_TC(5, 8) I2CW_TC(4, 9)                                                          // alpha 12
    I2CW_TC(10, 7) I2CW_TC(9, 8) I2CW_TC(8, 9)                                           // alpha 16 (ablation)
#undef I2CW_TC
    default: return cudaErrorInvalidValue;
  }
}

}  // namespace i2cw
