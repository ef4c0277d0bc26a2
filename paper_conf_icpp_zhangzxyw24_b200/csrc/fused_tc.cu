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
  static constexpr int NWG = nwg_for(NT);
  static constexpr int NPASS = A / GP;
  static constexpr int VCOL = GP * NT;                // first V column in TMEM
  static constexpr int TMEM_COLS = 512;
  static constexpr int UBYTES = GP * 2 * NT * 32;     // one k-step of U (GP points, hi+lo)
  static constexpr int NTHREADS = tc_threads(GP, NT);
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
  constexpr int NPASS = Cfg::NPASS, VCOL = Cfg::VCOL, PPI = Cfg::PPI;
  const int NIS = pl.NIS;  // input stages (runtime: fills the shared-memory budget)
  constexpr uint32_t UBYTES = Cfg::UBYTES;

  extern __shared__ __align__(1024) uint8_t smem[];
  const uint32_t inplane = (uint32_t)pl.PLANE;  // plane stride (128-aligned)
  const int NUS = pl.NUS;  // U ring slots (runtime: deeper than the TMEM V stages to hide L2 latency)
  uint8_t* u_smem = smem;                                        // [NUS][UBYTES]         (1024-aligned)
  uint8_t* o_smem = u_smem + (size_t)NUS * UBYTES;               // [NWG][NOB][OSTRIDE]   (1024-aligned)
  uint8_t* in_smem = o_smem + (size_t)NWG * pl.NOB * pl.OSTRIDE;  // [NIS][2 planes][PLANE]
  uint64_t* bars = reinterpret_cast<uint64_t*>(in_smem + (size_t)NIS * 2 * inplane);
  uint64_t* in_full = bars;             // [NIS]
  uint64_t* in_empty = in_full + NIS;   // [NIS]
  uint64_t* st_full = in_empty + NIS;   // [NS]
  uint64_t* st_empty = st_full + NS;    // [NS]
  uint64_t* d_full = st_empty + NS;     // [1]
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
  constexpr int PROD_WARP = NWG * 4, UPROD_WARP = NWG * 4 + 1, ISS_WARP0 = NWG * 4 + 2;

  if (threadIdx.x == 0) {
    for (int i = 0; i < NIS; ++i) { mbar_init(&in_full[i], 1); mbar_init(&in_empty[i], NWG * 128); }
    for (int i = 0; i < NS; ++i) { mbar_init(&st_full[i], 128); mbar_init(&st_empty[i], NISS); }
    for (int i = 0; i < NUS; ++i) { mbar_init(&u_full[i], 1); mbar_init(&u_empty[i], NISS); }
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
    // staged row of this tile in the output box (box order: channels, tiles, rows) and its
    // TMA swizzle: 128B rows (CPW = 32) XOR chunk with r & 7; 64B rows (CPW = 16) with (r>>1) & 3
    constexpr int CPW = NT / NWG;
    const int orow = has_slot ? row_l * pl.TS + tw_l : 0;
    const int oswz = CPW == 32 ? (orow & 7) : ((orow >> 1) & 3);

    int ist = 0, iph = 0;  // input ring slot / phase (incremental: no runtime division)
    static_for<NPASS>([&](auto PASS_) {
      constexpr int PASS = PASS_;
      for (int cc = 0; cc < pl.NCC; ++cc) {
        const int li = PASS * pl.NCC + cc;
        if (l == 0) trace_rec(pl.trace, 19 + g, li);
        mbar_wait(&in_full[ist], iph);
        if (l == 0) trace_rec(pl.trace, 23 + g, li);
        const float4* planes = reinterpret_cast<const float4*>(in_smem + (size_t)ist * 2 * inplane);
        for (int fh = 0; fh < pl.R; ++fh) {
          const int kg = PASS * NKS + cc * pl.R + fh;  // global k-step index
          if (kg % NWG != g) continue;
          const int s = kg % NS, use = kg / NS;
          if (l == 0) trace_rec(pl.trace, 0 + g, kg / NWG);
          if (use > 0) mbar_wait(&st_empty[s], (use - 1) & 1);
          if (l == 0) trace_rec(pl.trace, 4 + g, kg / NWG);
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
          if (l == 0) trace_rec(pl.trace, 8 + g, kg / NWG);
          if (g == 0 && (l & 31) == 0) trace_rec(pl.trace, 12 + (l >> 5), kg / NWG);
        }
        mbar_arrive(&in_empty[ist]);
        if (++ist == NIS) { ist = 0; iph ^= 1; }
      }
      // ---------- epilogue of this pass: y (+)= A^T M via shared memory + TMA ----------
      if (l == 0 && g == 0) trace_rec(pl.trace, 27, 2 * PASS);
      mbar_wait(d_full, PASS & 1);
      tc_fence_after();
      if (l == 0 && g == 0) trace_rec(pl.trace, 27, 2 * PASS + 1);
      // One output column i at a time over this warpgroup's CPW channels: every tile's
      // y[q0 + i][cbase .. cbase+CPW) is one 128-byte (64-byte) row of the staging box,
      // and the TMA store walks Q with element stride m (positions q0 + i of all tiles).
      const int qbase = seg * TSM;
      const int cbase = g * CPW;
      static_for<M>([&](auto I_) {
        constexpr int i = I_;
        // staging buffer reuse: the TMA store that last read it must be done reading
        const int ob = i % pl.NOB;
        if (l == 0) {
          if (pl.NOB == 2) bulk_wait_group_read<1>();
          else bulk_wait_group_read<0>();
        }
        named_bar_sync(1 + g, 128);
        float4* stg = reinterpret_cast<float4*>(ostage + (size_t)ob * (pl.OSTRIDE / 4)) + (size_t)orow * (CPW / 4);
#pragma unroll 1
        for (int hh = 0; hh < CPW / 16; ++hh) {  // 16 channels at a time (register budget)
          float o[16];
#pragma unroll
          for (int e = 0; e < 16; ++e) o[e] = 0.f;
          static_for<GP / 2>([&](auto Q_) {
            constexpr int idx0 = PASS * GP + 2 * (int)Q_;  // pair slot (internal points idx0, idx0+1)
            constexpr int tl0 = 2 * (int)Q_;
            float ma[16], mb[16];
            tmem_ld_x16(lane_addr + tl0 * NT + cbase + 16 * hh, ma);
            tmem_ld_x16(lane_addr + (tl0 + 1) * NT + cbase + 16 * hh, mb);
            tmem_wait_ld();
            if constexpr (idx0 == 0) {
              constexpr float c0 = T::AT(i, 0), c1 = T::AT(i, A - 1);
#pragma unroll
              for (int e = 0; e < 16; ++e) {
                if constexpr (c0 != 0.f) o[e] = fmaf(c0, ma[e], o[e]);
                if constexpr (c1 != 0.f) o[e] = fmaf(c1, mb[e], o[e]);
              }
            } else {  // AT[i][a+1] = (-1)^i AT[i][a] (pair structure)
              constexpr int pa = point_of(idx0, A);
              constexpr float ca = T::AT(i, pa);
#pragma unroll
              for (int e = 0; e < 16; ++e) {
                const float sv = (i % 2 == 0) ? (ma[e] + mb[e]) : (ma[e] - mb[e]);
                if constexpr (ca == 1.f) o[e] += sv;
                else if constexpr (ca != 0.f) o[e] = fmaf(ca, sv, o[e]);
              }
            }
          });
          if (has_slot) {
#pragma unroll
            for (int j = 0; j < 4; ++j)
              stg[(4 * hh + j) ^ oswz] = make_float4(o[4 * j], o[4 * j + 1], o[4 * j + 2], o[4 * j + 3]);
          }
        }
        if constexpr (i == M - 1) {  // accumulators fully read: the issuers may start the next pass
          tc_fence_before();
          mbar_arrive(d_empty);
        }
        fence_proxy_async_smem();
        named_bar_sync(1 + g, 128);
        if (l == 0) {
          const float* box = ostage + (size_t)ob * (pl.OSTRIDE / 4);
          const int k0 = nb * NT + cbase;
          if constexpr (PASS == 0) tma_store_4d(&ymap, box, k0, qbase + i, p0, n);
          else tma_reduce_add_4d(&ymap, box, k0, qbase + i, p0, n);
          bulk_commit_group();
        }
      });
      // this pass's writes must be complete before the next pass's reduce-add
      if (l == 0) bulk_wait_group_all();
      if (l == 0 && g == 0) trace_rec(pl.trace, 28, PASS);
    });
  } else if (warp == PROD_WARP) {
    // ====================== input-row TMA producer ======================
    if (lane32 == 0) {
      tma_prefetch_desc(&xmap);
      tma_prefetch_desc(&ymap);
      const int wstart = seg * pl.TS * M - pl.pad_w;
      const int hstart = p0 - pl.pad_h;
      int ist = 0, iph = 0, first = 1;  // slot, round parity, still in the first round
      for (int pass = 0; pass < NPASS; ++pass) {
        for (int cc = 0; cc < pl.NCC; ++cc) {
          if (!first) mbar_wait(&in_empty[ist], iph ^ 1);
          uint8_t* dst = in_smem + (size_t)ist * 2 * inplane;
          mbar_expect_tx(&in_full[ist], 2u * (uint32_t)pl.BOXB);
          tma_load_4d(dst, &xmap, &in_full[ist], cc * 8, wstart, hstart, n);
          tma_load_4d(dst + inplane, &xmap, &in_full[ist], cc * 8 + 4, wstart, hstart, n);
          if (++ist == NIS) { ist = 0; iph ^= 1; first = 0; }
        }
      }
    }
    __syncwarp();
  } else if (warp == UPROD_WARP) {
    // ======================= U (transformed filter) ring =======================
    if (lane32 == 0) {
      int us = 0, uph = 0, first = 1;
      for (int pass = 0; pass < NPASS; ++pass) {
        const float* src = u + u_offset(NT, A, nb, NKS, 0, pass * GP, 0);
        for (int ks = 0; ks < NKS; ++ks, src += (size_t)A * 2 * NT * 8) {
          if (!first) mbar_wait(&u_empty[us], uph ^ 1);
          mbar_expect_tx(&u_full[us], UBYTES);
          bulk_load(u_smem + (size_t)us * UBYTES, src, UBYTES, &u_full[us]);
          if (++us == NUS) { us = 0; uph ^= 1; first = 0; }
        }
      }
    }
    __syncwarp();
  } else {
    // ============================= MMA issuers =============================
    const int iss = warp - ISS_WARP0;  // owns points tl = iss * PPI .. iss * PPI + PPI - 1
    if (lane32 == 0) {
      constexpr uint32_t idesc = idesc_tf32(128, NT);
      // descriptor of U slot 0, point 0, hi; other images = + (byte offset >> 4) in the start field
      const uint64_t bdesc0 = umma_desc_kmajor_noswizzle(smem_u32(u_smem), NT * 16, 128);
      int s = 0, sph = 0, us = 0, uph = 0;  // V stage / U slot and their round parities
      int kg = 0;
      for (int pass = 0; pass < NPASS; ++pass) {
        if (pass > 0) {
          mbar_wait(d_empty, (pass - 1) & 1);
          tc_fence_after();
        }
        for (int ks = 0; ks < NKS; ++ks, ++kg) {
          if (iss == 0) trace_rec(pl.trace, 29, kg);
          mbar_wait(&st_full[s], sph);
          mbar_wait(&u_full[us], uph);
          tc_fence_after();
          if (iss == 0) trace_rec(pl.trace, 16, kg);
          const uint64_t bslot = bdesc0 + (uint64_t)((us * UBYTES) >> 4);
          const uint32_t va = tbase + VCOL + s * GP * 16;
          // product order lo*hi, hi*lo, hi*hi (small terms first), points innermost
#pragma unroll
          for (int prod = 0; prod < 3; ++prod) {
#pragma unroll
            for (int pi = 0; pi < PPI; ++pi) {
              const int tl = iss * PPI + pi;
              const uint32_t a = va + tl * 16 + (prod == 0 ? 8 : 0);
              const uint64_t bd = bslot + (uint64_t)(((tl * 2 + (prod == 1 ? 1 : 0)) * NT * 32) >> 4);
              mma_tf32_ts(tbase + tl * NT, a, bd, idesc, (ks > 0 || prod > 0) ? 1u : 0u);
            }
          }
          if (iss == 0) trace_rec(pl.trace, 17, kg);
          mma_commit(&st_empty[s]);
          mma_commit(&u_empty[us]);
          if (iss == 0) trace_rec(pl.trace, 18, kg);
          if (++s == NS) { s = 0; sph ^= 1; }
          if (++us == NUS) { us = 0; uph ^= 1; }
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
