// Strip variant of the fused Im2col-Winograd kernel (rows a2-a5 of SURVEY.md §8(a)):
// one input-row transform per channel chunk serves all R filter rows, through tcgen05.shift.
//
// Method (§4.1, Fig 2): for tile (n, p, q0) and filter row fh,
//   V_t[(fh,c)] = sum_j BT[t][j] x[n][p-ph+fh][q0-pw+j][c]
// depends on (p, fh) only through the input row rho = p + fh: V_t[(fh,c)](p) = V'_t[c](p + fh).
// The base kernel (fused_tc.cuh) computes V once per (tile, fh), i.e. each input row's
// transform R times. Here a "strip" is one tile column tw of SL <= 32 consecutive input rows
// held by the 32 TMEM lanes of one subpartition (lane j <-> input row rb*RB - ph + j); each lane
// transforms its own row ONCE per 8-channel chunk. The MMAs of filter row fh need lane j to hold
// row j + fh: between filter rows the issuer shifts the V slot up by one lane
// (tcgen05.shift.cta_group::1.down: lane l <- lane l+1 inside each 32-lane subpartition,
// executed in order with the MMAs; tools/shift_bench.cu measured its semantics, ordering and
// ~8-12 cycles per 32-byte column block inside an MMA stream). Lanes j < RB = SL - (R-1) are
// output rows; lanes j >= RB only feed their input rows to the shift (their outputs are never
// stored). Accumulation over fh and c, the output transform y = A^T M and the boundary
// (TMA clipping) are the base kernel's.
//
// Work unit = (strip group sg, output-channel block nb): the 4 consecutive strips 4sg..4sg+3 in
// (n, rb, tw) order, one per subpartition. k-step ks = (channel chunk cc, filter row fh) as in
// the base kernel (same U layout); the V ring holds one CHUNK per slot (R k-steps of MMAs per V).
// Warp roles as the base kernel: 4 transform/epilogue warpgroups (WG g owns the chunks gc = g mod
// 4 and V slot g), one input-TMA warp, one U-ring warp, two MMA issuer warps.
#pragma once
#include "fused_tc.cuh"

namespace i2cw {

// Light profiling (make EXTRA=-DI2CW_LTRACE=1, tools only): per-CTA cycle sums of the pipeline
// phases kept in registers and written once at the end (pl.trace[blockIdx * 32 + k]).
#ifndef I2CW_LTRACE
#define I2CW_LTRACE 0
#endif
__device__ __forceinline__ long long lclock() {
#if I2CW_LTRACE
  long long t;
  asm volatile("mov.u64 %0, %%clock64;" : "=l"(t));
  return t;
#else
  return 0;
#endif
}

// Issuer-side wait for barriers that the pair peer completes remotely. Default: the cluster-scope
// acquire wait. Experiment (I2CW_STRIP_ISSWAIT=1): CTA-scope try_wait with a 64 ns suspend hint
// (a remote arrive does not wake a suspended waiter promptly), no L1 invalidate per wait.
#ifndef I2CW_STRIP_ISSWAIT
#define I2CW_STRIP_ISSWAIT 0  // measured +0.4..0.8% only: the cluster-scope wait is kept (1 = CTA-scope wait with a hint)
#endif
__device__ __forceinline__ bool mbar_try_wait_hint(uint64_t* bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\t"
      "selp.u32 %0, 1, 0, p;\n\t}"
      : "=r"(ok)
      : "r"(smem_u32(bar)), "r"(parity), "r"(64u)
      : "memory");
  return ok != 0;
}
template <bool PAIR>
__device__ __forceinline__ void mbar_wait_iss(uint64_t* bar, uint32_t parity) {
  if constexpr (PAIR && I2CW_STRIP_ISSWAIT) {
    if (mbar_try_wait_hint(bar, parity)) return;
    const uint64_t t0 = globaltimer();
    while (!mbar_try_wait_hint(bar, parity)) {
      if (globaltimer() - t0 > 4000000000ull) __trap();
    }
  } else {
    mbar_wait_tc<PAIR>(bar, parity);
  }
}

template <bool PAIR>
__device__ __forceinline__ void tmem_shift_up_warp(uint32_t taddr) {
  // PTX ".down" moves each row's 32-byte element to the row below in the matrix view, i.e. lane l
  // receives lane l+1's value (measured, tools/shift_bench.cu); one elected lane issues. The
  // cta_group::2 form shifts both CTAs of a pair (tools/shift2_bench.cu).
  if constexpr (PAIR)
    asm volatile(
        "{\n\t.reg .pred e;\n\t"
        "elect.sync _|e, 0xffffffff;\n\t"
        "@e tcgen05.shift.cta_group::2.down [%0];\n\t}" ::"r"(taddr)
        : "memory");
  else
    asm volatile(
        "{\n\t.reg .pred e;\n\t"
        "elect.sync _|e, 0xffffffff;\n\t"
        "@e tcgen05.shift.cta_group::1.down [%0];\n\t}" ::"r"(taddr)
        : "memory");
}

constexpr int kStripLanes = 32;  // input rows per strip box (one TMEM subpartition)
#ifndef I2CW_STRIP_PAIRSTORE
#define I2CW_STRIP_PAIRSTORE 1  // warp pairs store 32-channel boxes (ym.m[1]); 0 = per-warp 16-channel boxes (ym.m[0])
#endif
#ifndef I2CW_STRIP_WARPSTORE
#define I2CW_STRIP_WARPSTORE 1  // per-warp y stores (measured +1..3% over the warpgroup-run stores, 0)
#endif
struct alignas(64) YMaps { CUtensorMap m[4]; };  // y store maps for runs of 1..4 strips

template <int M, int RW, bool PAIR>
struct StripCfg {
  using T = Wino<M, RW>;
  static constexpr int A = T::alpha;
  static constexpr int NT = 64;
  static constexpr int GP = gp_for(A, NT);  // points per pass
  static constexpr int NPASS = A / GP;
  static constexpr int NWG = 4;
  static constexpr int NSLOT = 4;           // V slots (one chunk each, one per warpgroup)
  static constexpr int NISS = niss_for(GP);
  static constexpr int PPI = GP / NISS;
  static constexpr int VCOL = GP * NT;
  static constexpr int BROWS = PAIR ? NT / 2 : NT;               // B rows (output channels) held per CTA
  static constexpr int UBYTES = GP * 2 * BROWS * 32;             // one k-step of this CTA's U (GP points, hi + lo)
  // one strip's input box: 8 ch x (A + 1) cols x 32 rows, smem image [row][col][8 ch] with the TMA
  // 32B swizzle; the 9th column makes the row stride 288 B, so 8 consecutive rows read 8 distinct
  // 16-byte bank groups (a 256-byte stride with any swizzle leaves 2-way conflicts)
  static constexpr int WCOL = A + 1;
  static constexpr int SBOX = WCOL * kStripLanes * 32;
  static constexpr int NTHREADS = NWG * 128 + 64 + NISS * 32;
  static_assert(GP * NT + NSLOT * GP * 16 <= 512, "TMEM budget");
  static_assert(SBOX % 1024 == 0, "boxes stay 1024-aligned");
  static constexpr int TSTRIDE = 2048;  // y staging bytes per strip (32 rows x 64 B)
};

// Plan fields used: strip layout NSTRIP, ROWS (= RB valid rows per strip), PB, T_r, NB; rings
// NUS (U k-step slots), NIS (input stages of 4 strip boxes), NOB, OSTRIDE; items NFULL/NITEMS;
// K-chunk CC0/CC1/ACCUM. xmap: x (C, W, H, N) with box (8, A + 1, 32, 1), 32B swizzle
// (tools/tma_view_test.cu checks the layout). ym.m[L-1]: y (K, Q, P, N) with box (16 ch, L tiles
// at element stride m, ROWS rows, 1 image): one TMA op per run of L strips with the same (n, rb)
// per output column (a box may not start at a negative column, so a run that starts inside the
// unit needs its exact length); swizzle 64B for L = 3, else 128B (conflict-free or 2-way
// staging writes).
// PAIR: a cluster of 2 CTAs on an SM pair, tcgen05.mma.cta_group::2 with M = 256 (each CTA's 4
// strips) and N = 64; each CTA stages only its half of the U rows (halving the per-SM filter
// stream from L2 and the B-operand reads from shared memory). The leader (rank 0) issues all
// MMAs and shifts; the peer's warps arrive remotely on the leader's V / accumulator barriers and
// a peer thread forwards "my U half landed"; commits are multicast to both CTAs.
template <int M, int RW, bool PAIR, bool UCH>
__global__ void __launch_bounds__(StripCfg<M, RW, PAIR>::NTHREADS, 1)
    fused_strip_kernel(const __grid_constant__ CUtensorMap xmap, const __grid_constant__ YMaps ym,
                       const __grid_constant__ Plan pl, const float* __restrict__ u) {
  using Cfg = StripCfg<M, RW, PAIR>;
  using T = typename Cfg::T;
  constexpr int BROWS = Cfg::BROWS;
  const uint32_t rank = PAIR ? cluster_ctarank() : 0u;  // 0 = MMA leader
  constexpr int A = Cfg::A, GP = Cfg::GP, NPASS = Cfg::NPASS, NWG = Cfg::NWG, NSLOT = Cfg::NSLOT;
  constexpr int NISS = Cfg::NISS, PPI = Cfg::PPI, VCOL = Cfg::VCOL, NT = Cfg::NT;
  constexpr uint32_t UBYTES = Cfg::UBYTES, SBOX = Cfg::SBOX;
  constexpr int CPW = NT / NWG;  // epilogue channels per warpgroup (64-byte staging rows)
  const int NIS = pl.NIS, NUS = pl.NUS, R = pl.R, KU = pl.KU;
  constexpr bool uchunk = UCH;                    // one U slot per chunk (KU = R k-steps), else per k-step
  const uint32_t USLOT = (uint32_t)KU * UBYTES;  // one U ring slot: KU k-steps

  extern __shared__ __align__(1024) uint8_t smem[];
  uint8_t* u_smem = smem;                                        // [NUS][KU][UBYTES]
  uint8_t* o_smem = u_smem + (size_t)NUS * USLOT;                // [NWG][NOB][OSTRIDE]
  uint8_t* in_smem = o_smem + (size_t)NWG * pl.NOB * pl.OSTRIDE;  // [NIS][4][SBOX]
  uint64_t* bars = reinterpret_cast<uint64_t*>(in_smem + (size_t)NIS * 4 * SBOX);
  // Input ring: the data stages rotate with gc mod NIS, but "chunk gc landed" is signalled on
  // in_full[gc mod 4], the consuming warpgroup's own barrier. A warpgroup consumes every 4th chunk
  // and its 4 warps are not synchronised with each other, so a per-stage full barrier could be
  // waited on two phases ahead (parity waits alias phase k and k - 2: measured as stale boxes).
  // Per warpgroup, each warp waits every phase of its barrier in order.
  uint64_t* in_full = bars;              // [4]
  uint64_t* in_empty = in_full + 4;      // [NIS]
  uint64_t* st_full = in_empty + NIS;    // [NSLOT]
  uint64_t* st_empty = st_full + NSLOT;  // [NSLOT]
  uint64_t* d_full = st_empty + NSLOT;   // [1]
  uint64_t* d_empty = d_full + 1;        // [1]
  uint64_t* u_full = d_empty + 1;        // [NUS]
  uint64_t* u_empty = u_full + NUS;      // [NUS]
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(u_empty + NUS);
  // [NWG][4] store ops of the pending epilogue (16-byte aligned, after the TMEM slot word)
  int4* epi_ops = reinterpret_cast<int4*>((reinterpret_cast<uintptr_t>(u_empty + NUS + 1) + 15) & ~uintptr_t(15));

  const int warp = threadIdx.x / 32, lane32 = threadIdx.x % 32;
  const int NITEMS = pl.NITEMS;
  // persistent schedule over work units (CTA pairs share a unit: strip groups 2k, 2k + 1)
  const int unit0 = PAIR ? (int)(blockIdx.x >> 1) : (int)blockIdx.x;
  const int ustride = PAIR ? (int)(gridDim.x >> 1) : (int)gridDim.x;
  auto sg0_of = [&](int ui) { return ((PAIR ? 2 * (ui / pl.NB) + (int)rank : ui / pl.NB)) * 4; };
  struct Item { int ui, pb, pe; bool split; };
  auto item_at = [&](int it) {
    Item I;
    if (it < pl.NFULL) { I.ui = it; I.pb = 0; I.pe = NPASS; I.split = false; }
    else { const int h = it - pl.NFULL; I.ui = pl.NFULL + h / 2; I.pb = h % 2; I.pe = I.pb + 1; I.split = true; }
    return I;
  };
  struct Strip { int n, rb, tw; };
  auto strip_at = [&](int sg) {  // strip index -> (image, row block, tile column); tw fastest
    Strip s;
    s.tw = sg % pl.T_r;
    const int r = sg / pl.T_r;
    s.rb = r % pl.PB;
    s.n = r / pl.PB;
    return s;
  };
  const int CC0 = pl.CC0, NCCL = pl.CC1 - pl.CC0;
  // Channel-chunk rotation (SMs do not all stream the same U image at once): a function of the
  // strip-group PAIR and nb only, so the CTA-pair and single-CTA kernels sum every output in the
  // same order (bitwise-identical results; the '*' path may run the single-CTA form)
  auto chunk_of = [&](int ui, int cc) {
    const int sgp = PAIR ? ui / pl.NB : (ui / pl.NB) >> 1, nbu = ui % pl.NB;
    const int cr = (int)(((unsigned)(sgp * pl.NB + nbu) * 5u) % (unsigned)NCCL);
    return CC0 + (cc + cr < NCCL ? cc + cr : cc + cr - NCCL);
  };
  constexpr int PROD_WARP = NWG * 4, UPROD_WARP = PROD_WARP + 1, ISS_WARP0 = NWG * 4 + 2;

  if (threadIdx.x == 0) {
    for (int i = 0; i < 4; ++i) mbar_init(&in_full[i], 1);
    for (int i = 0; i < NIS; ++i) mbar_init(&in_empty[i], 4);
    const int lead2 = PAIR && rank == 0 ? 2 : 1;  // the pair leader also counts the peer's arrivals
    for (int i = 0; i < NSLOT; ++i) { mbar_init(&st_full[i], 4 * lead2); mbar_init(&st_empty[i], NISS); }
    for (int i = 0; i < NUS; ++i) { mbar_init(&u_full[i], lead2); mbar_init(&u_empty[i], NISS); }
    mbar_init(d_full, NISS);
    mbar_init(d_empty, NWG * 4 * lead2);
    fence_mbar_init();
  }
  if (warp == ISS_WARP0) {
    if constexpr (PAIR) { tmem_alloc2(tmem_slot, 512); tmem_relinquish2(); }
    else { tmem_alloc(tmem_slot, 512); tmem_relinquish(); }
  }
  tc_fence_before();
  if constexpr (PAIR) cluster_sync_all();
  else __syncthreads();
  tc_fence_after();
  const uint32_t tbase = *tmem_slot;
#if I2CW_TRACE
  // per-CTA start / end (globaltimer ns) after the 32 x 512 x 2 timeline records
  if (pl.trace != nullptr && threadIdx.x == 0) pl.trace[2 * 32 * 512 + 2 * blockIdx.x] = globaltimer();
#endif

  if (warp < NWG * 4) {
    setmaxnreg_inc<104>();
    // ===================== transform + epilogue warpgroups =====================
    const int g = warp / 4;           // chunks gc = g (mod 4), V slot g
    const int sub = warp % 4;         // TMEM subpartition = strip of the unit
    const int l = threadIdx.x % 128;  // TMEM lane
    const int jr = lane32;            // input row of the strip box held by this lane
    const uint32_t lane_addr = tbase + ((uint32_t)(l & ~31) << 16);
    const uint32_t vslot = lane_addr + VCOL + (uint32_t)g * GP * 16;
    const uint32_t rofs = (uint32_t)jr * (Cfg::WCOL * 32);  // this lane's row in the box
    const bool out_row = jr < pl.ROWS;  // output row of the strip (else: halo input row only)
    uint8_t* ostage = o_smem + (size_t)g * pl.NOB * pl.OSTRIDE;
    const uint32_t st_full_lead = PAIR ? mapa_shared(st_full, 0) : 0u, d_empty_lead = PAIR ? mapa_shared(d_empty, 0) : 0u;
    long long lt[8] = {0, 0, 0, 0, 0, 0, 0, 0};  // I2CW_LTRACE sums: in_full, math, st_empty, sttm, n, d_full, epi, n
    // ---- one chunk of V (this warpgroup's chunk gc of a pass with point group PASS) ----
    auto do_chunk = [&](auto PASS_, int gc) {
      constexpr int PASS = PASS_;
      const int ist = gc % NIS;
      trace_rec(pl.trace, 0 + g, gc / NWG, l == 0);
      long long lt0 = lclock();
      mbar_wait(&in_full[g], (gc / NWG) & 1);
      long long lt1 = lclock();
      lt[0] += lt1 - lt0;
      trace_rec(pl.trace, 4 + g, gc / NWG, l == 0);
      const uint8_t* box = in_smem + ((size_t)ist * 4 + sub) * SBOX;
      // All 16 loads first, then release the box, then the B^T math from registers: the stage is
      // held only for the loads, so the producer refills it while the math runs. The release
      // waits on a branch that reads a sum of every loaded vector (an arrive issued right after the
      // LDS instructions can overtake them -- ptxas adds no wait -- and the next TMA fill would
      // land under the reads); the bit pattern is a signalling NaN, which no sum produces.
      float2 d2[2][A][2];
#pragma unroll
      for (int h = 0; h < 2; ++h)
#pragma unroll
        for (int j = 0; j < A; ++j) {
          const uint32_t o = rofs + (uint32_t)j * 32;  // 32B swizzle: bit 4 ^= bit 7
          const float4 v = *reinterpret_cast<const float4*>(box + ((o ^ ((o >> 3) & 16u)) ^ (uint32_t)(h << 4)));
          d2[h][j][0] = make_float2(v.x, v.y);
          d2[h][j][1] = make_float2(v.z, v.w);
        }
      {
        float2 acc2 = make_float2(0.f, 0.f);
#pragma unroll
        for (int h = 0; h < 2; ++h)
#pragma unroll
          for (int j = 0; j < A; ++j) acc2 = __fadd2_rn(acc2, __fadd2_rn(d2[h][j][0], d2[h][j][1]));
        if (__float_as_uint(acc2.x + acc2.y) != 0x7f800001u) {
          __syncwarp();
          if (lane32 == 0) mbar_arrive(&in_empty[ist]);
        }
      }
      float2 V[GP][4];  // point tl, channel pair cp
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const float2 (&d)[A][2] = d2[h];
        static_for<GP / 2>([&](auto Q_) {
          constexpr int idx0 = PASS * GP + 2 * (int)Q_;
          constexpr int tl0 = 2 * (int)Q_;
#pragma unroll
          for (int p = 0; p < 2; ++p) {
            if constexpr (idx0 == 0) {
              V[tl0][2 * h + p] = bt_dot2<T, 0, 1, 0>(d, p);
              V[tl0 + 1][2 * h + p] = bt_dot2<T, A - 1, 1, 0>(d, p);
            } else {
              constexpr int pa = point_of(idx0, A);
              const float2 E = bt_dot2<T, pa, 2, 0>(d, p);
              const float2 O = bt_dot2<T, pa, 2, 1>(d, p);
              V[tl0][2 * h + p] = __fadd2_rn(E, O);
              V[tl0 + 1][2 * h + p] = __ffma2_rn(make_float2(-1.f, -1.f), O, E);
            }
          }
        });
      }
      trace_rec(pl.trace, 8 + g, gc / NWG, l == 0);
      lt0 = lclock();
      lt[1] += lt0 - lt1;
      const int use = gc / NSLOT;
      if (use > 0) mbar_wait_tc<PAIR>(&st_empty[g], (use - 1) & 1);
      lt1 = lclock();
      lt[2] += lt1 - lt0;
      trace_rec(pl.trace, 12 + g, gc / NWG, l == 0);
      tc_fence_after();
#pragma unroll
      for (int t = 0; t < GP; ++t) {
        float v16[16];
#pragma unroll
        for (int cp = 0; cp < 4; ++cp) {
          float2 hi, lo;
          split_tf32x2(V[t][cp], hi, lo);
          v16[2 * cp] = hi.x; v16[2 * cp + 1] = hi.y;
          v16[8 + 2 * cp] = lo.x; v16[8 + 2 * cp + 1] = lo.y;
        }
        tmem_st_x16(vslot + t * 16, v16);
      }
      tmem_wait_st();
      tc_fence_before();
      __syncwarp();
      if (lane32 == 0) {
        if (PAIR && rank == 1) mbar_arrive_remote(st_full_lead + 8u * (uint32_t)g);
        else mbar_arrive(&st_full[g]);
      }
      trace_rec(pl.trace, 16 + g, gc / NWG, l == 0);
      lt[3] += lclock() - lt1;
      lt[4] += 1;
    };

    // ---- epilogue of one pass: y (+)= A^T M via shared memory + TMA ----
    struct Epi { int gpass, pass, sg0, nb; bool split; };
    auto do_epilogue = [&](auto PASS_, const Epi& E) {
      constexpr int PASS = PASS_;
      const int nvalid = max(0, min(4, pl.NSTRIP - E.sg0));  // 0: a pair's idle half
#if !I2CW_STRIP_WARPSTORE
      // runs of the unit: strips with the same (n, rb) (a run starts at s = 0 or where tw = 0).
      // This warp's strip sub is tile t = sub - r0 of the run [r0, r0 + rl); the run's staging
      // region starts at r0 * TSTRIDE and holds [row][rl tiles][16 ch] (the box image of map rl)
      int r0 = 0, rl = 1;
      for (int s = 1; s <= sub; ++s)
        if (s < nvalid && strip_at(E.sg0 + s).tw == 0) r0 = s;
      while (r0 + rl < nvalid && strip_at(E.sg0 + r0 + rl).tw != 0) ++rl;
      // a run of 4 is stored as 3 + 1 tiles: with 64-byte staging rows the 4-tile box image puts
      // 8 consecutive rows of one tile in 2 bank groups (4-way conflicts, measured), 3 and 1 tiles
      // are conflict-free
      if (rl == 4) { if (sub < r0 + 3) rl = 3; else { r0 += 3; rl = 1; } }
      // staging offset of this lane's row (bytes, before the swizzle) and the swizzle of map rl
      // (64B for rl = 3: chunk bits [5:4] ^= [8:7]; else 128B: [6:4] ^= [9:7])
      const uint32_t obase = (uint32_t)(r0 * Cfg::TSTRIDE + (jr * rl + (sub - r0)) * 64);
      const uint32_t oxor = ((obase >> 7) & 3u) << 4;
      const bool live = out_row && sub < nvalid;
      // the unit's TMA store ops (one per run piece), computed once for all columns by thread 0
      // into shared memory: {staging start s | (length - 1) << 8, column tw m, row, image}
      int4* ops = epi_ops + g * 4;
      int nops = 0;
      if (l == 0) {
        int cur_s = 0, cur_L = 0;
        for (int s = 0; s < nvalid; ++s) {
          const Strip st = strip_at(E.sg0 + s);
          if (s == 0 || st.tw == 0 || cur_L == 3) {
            ops[nops] = make_int4(s, st.tw * M, st.rb * pl.ROWS, st.n);
            cur_s = s; cur_L = 1;
            ++nops;
          } else {
            ++cur_L;
          }
          ops[nops - 1].x = cur_s | ((cur_L - 1) << 8);
        }
      }
#endif
      trace_rec(pl.trace, 20 + g, 2 * E.gpass, l == 0);
      const long long le0 = lclock();
      mbar_wait_tc<PAIR>(d_full, E.gpass & 1);
      const long long le1 = lclock();
      lt[5] += le1 - le0;
      trace_rec(pl.trace, 20 + g, 2 * E.gpass + 1, l == 0);
      tc_fence_after();
      const int cbase = g * CPW;
      float mv[GP][CPW];
#pragma unroll
      for (int t = 0; t < GP; ++t) tmem_ld_x16(lane_addr + t * NT + cbase, &mv[t][0]);
      tmem_wait_ld();
      tc_fence_before();
      __syncwarp();
      if (lane32 == 0) {  // accumulators read: the next pass's MMAs may start
        if (PAIR && rank == 1) mbar_arrive_remote(d_empty_lead);
        else mbar_arrive(d_empty);
      }
      if (ABL(4)) return;  // DEBUG timing ablation: no output transform / y
      static_for<GP / 2>([&](auto Q_) {  // pair (a, a+1): AT[i][a+1] = (-1)^i AT[i][a]
        constexpr int idx0 = PASS * GP + 2 * (int)Q_;
        constexpr int tl0 = 2 * (int)Q_;
        if constexpr (idx0 != 0) {
#pragma unroll
          for (int e = 0; e < CPW; e += 2) {
            const float2 a = make_float2(mv[tl0][e], mv[tl0][e + 1]), b = make_float2(mv[tl0 + 1][e], mv[tl0 + 1][e + 1]);
            const float2 sa = __fadd2_rn(a, b), da = __ffma2_rn(make_float2(-1.f, -1.f), b, a);
            mv[tl0][e] = sa.x; mv[tl0][e + 1] = sa.y;
            mv[tl0 + 1][e] = da.x; mv[tl0 + 1][e + 1] = da.y;
          }
        }
      });
#if I2CW_STRIP_WARPSTORE && I2CW_STRIP_PAIRSTORE
      // Warp-pair stores: warps (g, sub) and (g ^ 1, sub) stage their 16-channel halves of the
      // strip's rows into one [row][32 ch] buffer (128-byte rows, 128B swizzle, conflict-free) and
      // the even warp issues one 32-channel box per column: half the TMA ops of per-warp stores,
      // one 64-thread named barrier per column.
      {
        const bool mine = sub < nvalid;
        Strip ms = strip_at(E.sg0 + (mine ? sub : 0));
        const int gp = g >> 1, hh = g & 1;
        const int pid = gp * 4 + sub;  // warp pair: named barrier 1 + pid, staging buffers
        const bool lead = hh == 0;
        uint8_t* pbase = o_smem + (size_t)pid * pl.NOB * 4096;
        const uint32_t rbase = (uint32_t)(jr * 128);
        const uint32_t rsw = (uint32_t)(jr & 7);
        if (lead && lane32 == 0) {
          bulk_wait_group_read_dyn(pl.NOB - 1);
          if (PASS > 0 && !E.split) bulk_wait_group_all();  // this pair's pass-0 stores of the unit landed
        }
        named_bar_sync(1 + pid, 64);
        const bool store = PASS == 0 && !E.split && !pl.ACCUM;
        static_for<M>([&](auto I_) {
          constexpr int i = I_;
          const int ob = i % pl.NOB;
          uint8_t* stg = pbase + (size_t)ob * 4096;
#pragma unroll
          for (int j = 0; j < CPW / 4; ++j) {
            float2 o[2] = {make_float2(0.f, 0.f), make_float2(0.f, 0.f)};
            static_for<GP / 2>([&](auto Q_) {
              constexpr int idx0 = PASS * GP + 2 * (int)Q_;
              constexpr int tl0 = 2 * (int)Q_;
              if constexpr (idx0 == 0) {
                constexpr float c0 = T::AT(i, 0), c1 = T::AT(i, A - 1);
#pragma unroll
                for (int e = 0; e < 2; ++e) {
                  const float2 m0 = make_float2(mv[tl0][4 * j + 2 * e], mv[tl0][4 * j + 2 * e + 1]);
                  const float2 m1 = make_float2(mv[tl0 + 1][4 * j + 2 * e], mv[tl0 + 1][4 * j + 2 * e + 1]);
                  if constexpr (c0 != 0.f) o[e] = __ffma2_rn(make_float2(c0, c0), m0, o[e]);
                  if constexpr (c1 != 0.f) o[e] = __ffma2_rn(make_float2(c1, c1), m1, o[e]);
                }
              } else {
                constexpr float ca = T::AT(i, point_of(idx0, A));
                constexpr int src = (i % 2 == 0) ? tl0 : tl0 + 1;
#pragma unroll
                for (int e = 0; e < 2; ++e) {
                  const float2 mz = make_float2(mv[src][4 * j + 2 * e], mv[src][4 * j + 2 * e + 1]);
                  if constexpr (ca == 1.f) o[e] = __fadd2_rn(o[e], mz);
                  else if constexpr (ca != 0.f) o[e] = __ffma2_rn(make_float2(ca, ca), mz, o[e]);
                }
              }
            });
            if (out_row && mine)
              *reinterpret_cast<float4*>(stg + rbase + ((((uint32_t)(hh * 4 + j)) ^ rsw) << 4)) =
                  make_float4(o[0].x, o[0].y, o[1].x, o[1].y);
          }
          fence_proxy_async_smem();
          // the buffer the next column writes was last read by column i + 1 - NOB
          if (lead && lane32 == 0) bulk_wait_group_read_dyn(pl.NOB - 2);
          named_bar_sync(1 + pid, 64);
          if (lead && lane32 == 0) {
            if (mine && !ABL(32)) {
              if (store) tma_store_4d(&ym.m[1], stg, E.nb * NT + gp * 32, ms.tw * M + i, ms.rb * pl.ROWS, ms.n);
              else tma_reduce_add_4d(&ym.m[1], stg, E.nb * NT + gp * 32, ms.tw * M + i, ms.rb * pl.ROWS, ms.n);
            }
            bulk_commit_group();
          }
        });
        if (lead && lane32 == 0) bulk_wait_group_read<0>();
        lt[6] += lclock() - le1;
        lt[7] += 1;
        return;
      }
#elif I2CW_STRIP_WARPSTORE
      // Per-warp stores: warp (g, sub) stages its own strip's rows (64-byte rows, 64B swizzle,
      // conflict-free) and its lane 0 issues that strip's box (16 channels x 1 tile x ROWS rows)
      // per output column -- no warpgroup barrier, each warp tracks its own bulk groups.
      {
        const bool mine = sub < nvalid;
        Strip ms = strip_at(E.sg0 + (mine ? sub : 0));
        const uint32_t wbase = (uint32_t)(sub * Cfg::TSTRIDE + jr * 64);
        const uint32_t wxor = ((wbase >> 7) & 3u) << 4;
        if (lane32 == 0) {
          bulk_wait_group_read_dyn(pl.NOB - 1);
          if (PASS > 0 && !E.split) bulk_wait_group_all();  // this warp's pass-0 stores of the unit landed
        }
        __syncwarp();
        const bool store = PASS == 0 && !E.split && !pl.ACCUM;
        static_for<M>([&](auto I_) {
          constexpr int i = I_;
          const int ob = i % pl.NOB;
          uint8_t* stg = ostage + (size_t)ob * pl.OSTRIDE;
#pragma unroll
          for (int j = 0; j < CPW / 4; ++j) {
            float2 o[2] = {make_float2(0.f, 0.f), make_float2(0.f, 0.f)};
            static_for<GP / 2>([&](auto Q_) {
              constexpr int idx0 = PASS * GP + 2 * (int)Q_;
              constexpr int tl0 = 2 * (int)Q_;
              if constexpr (idx0 == 0) {
                constexpr float c0 = T::AT(i, 0), c1 = T::AT(i, A - 1);
#pragma unroll
                for (int e = 0; e < 2; ++e) {
                  const float2 m0 = make_float2(mv[tl0][4 * j + 2 * e], mv[tl0][4 * j + 2 * e + 1]);
                  const float2 m1 = make_float2(mv[tl0 + 1][4 * j + 2 * e], mv[tl0 + 1][4 * j + 2 * e + 1]);
                  if constexpr (c0 != 0.f) o[e] = __ffma2_rn(make_float2(c0, c0), m0, o[e]);
                  if constexpr (c1 != 0.f) o[e] = __ffma2_rn(make_float2(c1, c1), m1, o[e]);
                }
              } else {
                constexpr float ca = T::AT(i, point_of(idx0, A));
                constexpr int src = (i % 2 == 0) ? tl0 : tl0 + 1;
#pragma unroll
                for (int e = 0; e < 2; ++e) {
                  const float2 mz = make_float2(mv[src][4 * j + 2 * e], mv[src][4 * j + 2 * e + 1]);
                  if constexpr (ca == 1.f) o[e] = __fadd2_rn(o[e], mz);
                  else if constexpr (ca != 0.f) o[e] = __ffma2_rn(make_float2(ca, ca), mz, o[e]);
                }
              }
            });
            if (out_row && mine)
              *reinterpret_cast<float4*>(stg + ((wbase + (uint32_t)j * 16u) ^ wxor)) = make_float4(o[0].x, o[0].y, o[1].x, o[1].y);
          }
          fence_proxy_async_smem();
          __syncwarp();
          if (lane32 == 0) {
            if (mine && !ABL(32)) {
              const uint8_t* src = stg + sub * Cfg::TSTRIDE;
              if (store) tma_store_4d(&ym.m[0], src, E.nb * NT + cbase, ms.tw * M + i, ms.rb * pl.ROWS, ms.n);
              else tma_reduce_add_4d(&ym.m[0], src, E.nb * NT + cbase, ms.tw * M + i, ms.rb * pl.ROWS, ms.n);
            }
            bulk_commit_group();
            // the buffer the next column writes was last read by column i + 1 - NOB
            bulk_wait_group_read_dyn(pl.NOB - 1);
          }
          __syncwarp();
        });
        if (lane32 == 0) bulk_wait_group_read<0>();
        lt[6] += lclock() - le1;
        lt[7] += 1;
        return;
      }
#endif
#if !I2CW_STRIP_WARPSTORE
      trace_rec(pl.trace, 28 + (g == 0 ? 3 : 0), 0, false);
      if (l == 0) {
        bulk_wait_group_read_dyn(pl.NOB - 1);
        if (PASS > 0 && !E.split) bulk_wait_group_all();  // the pass-0 stores of this unit landed
      }
      named_bar_sync(1 + g, 128);
      trace_rec(pl.trace, 24 + g, E.gpass * 8 + 6, l == 0);
      static_for<M>([&](auto I_) {
        constexpr int i = I_;
        const int ob = i % pl.NOB;
        uint8_t* stg = ostage + (size_t)ob * pl.OSTRIDE;
#pragma unroll
        for (int j = 0; j < CPW / 4; ++j) {
          float2 o[2] = {make_float2(0.f, 0.f), make_float2(0.f, 0.f)};
          static_for<GP / 2>([&](auto Q_) {
            constexpr int idx0 = PASS * GP + 2 * (int)Q_;
            constexpr int tl0 = 2 * (int)Q_;
            if constexpr (idx0 == 0) {
              constexpr float c0 = T::AT(i, 0), c1 = T::AT(i, A - 1);
#pragma unroll
              for (int e = 0; e < 2; ++e) {
                const float2 m0 = make_float2(mv[tl0][4 * j + 2 * e], mv[tl0][4 * j + 2 * e + 1]);
                const float2 m1 = make_float2(mv[tl0 + 1][4 * j + 2 * e], mv[tl0 + 1][4 * j + 2 * e + 1]);
                if constexpr (c0 != 0.f) o[e] = __ffma2_rn(make_float2(c0, c0), m0, o[e]);
                if constexpr (c1 != 0.f) o[e] = __ffma2_rn(make_float2(c1, c1), m1, o[e]);
              }
            } else {
              constexpr float ca = T::AT(i, point_of(idx0, A));
              constexpr int src = (i % 2 == 0) ? tl0 : tl0 + 1;
#pragma unroll
              for (int e = 0; e < 2; ++e) {
                const float2 ms = make_float2(mv[src][4 * j + 2 * e], mv[src][4 * j + 2 * e + 1]);
                if constexpr (ca == 1.f) o[e] = __fadd2_rn(o[e], ms);
                else if constexpr (ca != 0.f) o[e] = __ffma2_rn(make_float2(ca, ca), ms, o[e]);
              }
            }
          });
          if (live)
            *reinterpret_cast<float4*>(stg + ((obase + (uint32_t)j * 16u) ^ oxor)) = make_float4(o[0].x, o[0].y, o[1].x, o[1].y);
        }
        fence_proxy_async_smem();
        if (l == 0) bulk_wait_group_read_dyn(pl.NOB - 2);
        named_bar_sync(1 + g, 128);
        if (l == 0) {
          const uint8_t* sbuf = ostage + (size_t)ob * pl.OSTRIDE;
          const bool store = PASS == 0 && !E.split && !pl.ACCUM;
          // one TMA op per run: columns tw m + i for the run's L tiles, rows [rb ROWS, +ROWS)
          // (rows >= P and columns >= Q clipped by the TMA unit: the in-kernel boundary)
#pragma unroll 1
          for (int k = 0; k < nops; ++k) {
            if (ABL(32)) break;  // DEBUG timing ablation: no y writes
            const int4 op = ops[k];
            const uint8_t* src = sbuf + (op.x & 0xff) * Cfg::TSTRIDE;
            const CUtensorMap* ymp = &ym.m[op.x >> 8];
            if (store) tma_store_4d(ymp, src, E.nb * NT + cbase, op.y + i, op.z, op.w);
            else tma_reduce_add_4d(ymp, src, E.nb * NT + cbase, op.y + i, op.z, op.w);
          }
          bulk_commit_group();
        }
        trace_rec(pl.trace, 24 + g, E.gpass * 8 + i, l == 0);
      });
      if (l == 0) bulk_wait_group_read<0>();
      lt[6] += lclock() - le1;
      lt[7] += 1;
      trace_rec(pl.trace, 24 + g, E.gpass * 8 + 7, l == 0);
#endif
    };
    auto epilogue = [&](const Epi& E) {
      static_for<NPASS>([&](auto P_) { if ((int)P_ == E.pass) do_epilogue(P_, E); });
    };

    // Schedule: a pass's epilogue is deferred until after this warpgroup's FIRST chunk of the
    // next pass (whose V slot frees as the pass's own MMAs complete), so while the MMAs drain
    // the warpgroups already stage the next pass, and the next pass's first 4 chunks (one per
    // warpgroup) are ready the moment every warpgroup has read its accumulators (d_empty).
    // Only one chunk may run ahead: the next one would wait for MMAs that wait for d_empty.
    int pc = 0;  // passes done
    int gc = 0;  // global chunk counter (all passes of all items of this CTA)
    bool pend = false;
    Epi pe{0, 0, 0, 0, false};
    for (int it = unit0; it < NITEMS; it += ustride) {
      const Item I = item_at(it);
      const int sg0 = sg0_of(I.ui), nb = I.ui % pl.NB;
      for (int pass = I.pb; pass < I.pe; ++pass) {
        const int gpass = pc++;
        for (int cc = 0; cc < NCCL; ++cc, ++gc) {
          if ((gc & (NWG - 1)) != g) continue;
          static_for<NPASS>([&](auto P_) { if ((int)P_ == pass) do_chunk(P_, gc); });
          if (pend) { epilogue(pe); pend = false; }
        }
        if (pend) { epilogue(pe); pend = false; }  // no chunk of this pass for this warpgroup
        pe = Epi{gpass, pass, sg0, nb, I.split};
        pend = true;
      }
    }
    if (pend) epilogue(pe);
#if I2CW_LTRACE
    if (pl.trace != nullptr && lane32 == 0 && sub == 0)
      for (int k = 0; k < 8; ++k) pl.trace[(size_t)blockIdx.x * 48 + g * 8 + k] = lt[k];
#endif
  } else {
    setmaxnreg_dec<64>();
    if (warp == PROD_WARP) {
      // ====================== input strip boxes (TMA) ======================
      if (lane32 == 0) {
        tma_prefetch_desc(&xmap);
        for (int L = 0; L < 4; ++L) tma_prefetch_desc(&ym.m[L]);
        asm volatile("griddepcontrol.wait;" ::: "memory");
        int ist = 0, iph = 0, first = 1, gcp = 0;
        for (int it = unit0; it < NITEMS; it += ustride) {
          const Item I = item_at(it);
          const int sg0 = sg0_of(I.ui);
          Strip st[4];
#pragma unroll
          for (int s = 0; s < 4; ++s) st[s] = strip_at(min(sg0 + s, pl.NSTRIP - 1));
          for (int pass = I.pb; pass < I.pe; ++pass) {
            for (int cc = 0; cc < NCCL; ++cc, ++gcp) {
              if (!first) mbar_wait(&in_empty[ist], iph ^ 1);
              trace_rec(pl.trace, 31, gcp);
              const int ca = chunk_of(I.ui, cc);
              uint64_t* full = &in_full[gcp & 3];
              if (ABL(8)) { mbar_arrive(full); if (++ist == NIS) { ist = 0; iph ^= 1; first = 0; } continue; }
              mbar_expect_tx(full, 4u * SBOX);
#pragma unroll
              for (int s = 0; s < 4; ++s)
                tma_load_4d(in_smem + ((size_t)ist * 4 + s) * SBOX, &xmap, full, ca * 8,
                            st[s].tw * M - pl.pad_w, st[s].rb * pl.ROWS - pl.pad_h, st[s].n);
              if (++ist == NIS) { ist = 0; iph ^= 1; first = 0; }
            }
          }
        }
      }
      __syncwarp();
    } else if (warp == UPROD_WARP) {
      // ================= U (transformed filter) k-step ring =================
      if (lane32 == 0) {
        asm volatile("griddepcontrol.wait;" ::: "memory");
        if (!I2CW_NO_TAGCHECK && blockIdx.x == 0) {
          const UTag* tg = reinterpret_cast<const UTag*>(reinterpret_cast<const uint8_t*>(u) - kUTagBytes);
          if (tg->magic != kUMagic || (int)tg->alpha != A || (int)tg->m != M || (int)tg->is_deconv != pl.is_deconv ||
              (int)tg->C != pl.C || (int)tg->K != pl.K || (int)tg->R != pl.R || (int)tg->S != RW ||
              (int)tg->NT != NT || (int)tg->halves != (PAIR ? 2 : 1) || (int)tg->T != 1)
            __trap();
        }
        const size_t kstride = (size_t)A * 2 * NT * 8;  // floats per k-step
        int us = 0, uph = 0, first = 1;
        for (int it = unit0; it < NITEMS; it += ustride) {
          const Item I = item_at(it);
          const int nb = I.ui % pl.NB;
          for (int pass = I.pb; pass < I.pe; ++pass) {
            // this CTA's B rows of the pass's GP points, hi + lo, contiguous (pair: its N half)
            const float* src0 = u + (PAIR ? u_offset_pair(NT, A, nb, pl.NKS, 0, (int)rank, pass * GP)
                                          : u_offset(NT, A, nb, pl.NKS, 0, pass * GP, 0));
            for (int cc = 0; cc < NCCL; ++cc) {
              const int ca = chunk_of(I.ui, cc);
              for (int fh = 0; fh < R; ++fh) {
                const int kin = uchunk ? fh : 0;  // position in the U slot
                if (kin == 0) {
                  if (!first) mbar_wait_tc<PAIR>(&u_empty[us], uph ^ 1);
                  if (ABL(16)) mbar_arrive(&u_full[us]);
                  else mbar_expect_tx(&u_full[us], USLOT);
                }
                if (!ABL(16))
                  bulk_load(u_smem + (size_t)us * USLOT + (size_t)kin * UBYTES, src0 + (size_t)(ca * R + fh) * kstride,
                            UBYTES, &u_full[us]);
                if (!uchunk || fh == R - 1) { if (++us == NUS) { us = 0; uph ^= 1; first = 0; } }
              }
            }
          }
        }
      }
      __syncwarp();
    } else {
      // ============================= MMA issuers =============================
      const int iss = warp - ISS_WARP0;  // owns points tl = iss * PPI .. + PPI - 1
      constexpr uint32_t idesc = idesc_tf32(PAIR ? 256 : 128, NT);
      const uint64_t bdesc0 = umma_desc_kmajor_noswizzle(smem_u32(u_smem), BROWS * 16, 128);
      int us = 0, uph = 0, gc = 0, gpass = 0;
      long long ilt[4] = {0, 0, 0, 0};  // I2CW_LTRACE: st_full waits, u_full waits, d_empty waits, total
      const long long ilt_start = lclock();
      if (PAIR && rank == 1) {
        // pair peer: forward "my U half landed" to the leader's U slot (off the critical path:
        // the U ring runs ahead)
        if (iss == 0 && lane32 == 0) {
          const uint32_t lead_ufull = mapa_shared(u_full, 0);
          for (int it = unit0; it < NITEMS; it += ustride) {
            const Item I = item_at(it);
            for (int pass = I.pb; pass < I.pe; ++pass)
              for (int k = 0; k < NCCL * (uchunk ? 1 : R); ++k) {
                mbar_wait(&u_full[us], uph);  // this CTA's own U half (local TMA completion)
                mbar_arrive_remote(lead_ufull + 8u * (uint32_t)us);
                if (++us == NUS) { us = 0; uph ^= 1; }
              }
          }
        }
      } else
      for (int it = unit0; it < NITEMS; it += ustride) {
        const Item I = item_at(it);
        for (int pass = I.pb; pass < I.pe; ++pass, ++gpass) {
          if (gpass > 0) {
            const long long dt0 = lclock();
            mbar_wait_iss<PAIR>(d_empty, (gpass - 1) & 1);
            ilt[2] += lclock() - dt0;
            tc_fence_after();
          }
          for (int cc = 0; cc < NCCL; ++cc, ++gc) {
            const int slot = gc & (NSLOT - 1);
            trace_rec(pl.trace, 28, gc, iss == 0 && lane32 == 0);
            long long it0 = lclock();
            mbar_wait_iss<PAIR>(&st_full[slot], (gc / NSLOT) & 1);
            ilt[0] += lclock() - it0;
            trace_rec(pl.trace, 29, gc, iss == 0 && lane32 == 0);
            tc_fence_after();
            const uint32_t va = tbase + VCOL + (uint32_t)slot * GP * 16;
            for (int fh = 0; fh < R; ++fh) {
              const int kin = uchunk ? fh : 0;
              if (kin == 0) {
                it0 = lclock();
                mbar_wait_iss<PAIR>(&u_full[us], uph);  // pair: both halves (the peer's arrives remotely)
                ilt[1] += lclock() - it0;
                tc_fence_after();
              }
              const uint64_t bk = bdesc0 + (uint64_t)((us * USLOT + kin * UBYTES) >> 4);
              if (!ABL(2)) {
#pragma unroll
              for (int prod = 0; prod < 3; ++prod) {
#pragma unroll
                for (int pi = 0; pi < PPI; ++pi) {
                  const int tl = iss * PPI + pi;
                  const uint32_t a = va + tl * 16 + (prod == 0 ? 8 : 0);
                  const uint64_t bd = bk + (uint64_t)(((tl * 2 + (prod == 1 ? 1 : 0)) * BROWS * 32) >> 4);
                  const uint32_t acc = (cc > 0 || fh > 0 || prod > 0) ? 1u : 0u;
                  if constexpr (PAIR) mma2_tf32_ts_warp(tbase + tl * NT, a, bd, idesc, acc);
                  else mma_tf32_ts_warp(tbase + tl * NT, a, bd, idesc, acc);
                }
              }
              }
              if (!uchunk || fh == R - 1) {
                if constexpr (PAIR) mma_commit2_warp(&u_empty[us]);
                else mma_commit_warp(&u_empty[us]);
                if (++us == NUS) { us = 0; uph ^= 1; }
              }
              if (fh + 1 < R && !ABL(2)) {  // next filter row: lane j takes lane j+1's input row
#pragma unroll
                for (int pi = 0; pi < PPI; ++pi) {
                  const int tl = iss * PPI + pi;
                  tmem_shift_up_warp<PAIR>(va + tl * 16);
                  tmem_shift_up_warp<PAIR>(va + tl * 16 + 8);
                }
              }
            }
            if constexpr (PAIR) mma_commit2_warp(&st_empty[slot]);
            else mma_commit_warp(&st_empty[slot]);
            trace_rec(pl.trace, 30, gc, iss == 0 && lane32 == 0);
          }
          if constexpr (PAIR) mma_commit2_warp(d_full);
          else mma_commit_warp(d_full);
        }
      }
#if I2CW_LTRACE
      ilt[3] = lclock() - ilt_start;
      if (pl.trace != nullptr && lane32 == 0 && iss == 0)
        for (int k = 0; k < 4; ++k) pl.trace[(size_t)blockIdx.x * 48 + 32 + k] = ilt[k];
#endif
      __syncwarp();
    }
  }

  tc_fence_before();
  if constexpr (PAIR) cluster_sync_all();
  else __syncthreads();
#if I2CW_TRACE
  if (pl.trace != nullptr && threadIdx.x == 0) pl.trace[2 * 32 * 512 + 2 * blockIdx.x + 1] = globaltimer();
#endif
  if (warp == ISS_WARP0) {
    tc_fence_after();
    if constexpr (PAIR) tmem_dealloc2(tbase, 512);
    else tmem_dealloc(tbase, 512);
  }
}

template <int M, int RW, bool PAIR>
static cudaError_t launch_strip_t2(const CUtensorMap& xmap, const YMaps& ym, const Plan& pl, const float* u,
                                  cudaStream_t stream) {
  using Cfg = StripCfg<M, RW, PAIR>;
  auto kern = pl.KU > 1 ? fused_strip_kernel<M, RW, PAIR, true> : fused_strip_kernel<M, RW, PAIR, false>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, pl.smem_bytes);
  if (e != cudaSuccess) return e;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(persistent_ctas(pl.NITEMS, PAIR ? 2 : 1));
  cfg.blockDim = dim3(Cfg::NTHREADS);
  cfg.dynamicSmemBytes = pl.smem_bytes;
  cfg.stream = stream;
  cudaLaunchAttribute attr[2];
  int na = 0;
  if constexpr (PAIR) {
    attr[na].id = cudaLaunchAttributeClusterDimension;
    attr[na].val.clusterDim.x = 2;
    attr[na].val.clusterDim.y = 1;
    attr[na].val.clusterDim.z = 1;
    ++na;
  }
  attr[na].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[na].val.programmaticStreamSerializationAllowed = 1;
  ++na;
  cfg.attrs = attr;
  cfg.numAttrs = na;
  e = cudaLaunchKernelEx(&cfg, kern, xmap, ym, pl, u);
  if (e != cudaSuccess) return e;
  return cudaGetLastError();
}

}  // namespace i2cw
