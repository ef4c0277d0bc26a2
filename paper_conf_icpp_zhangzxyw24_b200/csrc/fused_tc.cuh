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
//    rows of the block as one 8-channel (32-byte, TMA-swizzled) box (OOB zero fill = padding,
//    PAPER.md:337-338); the rows are reused across all fh (vertical overlap)
//    and by neighbouring windows (the (r-1) horizontal overlap, §5.4).
//    The same warp streams each k-step's U image (1D bulk copy) into a ring.
//  * a3: NWG transform warpgroups (thread = tile) read the alpha-window from
//    shared memory, apply BT with zeros/±1 folded at compile time and the ±
//    pair trick, split 3xTF32 hi/lo and write V into TMEM
//    with tcgen05.st (V is the UMMA A operand, "TS" mode: no SMEM read for A).
//  * a4: NISS issuer warps, each owning GP/NISS points' accumulators, issue per
//    k-step 3 tcgen05.mma.kind::tf32 per point (lo*hi, hi*lo, hi*hi). A single
//    lane issuing in a loop manages one UMMA per ~45 cycles, a warp issuing
//    warp-uniformly (elect.sync inside the asm) the full 32 cycles of a 128x64x8
//    UMMA (tools/mma_bench.cu); two such warps split the points. Each accumulator
//    has exactly one issuer, so results are bitwise deterministic.
//  * k-step stages: NS slots, each = V (TMEM) + U (SMEM); one "full" barrier
//    (128 transform arrivals + U tx bytes) and one "empty" barrier (NISS commits).
//  * a5: the warpgroups tcgen05.ld the accumulators, apply A^T in registers
//    (pair trick), stage 8-channel slices in shared memory and TMA-store them
//    (TMA clips q >= Q, p >= P, k >= K: the in-kernel boundary). Passes > 0 use a
//    TMA reduce-add into y (the accumulators hold GP of alpha points per pass).
#pragma once
#include <cstdlib>
#include <utility>

#include "common.cuh"
#include "transforms_generated.h"

// Timing ablations (I2CW_ABLATE, results wrong) exist only in builds with -DI2CW_ABLATION=1
// (make ABLATION=1); the production kernel carries no ablation branches.
#define ABL(b) (I2CW_ABLATION && (pl.ablate & (b)))

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

// Packed (sm_100 FFMA2/FADD2/FMUL2) form of bt_dot over one channel pair p: d[j][p] holds
// channels (2p, 2p+1) of input position j. Halves the FP issue slots of the transform.
template <class T, int PT, int JSTEP, int JOFF, int A>
__host__ __device__ constexpr int bt_first_nz() {
  for (int j = 0; j < A; ++j)
    if (j % JSTEP == JOFF && T::BT(PT, j) != 0.f) return j;
  return -1;
}
template <class T, int PT, int JSTEP, int JOFF, int A>
__device__ __forceinline__ float2 bt_dot2(const float2 (&d)[A][2], int p) {
  constexpr int j0 = bt_first_nz<T, PT, JSTEP, JOFF, A>();
  if constexpr (j0 < 0) {
    return make_float2(0.f, 0.f);
  } else {
    constexpr float c0 = T::BT(PT, j0);
    float2 acc = c0 == 1.f ? d[j0][p] : __fmul2_rn(make_float2(c0, c0), d[j0][p]);
    static_for<A>([&](auto J) {
      constexpr int j = J;
      if constexpr (j > j0 && j % JSTEP == JOFF) {
        constexpr float c = T::BT(PT, j);
        if constexpr (c == 1.f) acc = __fadd2_rn(acc, d[j][p]);
        else if constexpr (c != 0.f) acc = __ffma2_rn(make_float2(c, c), d[j][p], acc);
      }
    });
    return acc;
  }
}
// 3xTF32 operand split of a channel pair (reading R10): hi = v rounded to tf32 (11
// significant bits, exactly representable, so the tensor core's own fp32->tf32 conversion does
// not matter), lo = v - hi (exact in fp32; the tensor core drops lo's low bits, < 2^-22 |v|).
// I2CW_SPLIT (build-time): 2 = Veltkamp splitting p = (2^13 + 1) v, hi = p - (p - v): round to
// nearest (ties to even) in 3 packed FP ops, so lo takes either sign and its truncation by the
// tensor core is unbiased (valid while |v| < FLT_MAX / 8193 ~ 4e34); 1 = the same rounding
// (ties away) with integer ops, +5% kernel time (profiles/r02_ab_split.txt); 0 = truncation
// (hi = v & ~0x1fff; lo one-signed: measured mean error on U[1,2] +60%).
#ifndef I2CW_SPLIT
#define I2CW_SPLIT 2
#endif
#ifndef I2CW_NO_TAGCHECK
#define I2CW_NO_TAGCHECK 0      // experiment switch: 1 = no device-side U tag check
#endif
__device__ __forceinline__ void split_tf32x2(float2 v, float2& hi, float2& lo) {
  const float2 neg1 = make_float2(-1.f, -1.f);
#if I2CW_SPLIT == 2
  const float2 p = __fmul2_rn(make_float2(8193.f, 8193.f), v);
  hi = __ffma2_rn(neg1, __ffma2_rn(neg1, v, p), p);  // p - (p - v)
#elif I2CW_SPLIT == 1
  hi.x = __uint_as_float((__float_as_uint(v.x) + 0x1000u) & 0xFFFFE000u);
  hi.y = __uint_as_float((__float_as_uint(v.y) + 0x1000u) & 0xFFFFE000u);
#else
  hi.x = __uint_as_float(__float_as_uint(v.x) & 0xFFFFE000u);
  hi.y = __uint_as_float(__float_as_uint(v.y) & 0xFFFFE000u);
#endif
  lo = __ffma2_rn(neg1, hi, v);
}

template <int M, int RW, int NT, bool PAIR>
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
  // one k-step of U in this CTA's shared memory (GP points, hi+lo); a CTA pair splits N
  static constexpr int UBYTES = GP * 2 * NT * 32 / (PAIR ? 2 : 1);
  static constexpr int BROWS = PAIR ? NT / 2 : NT;    // B rows (output channels) held per CTA
  static constexpr int NTHREADS = tc_threads(GP, NT);
  static constexpr int PPI = GP / NISS;               // points per issuer

  static_assert(A % GP == 0 && GP % 2 == 0, "passes must hold whole ± pairs");
  static_assert(NS >= 2 && NS % NWG == 0, "stage ring");
  static_assert(GP * NT + NS * GP * 16 <= TMEM_COLS, "TMEM budget");
  static_assert(NT % 16 == 0 && NT >= 16 && NT <= 256, "UMMA N for M=128");
  static_assert(!PAIR || (NT % 32 == 0 && NT >= 32), "UMMA N for cta_group::2, M=256");
  static_assert((NT / NWG) % 8 == 0, "epilogue column split");
  static_assert(GP % NISS == 0, "issuer split");
};

// PAIR = true: a cluster of 2 CTAs on an SM pair runs tcgen05.mma.cta_group::2 with
// M = 256 (each CTA's 128 tiles) and N = NT; each CTA stages only its half of the U rows
// (BROWS = NT/2 output channels), halving the U fill and the B-operand reads per SM. The
// leader (rank 0) issues all MMAs; the peer's "relay" thread forwards "my V stage and U
// half are in place" with one remote mbarrier arrive per k-step, and its epilogue's "D
// read" with one per pass. Commits are multicast to the barriers of both CTAs.
// VOL = true: 3D convolution ("expanding Stage1 Im2col to ND, while remaining
// Stage2 unchanged"). x is [N][D][H][W][C], the filter [K][T][R][S][C] is used as the 2D filter
// [K][T*R][S][C] (so U and the filter transform are the 2D ones with R' = T*R), and a "chunk" of
// the K loop is a virtual chunk vc = cc * T + fd: channel chunk cc at depth tap fd, staged as one
// input box at depth d0 - pad_d + fd. The NI slices a tile block stacks are consecutive OUTPUT
// depths of one image (2D: consecutive images). Stage 2 (the 1D Winograd along W) is unchanged.
// P1 = true: the 1xTF32 precision mode ("1xTF32 with looser tolerance"):
// only the hi*hi product per point (one UMMA instead of three), V stored as its
// round-to-nearest tf32 hi only; U still carries hi and lo, the lo images are not read.
template <int M, int RW, int NT, bool PAIR, bool VOL = false, bool P1 = false>
__global__ void __launch_bounds__(TcCfg<M, RW, NT, PAIR>::NTHREADS, 1)
    fused_tc_kernel(const __grid_constant__ CUtensorMap xmap, const __grid_constant__ CUtensorMap ymap,
                    const __grid_constant__ Plan pl, const float* __restrict__ u) {
  using Cfg = TcCfg<M, RW, NT, PAIR>;
  using T = typename Cfg::T;
  constexpr int A = Cfg::A, GP = Cfg::GP, NS = Cfg::NS, NISS = Cfg::NISS, NWG = Cfg::NWG;
  constexpr int NPASS = Cfg::NPASS, VCOL = Cfg::VCOL, PPI = Cfg::PPI, BROWS = Cfg::BROWS;
  const int NIS = pl.NIS;  // input stages (runtime: fills the shared-memory budget)
#ifndef I2CW_CSPLIT
#define I2CW_CSPLIT 0  // experiment: 1 = two warpgroups per k-step, split by channel quads
#endif
  constexpr bool CS = I2CW_CSPLIT && NWG == 4 && !P1;
#ifndef I2CW_UWAIT_WG
#define I2CW_UWAIT_WG 0  // experiment: 1 = the transform warpgroups (not the issuer) wait for U
#endif
  // UW: each transform warpgroup checks its k-step's U super-slot (while it waits for its V slot
  // anyway) before arriving; the issuer's one wait per super-stage then covers V and U
  constexpr bool UW = I2CW_UWAIT_WG;
#ifndef I2CW_ISS_LOOKAHEAD
#define I2CW_ISS_LOOKAHEAD 0  // experiment: 1 = issuer waits for super-stage j+1 inside j's issue
#endif
  constexpr bool LA = I2CW_ISS_LOOKAHEAD && kps_for(A, NT) >= 2;
  constexpr uint32_t UBYTES = Cfg::UBYTES;
  const uint32_t rank = PAIR ? cluster_ctarank() : 0u;  // 0 = MMA leader

  // k-step V slots in TMEM and their grouping into super-stages of KPS k-steps: one
  // full/empty barrier pair and one U slot per super-stage, so the MMA issuers pay one
  // wait + commit per KPS k-steps (measured: ~400 cycles of barrier work per k-step with
  // KPS = 1, above the 384 cycles of UMMA work of a 4-point, N=64 k-step).
  constexpr int NSLOT = NS;                       // V slots in TMEM (k-step kg uses slot kg % NSLOT)
  static_assert(NSLOT % NWG == 0 && (NSLOT & (NSLOT - 1)) == 0 && (NWG & (NWG - 1)) == 0,
                "V slots: a power of 2, a whole number per warpgroup");
  constexpr int KPS = kps_for(A, NT);             // k-steps per super-stage
  constexpr int NSS = NSLOT / KPS;                // super-stages
  // epilogue: warpgroup g owns output channels [16g, 16g + 16): one 64-byte staging row per tile
  // and output column, NOB buffers per warpgroup
  constexpr int CPW = NT / NWG;                   // epilogue channels per warpgroup
  static_assert(CPW == 16 || CPW == 32, "epilogue channel split (64B / 128B staging rows)");

  extern __shared__ __align__(1024) uint8_t smem[];
  const uint32_t inplane = (uint32_t)pl.PLANE;  // half an input stage (stages 1024-aligned)
  const int NUS = pl.NUS;                         // U super-slots (runtime: SMEM budget)
  constexpr uint32_t USBYTES = KPS * UBYTES;      // one U super-slot
  uint8_t* u_smem = smem;                                        // [NUS][USBYTES]        (1024-aligned)
  uint8_t* o_smem = u_smem + (size_t)NUS * USBYTES;              // [NWG][NOB][OSTRIDE]   (1024-aligned)
  uint8_t* in_smem = o_smem + (size_t)NWG * pl.NOB * pl.OSTRIDE;  // [NIS][2 * PLANE]
  uint64_t* bars = reinterpret_cast<uint64_t*>(in_smem + (size_t)NIS * 2 * inplane);
  uint64_t* in_full = bars;             // [NIS]
  uint64_t* in_empty = in_full + NIS;   // [NIS]
  uint64_t* st_full = in_empty + NIS;   // [NSS]
  uint64_t* st_empty = st_full + NSS;   // [NSLOT]: one per V slot (its k-step's MMAs completed)
  uint64_t* r_full = st_empty + NSLOT;  // [NSS]  (unused since the peer arrives directly; keeps the layout)
  uint64_t* d_full = r_full + NSS;      // [1]
  uint64_t* d_empty = d_full + 1;       // [1]
  uint64_t* u_full = d_empty + 1;       // [NUS]
  uint64_t* u_empty = u_full + NUS;     // [NUS]
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(u_empty + NUS);

  const int warp = threadIdx.x / 32, lane32 = threadIdx.x % 32;
  // Persistent schedule: a work unit is (tile block tb, output-channel block nb); CTA (pair) c
  // takes units c, c + G, c + 2G, ... (G = number of CTAs, or of CTA pairs). Both CTAs of a
  // pair share nb and take consecutive tile blocks. The producers run ahead across units, so
  // the next unit's input rows and filter stream are in flight during this unit's epilogue.
  // Work items: items < NFULL are whole units (all passes); the NITEMS - NFULL items after them
  // split the last (tail) units into one item per pass (NPASS = 2 only, y pre-zeroed by the
  // host, both passes reduce-add: 0 + a + b is exact in either order, so results stay
  // deterministic). A tail of T <= #CTAs/2 units then costs half a unit time instead of one.
  const int NITEMS = pl.NITEMS;
  const int unit0 = PAIR ? (int)(blockIdx.x >> 1) : (int)blockIdx.x;
  const int ustride = PAIR ? (int)(gridDim.x >> 1) : (int)gridDim.x;
  struct Item { int ui, pb, pe; bool split; };
  auto item_at = [&](int it) {
    Item I;
    if (it < pl.NFULL) { I.ui = it; I.pb = 0; I.pe = NPASS; I.split = false; }
    else { const int h = it - pl.NFULL; I.ui = pl.NFULL + h / 2; I.pb = h % 2; I.pe = I.pb + 1; I.split = true; }
    return I;
  };
  struct Unit { int nb, tb, seg, n, d0, p0, crot; bool active; };
  auto unit_at = [&](int ui) {
    Unit U;
    U.nb = ui % pl.NB;
    U.tb = PAIR ? 2 * (ui / pl.NB) + (int)rank : ui / pl.NB;
    U.active = U.tb < pl.tile_blocks;  // odd tile-block count: the last peer only helps the MMA
    U.seg = U.tb % pl.SEGS;
    const int tbr = U.tb / pl.SEGS;
    U.p0 = (tbr % pl.PB) * pl.ROWS;
    if constexpr (VOL) {  // image block = (image n, NI output depths from d0)
      const int ib = tbr / pl.PB;
      U.n = ib / pl.DB;
      U.d0 = (ib - U.n * pl.DB) * pl.NI;
    } else {
      U.n = (tbr / pl.PB) * pl.NI;
      U.d0 = 0;
    }
    // Channel-chunk rotation: unit ui walks the chunks starting at crot, so SMs do not all
    // stream the same U image at the same time. Both CTAs of a pair rotate alike (their MMAs
    // consume the same k-step). The summation order is a function of the unit: results stay
    // run-to-run deterministic.
    U.crot = (int)(((unsigned)ui * 5u) % (unsigned)(pl.CC1 - pl.CC0));
    return U;
  };
  // This launch's channel chunks [CC0, CC1) (the whole K loop, or one K-chunk of it: the host
  // launches long K loops as several chunks, each accumulated from zero in TMEM and added into y
  // by the TMA reduce-add). NKS = this launch's k-steps.
  const int CC0 = pl.CC0, NCCL = pl.CC1 - pl.CC0;
  const int NKS = NCCL * pl.R;
  const int NKSP = (NKS + KPS - 1) / KPS * KPS;   // k-steps per pass padded to whole super-stages
#ifndef I2CW_ROLE_SWAP
#define I2CW_ROLE_SWAP 0  // experiment: 1 = issuer warps on SMSPs 0/1, producers on 2/3
#endif
  constexpr int PROD_WARP = NWG * 4 + (I2CW_ROLE_SWAP ? NISS : 0), UPROD_WARP = PROD_WARP + 1,
                ISS_WARP0 = NWG * 4 + (I2CW_ROLE_SWAP ? 0 : 2);

  if (threadIdx.x == 0) {
    // transform-warp arrivals are warp-elected (one lane after __syncwarp): 128 or 512
    // per-thread arrivals on one barrier word serialise in the shared-memory atomic unit
    for (int i = 0; i < NIS; ++i) { mbar_init(&in_full[i], 1); mbar_init(&in_empty[i], NWG * 4); }
    for (int i = 0; i < NSS; ++i) {
      // the 4 warps of each of the KPS warpgroups of this super-stage; a pair leader also counts
      // the peer's 4 x KPS warps, which arrive remotely (no relay thread on the V path)
      mbar_init(&st_full[i], KPS * 4 * (CS ? 2 : 1) * (PAIR && rank == 0 ? 2 : 1));
    }
    for (int i = 0; i < NSLOT; ++i) mbar_init(&st_empty[i], NISS);
    // pair leader's U slot: its own expect_tx arrive + the peer's "my half landed" arrive
    for (int i = 0; i < NUS; ++i) { mbar_init(&u_full[i], PAIR && rank == 0 ? 2 : 1); mbar_init(&u_empty[i], NISS); }
    mbar_init(d_full, NISS);
    mbar_init(d_empty, NWG * 4 * (PAIR && rank == 0 ? 2 : 1));  // pair: the peer's warps arrive remotely
    fence_mbar_init();
  }
  if (warp == ISS_WARP0) {  // the first issuer warp owns the TMEM allocation
    if constexpr (PAIR) { tmem_alloc2(tmem_slot, Cfg::TMEM_COLS); tmem_relinquish2(); }
    else { tmem_alloc(tmem_slot, Cfg::TMEM_COLS); tmem_relinquish(); }
  }
  tc_fence_before();
  if constexpr (PAIR) cluster_sync_all();
  else __syncthreads();
  tc_fence_after();
  const uint32_t tbase = *tmem_slot;

  // Register split (640-thread configs launch at 96 registers per thread): the transform /
  // epilogue warpgroups take 104, the producer + issuer warpgroup keeps 64 (the CTA's pool is
  // only what the launch allocated: 4 x 128 x 8 = 128 x 32 released).
  constexpr bool kRegSplit = Cfg::NTHREADS == 640;
  if (warp < NWG * 4) {
    if constexpr (kRegSplit) setmaxnreg_inc<104>();
    // ===================== transform + epilogue warpgroups =====================
    const int g = warp / 4;           // k-steps kg = g (mod NWG), V slots kg % NSLOT
    // CS (channel split, I2CW_CSPLIT): warpgroups 2p and 2p+1 share the k-steps kg = p (mod 2),
    // each transforming and storing one 4-channel quad (hs = g & 1) of every point: half the
    // loads, math and TMEM stores per warpgroup per k-step, a shorter slot round trip.
    const int kpar = CS ? (g >> 1) : g, hs = g & 1;
    const int l = threadIdx.x % 128;  // TMEM lane == tile slot
    const int row_l = pl.lane_row[l], tw_l = pl.lane_tw[l], in_l = pl.lane_in[l];
    const bool has_slot = row_l != 0xFF;
    const int col0 = has_slot ? tw_l * M : 0;
    const uint32_t lane_addr = tbase + ((uint32_t)(l & ~31) << 16);
    const int TSM = pl.TS * M;  // output columns per CTA row segment
    // Epilogue staging (warpgroup-private): buffer ob holds output column i of this warpgroup's
    // CPW channels for every tile, one CPW*4-byte row per tile (TMA 64B / 128B swizzle).
    float* ostage = reinterpret_cast<float*>(o_smem + (size_t)g * pl.NOB * pl.OSTRIDE);
    const int orow = has_slot ? row_l * pl.TS + tw_l : 0;
    // 16-byte chunk swizzle of the TMA store box rows: 64B rows (CPW 16) XOR (row >> 1) & 3,
    // 128B rows (CPW 32) XOR row & 7
    const int oswz = CPW == 16 ? (orow >> 1) & 3 : orow & 7;
    // Warpgroup g owns V slot g and computes the k-steps kg = g (mod NWG) of every pass
    // (kg = PASS * NKSP + cc * R + fh): the four warpgroups' transforms interleave on the
    // SMSPs, each k-step's full V (GP points x 8 channels, hi + lo) written by one warpgroup.
    const uint32_t vbase0 = lane_addr + VCOL;
    // "V of this k-step stored" / "accumulators read": local arrive, or for the pair peer a remote
    // arrive on the leader's barrier (the leader's MMAs read this CTA's TMEM; tcgen05.wait::st has
    // completed the stores before the arrive)
    const uint32_t st_full_lead = PAIR ? mapa_shared(st_full, 0) : 0u, d_empty_lead = PAIR ? mapa_shared(d_empty, 0) : 0u;
    auto arrive_st_full = [&](int idx) {
      if (PAIR && rank == 1) mbar_arrive_remote(st_full_lead + 8u * (uint32_t)idx);
      else mbar_arrive(&st_full[idx]);
    };
    auto arrive_d_empty = [&]() {
      if (PAIR && rank == 1) mbar_arrive_remote(d_empty_lead);
      else mbar_arrive(d_empty);
    };
    auto wait_slot = [&](int kg) {  // this slot's previous k-step consumed (tcgen05.commit per k-step)
      if constexpr (UW) {  // this k-step's U super-slot landed (both halves on a pair leader)
        if (!PAIR || rank == 0) {
          const int sg = kg / KPS;
          mbar_wait_tc<PAIR>(&u_full[sg % pl.NUS], (sg / pl.NUS) & 1);
        }
      }
      const int use = kg / NSLOT;
      if (use > 0) mbar_wait_tc<PAIR>(&st_empty[kg & (NSLOT - 1)], (use - 1) & 1);
    };
    int ist = 0, iph = 0;  // input ring slot / phase (incremental: no runtime division)
    int pc = 0;            // passes done by this CTA
    for (int it = unit0; it < NITEMS; it += ustride) {
    const Item I = item_at(it);
    const Unit U = unit_at(I.ui);
    static_for<NPASS>([&](auto PASS_) {
      constexpr int PASS = PASS_;
      if (PASS < I.pb || PASS >= I.pe) return;
      const int gpass = pc++;
      const int kgp = gpass * NKSP;  // global index of this pass's first k-step
      for (int cc = 0; cc < NCCL; ++cc) {
        const int kb = kgp + cc * pl.R;  // global index of the chunk's first k-step
        trace_rec(pl.trace, 19 + g, PASS * pl.NCC + cc, l == 0);
        // every warpgroup waits for every chunk (also one it has no k-step in, R < NWG) so
        // its in_empty arrival can never run ahead into the slot's next phase
        mbar_wait(&in_full[ist], iph);
        trace_rec(pl.trace, 23 + g, PASS * pl.NCC + cc, l == 0);
        const uint8_t* stage = in_smem + (size_t)ist * 2 * inplane;  // [NI*HBOX][WBOX][8 ch], 32B-swizzled
        for (int fh = CS ? ((kpar - kb) & 1) : ((g - kb) & (NWG - 1)); fh < pl.R; fh += CS ? 2 : NWG) {
          const int kg = kb + fh;
          trace_rec(pl.trace, 0 + g, kg / NWG, l == 0);
          // V for this k-step computed into registers BEFORE waiting for the V slot: the slot
          // round trip (MMA of the slot's previous k-step -> commit -> here) then covers only
          // the split + TMEM stores, not the shared-memory loads and the B^T math.
          if constexpr (CS) {
            float2 Vh[GP][2];  // point tl, channel pair p of this warpgroup's quad hs
            {
              const int x0 = (in_l + fh) * pl.WBOX + col0;
              const uint8_t* xrow = stage + (size_t)x0 * 32;
              float2 d[A][2];
#pragma unroll
              for (int j = 0; j < A; ++j) {
                const int sw = ((x0 + j) & 4) << 2;  // 16 * bit2(xs)
                const float4 v = *reinterpret_cast<const float4*>(xrow + j * 32 + (hs ? 16 - sw : sw));
                d[j][0] = make_float2(v.x, v.y);
                d[j][1] = make_float2(v.z, v.w);
              }
              static_for<GP / 2>([&](auto Q_) {
                constexpr int idx0 = PASS * GP + 2 * (int)Q_;
                constexpr int tl0 = 2 * (int)Q_;
#pragma unroll
                for (int p = 0; p < 2; ++p) {
                  if constexpr (idx0 == 0) {
                    Vh[tl0][p] = bt_dot2<T, 0, 1, 0>(d, p);
                    Vh[tl0 + 1][p] = bt_dot2<T, A - 1, 1, 0>(d, p);
                  } else {
                    constexpr int pa = point_of(idx0, A);
                    const float2 E = bt_dot2<T, pa, 2, 0>(d, p);
                    const float2 O = bt_dot2<T, pa, 2, 1>(d, p);
                    Vh[tl0][p] = __fadd2_rn(E, O);
                    Vh[tl0 + 1][p] = __ffma2_rn(make_float2(-1.f, -1.f), O, E);
                  }
                }
              });
            }
            wait_slot(kg);
            tc_fence_after();
            trace_rec(pl.trace, 4 + g, kg / NWG, l == 0);
            const uint32_t vbase = vbase0 + (uint32_t)(kg & (NSLOT - 1)) * GP * 16 + 4 * hs;
            // point tl: hi of this quad's 4 channels at columns 16 tl + 4 hs, lo at 16 tl + 8 + 4 hs
#pragma unroll
            for (int t = 0; t < GP; ++t) {
              float2 h0, l0, h1, l1;
              split_tf32x2(Vh[t][0], h0, l0);
              split_tf32x2(Vh[t][1], h1, l1);
              tmem_st_x4(vbase + t * 16, h0.x, h0.y, h1.x, h1.y);
              tmem_st_x4(vbase + t * 16 + 8, l0.x, l0.y, l1.x, l1.y);
            }
            trace_rec(pl.trace, 12 + g, kg / NWG, l == 0);
            tmem_wait_st();
            tc_fence_before();
            __syncwarp();
            if (lane32 == 0) arrive_st_full((kg / KPS) % NSS);
            trace_rec(pl.trace, 8 + g, kg / NWG, l == 0);
            continue;
          }
          float2 V[GP][4];  // point tl, channel pair cp (channels 2cp, 2cp+1 of the chunk)
          if (ABL(1)) {  // DEBUG timing ablation: V = 0 without loads or math
#pragma unroll
            for (int t = 0; t < GP; ++t)
#pragma unroll
              for (int cp = 0; cp < 4; ++cp) V[t][cp] = make_float2(0.f, 0.f);
          } else {
            // idle lanes (has_slot false: lane_in = 0, col0 = 0) read a valid window of row fh;
            // their V only feeds accumulator rows that are never stored. Unconditional loads
            // avoid zeroing 16 float4 per k-step.
            // Position xs of the staged box holds 8 channels (32 bytes); the TMA 32B swizzle
            // stores channel quad h at 16 * (h ^ bit2(xs)), so the 8 lanes of a quarter-warp
            // (distinct xs mod 8, host lane permutation) hit 8 distinct 16-byte bank groups.
            const int x0 = (in_l + fh) * pl.WBOX + col0;
            const uint8_t* xrow = stage + (size_t)x0 * 32;
#pragma unroll
            for (int h = 0; h < 2; ++h) {  // channel quads
              float2 d[A][2];
#pragma unroll
              for (int j = 0; j < A; ++j) {
                const int sw = ((x0 + j) & 4) << 2;  // 16 * bit2(xs)
                const float4 v = *reinterpret_cast<const float4*>(xrow + j * 32 + (h ? 16 - sw : sw));
                d[j][0] = make_float2(v.x, v.y);
                d[j][1] = make_float2(v.z, v.w);
              }
              static_for<GP / 2>([&](auto Q_) {
                constexpr int idx0 = PASS * GP + 2 * (int)Q_;  // internal index of this pair slot
                constexpr int tl0 = 2 * (int)Q_;
#pragma unroll
                for (int p = 0; p < 2; ++p) {
                  if constexpr (idx0 == 0) {  // singles: point 0 and point alpha-1
                    V[tl0][2 * h + p] = bt_dot2<T, 0, 1, 0>(d, p);
                    V[tl0 + 1][2 * h + p] = bt_dot2<T, A - 1, 1, 0>(d, p);
                  } else {  // ± pair (a, a+1): E over even j, O over odd j
                    constexpr int pa = point_of(idx0, A);
                    const float2 E = bt_dot2<T, pa, 2, 0>(d, p);
                    const float2 O = bt_dot2<T, pa, 2, 1>(d, p);
                    V[tl0][2 * h + p] = __fadd2_rn(E, O);
                    V[tl0 + 1][2 * h + p] = __ffma2_rn(make_float2(-1.f, -1.f), O, E);
                  }
                }
              });
            }
          }
          wait_slot(kg);
          tc_fence_after();
          trace_rec(pl.trace, 4 + g, kg / NWG, l == 0);
          const uint32_t vbase = vbase0 + (uint32_t)(kg & (NSLOT - 1)) * GP * 16;
          // point tl -> 16 TMEM columns: hi of channels 0..7, then lo of channels 0..7
#pragma unroll
          for (int t = 0; t < GP; ++t) {
            if (ABL(256)) break;  // DEBUG timing ablation: no TMEM stores of V
            if constexpr (P1) {  // 1xTF32: hi only (8 columns)
              float v8[8];
#pragma unroll
              for (int cp = 0; cp < 4; ++cp) {
                float2 hi, lo;
                split_tf32x2(V[t][cp], hi, lo);
                v8[2 * cp] = hi.x; v8[2 * cp + 1] = hi.y;
              }
              tmem_st_x8(vbase + t * 16, v8);
              continue;
            }
            float v16[16];
#pragma unroll
            for (int cp = 0; cp < 4; ++cp) {
              float2 hi, lo;
              split_tf32x2(V[t][cp], hi, lo);
              v16[2 * cp] = hi.x; v16[2 * cp + 1] = hi.y;
              v16[8 + 2 * cp] = lo.x; v16[8 + 2 * cp + 1] = lo.y;
            }
            tmem_st_x16(vbase + t * 16, v16);
          }
          trace_rec(pl.trace, 12 + g, kg / NWG, l == 0);
          tmem_wait_st();
          tc_fence_before();
          __syncwarp();
          if (lane32 == 0) arrive_st_full((kg / KPS) % NSS);
          trace_rec(pl.trace, 8 + g, kg / NWG, l == 0);
        }
        __syncwarp();
        if (lane32 == 0) mbar_arrive(&in_empty[ist]);
        if (++ist == NIS) { ist = 0; iph ^= 1; }
      }
      // padding k-steps of the last super-stage (NKS not a multiple of KPS): no V, but the
      // owning warpgroup still takes its turn so the super-stage's arrival count is met
      for (int kl = NKS; kl < NKSP; ++kl) {
        const int kg = kgp + kl;
        if (CS ? ((kg & 1) != kpar) : ((kg & (NWG - 1)) != g)) continue;
        wait_slot(kg);
        tc_fence_before();
        __syncwarp();
        if (lane32 == 0) arrive_st_full((kg / KPS) % NSS);
      }
      // ---------- epilogue of this pass: y (+)= A^T M via shared memory + TMA ----------
      trace_rec(pl.trace, 27, 2 * gpass, l == 0 && g == 0);
      mbar_wait_tc<PAIR>(d_full, gpass & 1);  // completed by tcgen05.commit
      tc_fence_after();
      trace_rec(pl.trace, 27, 2 * gpass + 1, l == 0 && g == 0);
      // Each accumulator is read from TMEM exactly once (TMEM reads run at 64 B/cycle/SM): the
      // GP points x 16 channels of this warpgroup go to registers (the issuers may then start the
      // next pass), the ± pair sums/differences are formed in place, and the M output columns
      // are produced one at a time. Column i of every tile, y[q0 + i][16g .. 16g+16), is one
      // 64-byte staging row; one TMA store per column writes the box, walking Q with element
      // stride m (positions q0 + i). One named barrier per column: before it, thread 0 makes
      // sure the store that last used the NEXT column's buffer has finished reading it.
      const int qbase = U.seg * TSM;
      const int cbase = g * CPW;
      if (ABL(4)) {  // DEBUG timing ablation: release the accumulators, no y
        tc_fence_before();
        __syncwarp();
        if (lane32 == 0) arrive_d_empty();
      } else {
        float mv[GP][CPW];
#pragma unroll
        for (int t = 0; t < GP; ++t)
#pragma unroll
          for (int c16 = 0; c16 < CPW / 16; ++c16) tmem_ld_x16(lane_addr + t * NT + cbase + 16 * c16, &mv[t][16 * c16]);
        tmem_wait_ld();
        tc_fence_before();
        __syncwarp();
        if (lane32 == 0) arrive_d_empty();  // accumulators read: the next pass may overwrite them
        trace_rec(pl.trace, 28, 128 + 2 * gpass, l == 0 && g == 0);
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
        if (l == 0) {
          bulk_wait_group_read_dyn(pl.NOB - 1);  // buffer 0: previous pass's stores
          // a later pass of the same unit reduce-adds onto what the previous pass wrote: those
          // writes must be complete (bulk operations are not ordered with each other). Waited
          // here, a whole mainloop after they were issued, instead of at the end of that pass
          // where the wait sat on the next pass's first V (thread 0 is in warp 0 of the group)
          if (PASS > 0 && !I.split) bulk_wait_group_all();
        }
        named_bar_sync(1 + g, 128);
        trace_rec(pl.trace, 28, 129 + 2 * gpass, l == 0 && g == 0);
        static_for<M>([&](auto I_) {
          constexpr int i = I_;
          const int ob = i % pl.NOB;
          trace_rec(pl.trace, 27, 64 + 4 * (gpass * M + i), l == 0 && g == 0);
          float4* stg = reinterpret_cast<float4*>(ostage + (size_t)ob * (pl.OSTRIDE / 4)) + (size_t)orow * (CPW / 4);
#pragma unroll
          for (int j = 0; j < CPW / 4; ++j) {  // channel quads: y column i = sum over the pass's points
            // channel pairs in packed f32x2 (FFMA2 / FADD2)
            float2 o[2] = {make_float2(0.f, 0.f), make_float2(0.f, 0.f)};
            static_for<GP / 2>([&](auto Q_) {
              constexpr int idx0 = PASS * GP + 2 * (int)Q_;
              constexpr int tl0 = 2 * (int)Q_;
              if constexpr (idx0 == 0) {  // singles: point 0 and point alpha-1
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
                constexpr int src = (i % 2 == 0) ? tl0 : tl0 + 1;  // sum (even i) or difference (odd i)
#pragma unroll
                for (int e = 0; e < 2; ++e) {
                  const float2 ms = make_float2(mv[src][4 * j + 2 * e], mv[src][4 * j + 2 * e + 1]);
                  if constexpr (ca == 1.f) o[e] = __fadd2_rn(o[e], ms);
                  else if constexpr (ca != 0.f) o[e] = __ffma2_rn(make_float2(ca, ca), ms, o[e]);
                }
              }
            });
            if (has_slot && !(ABL(64))) stg[j ^ oswz] = make_float4(o[0].x, o[0].y, o[1].x, o[1].y);
          }
          trace_rec(pl.trace, 27, 66 + 4 * (gpass * M + i), l == 0 && g == 0);
          fence_proxy_async_smem();
          // the store that last read the next column's buffer (column i + 1 - NOB) must be done
          if (l == 0) bulk_wait_group_read_dyn(pl.NOB - 2);
          trace_rec(pl.trace, 27, 67 + 4 * (gpass * M + i), l == 0 && g == 0);
          named_bar_sync(1 + g, 128);
          trace_rec(pl.trace, 27, 65 + 4 * (gpass * M + i), l == 0 && g == 0);
          if (l == 0) {
            const float* box = ostage + (size_t)ob * (pl.OSTRIDE / 4);
            if (U.active && !(ABL(32))) {  // DEBUG ablation 32: no y stores
              // first pass of the first K-chunk stores; others add (DEBUG ablation 512: stores only)
              if constexpr (VOL) {
                if (PASS == 0 && !I.split && !pl.ACCUM)
                  tma_store_5d(&ymap, box, U.nb * NT + cbase, qbase + i, U.p0, U.d0, U.n);
                else tma_reduce_add_5d(&ymap, box, U.nb * NT + cbase, qbase + i, U.p0, U.d0, U.n);
              } else {
                if ((PASS == 0 && !I.split && !pl.ACCUM) || ABL(512))
                  tma_store_4d(&ymap, box, U.nb * NT + cbase, qbase + i, U.p0, U.n);
                else tma_reduce_add_4d(&ymap, box, U.nb * NT + cbase, qbase + i, U.p0, U.n);
              }
            }
            bulk_commit_group();
          }
        });
      }
      // staging buffers free for the next pass (its writes complete later, see above)
      if (l == 0) bulk_wait_group_read<0>();
      trace_rec(pl.trace, 28, gpass, l == 0 && g == 0);
    });
    }  // units
  } else {
   if constexpr (kRegSplit) setmaxnreg_dec<64>();
   if (warp == PROD_WARP) {
    // ====================== input-row TMA producer ======================
    if (lane32 == 0) {
      tma_prefetch_desc(&xmap);
      tma_prefetch_desc(&ymap);
      // programmatic dependent launch: the prologue above overlapped the previous kernel;
      // its results (x, U) are visible only after this wait
      asm volatile("griddepcontrol.wait;" ::: "memory");
      int ist = 0, iph = 0, first = 1;  // slot, round parity, still in the first round
      for (int it = unit0; it < NITEMS; it += ustride) {
      const Item I = item_at(it);
      const Unit U = unit_at(I.ui);
      const int wstart = U.seg * pl.TS * M - pl.pad_w;
      const int hstart = U.p0 - pl.pad_h;
      for (int pass = I.pb; pass < I.pe; ++pass) {
        for (int cc = 0; cc < NCCL; ++cc) {
          if (!first) mbar_wait(&in_empty[ist], iph ^ 1);
          uint8_t* dst = in_smem + (size_t)ist * 2 * inplane;
          const int ca = CC0 + (cc + U.crot < NCCL ? cc + U.crot : cc + U.crot - NCCL);  // actual chunk
          if (ABL(16)) {  // DEBUG timing ablation: no input rows (stage reused as is)
            mbar_arrive(&in_full[ist]);
          } else {
            mbar_expect_tx(&in_full[ist], (uint32_t)pl.BOXB);
            if constexpr (VOL) {  // virtual chunk ca = channel chunk * T + depth tap
              const int cch = ca / pl.T, fd = ca - cch * pl.T;
              tma_load_5d(dst, &xmap, &in_full[ist], cch * 8, wstart, hstart, U.d0 - pl.pad_d + fd, U.n);
            } else {
              tma_load_4d(dst, &xmap, &in_full[ist], ca * 8, wstart, hstart, U.n);
            }
          }
          if (++ist == NIS) { ist = 0; iph ^= 1; first = 0; }
        }
      }
      }  // units
    }
    __syncwarp();
  } else if (warp == UPROD_WARP) {
    // ================= U (transformed filter) super-slot ring =================
    if (lane32 == 0) {
      asm volatile("griddepcontrol.wait;" ::: "memory");  // U written by the previous kernel
      // the device tag in front of U must describe this call (the host validated a copy of it;
      // a stale host copy for a reused address must not run a mismatched filter silently)
      if (!I2CW_NO_TAGCHECK && blockIdx.x == 0) {
        const UTag* tg = reinterpret_cast<const UTag*>(reinterpret_cast<const uint8_t*>(u) - kUTagBytes);
        if (tg->magic != kUMagic || (int)tg->alpha != A || (int)tg->m != M || (int)tg->is_deconv != pl.is_deconv ||
            (int)tg->C != pl.C || (int)tg->K != pl.K || (int)tg->R != pl.R || (int)tg->S != RW ||
            (int)tg->NT != NT || (int)tg->halves != (PAIR ? 2 : 1) || (int)tg->T != pl.T)
          __trap();
      }
      const size_t kstride = (size_t)A * 2 * NT * 8;  // floats per k-step (both layouts)
      int us = 0, uph = 0, first = 1;
      for (int it = unit0; it < NITEMS; it += ustride) {
      const Item I = item_at(it);
      const Unit U = unit_at(I.ui);
      for (int pass = I.pb; pass < I.pe; ++pass) {
        // this CTA's B rows of the pass's GP points, hi+lo, contiguous (pair: its N half)
        const float* src0 = u + (PAIR ? u_offset_pair(NT, A, U.nb, pl.NKS, 0, (int)rank, pass * GP)
                                      : u_offset(NT, A, U.nb, pl.NKS, 0, pass * GP, 0));
        for (int kl0 = 0; kl0 < NKSP; kl0 += KPS) {
          trace_rec(pl.trace, 30, pass * NKSP + kl0);
          if (!first) mbar_wait_tc<PAIR>(&u_empty[us], uph ^ 1);  // completed by tcgen05.commit
          trace_rec(pl.trace, 31, pass * NKSP + kl0);
          const int nreal = NKS - kl0 < KPS ? NKS - kl0 : KPS;
          const uint32_t ub = (ABL(8)) ? 1024u : UBYTES;  // DEBUG timing ablation: shrink
          mbar_expect_tx(&u_full[us], (uint32_t)nreal * ub);
          for (int pos = 0; pos < nreal; ++pos) {
            const int kl = kl0 + pos, cc = kl / pl.R, fh = kl - cc * pl.R;
            const int ca = CC0 + (cc + U.crot < NCCL ? cc + U.crot : cc + U.crot - NCCL);
            bulk_load(u_smem + (size_t)us * USBYTES + (size_t)pos * UBYTES, src0 + (size_t)(ca * pl.R + fh) * kstride,
                      ub, &u_full[us]);
          }
          if (++us == NUS) { us = 0; uph ^= 1; first = 0; }
        }
      }
      }  // units
    }
    __syncwarp();
  } else {
    // ============================= MMA issuers =============================
    const int iss = warp - ISS_WARP0;  // owns points tl = iss * PPI .. iss * PPI + PPI - 1
    if (rank == 0) {  // the whole warp runs the loop (warp-uniform operands); one lane issues
      constexpr uint32_t idesc = idesc_tf32(PAIR ? 256 : 128, NT);
      // descriptor of U super-slot 0, k-step 0, point 0, hi; other images = + (byte offset >> 4)
      const uint64_t bdesc0 = umma_desc_kmajor_noswizzle(smem_u32(u_smem), BROWS * 16, 128);
      int ss = 0, sph = 0, us = 0, uph = 0;  // super-stage / U super-slot and their round parities
      int sgi = 0, gpass = 0;
      for (int it = unit0; it < NITEMS; it += ustride) {
      const Item I = item_at(it);
      for (int pass = I.pb; pass < I.pe; ++pass, ++gpass) {
        if (gpass > 0) {  // the epilogue has read the previous pass's accumulators
          mbar_wait_tc<PAIR>(d_empty, (gpass - 1) & 1);
          tc_fence_after();
        }
        // wait for super-stage (V and U) readiness; with LA the wait for the NEXT super-stage of
        // the pass is done between this super-stage's two k-steps, while the tensor pipe still
        // holds queued MMAs, so it no longer sits between two super-stages' issue phases
        auto wait_ss = [&](int s_, int sp_, int u_, int up_) {
          if constexpr (PAIR) {  // both CTAs' V (peer arrivals are remote) and both U halves
            mbar_wait_cluster(&st_full[s_], sp_);
            if constexpr (!UW) mbar_wait_cluster(&u_full[u_], up_);
          } else {
            mbar_wait(&st_full[s_], sp_);
            if constexpr (!UW) mbar_wait(&u_full[u_], up_);
          }
        };
        bool ready = false;  // this super-stage already waited for (LA lookahead)
        for (int kl0 = 0; kl0 < NKSP; kl0 += KPS, ++sgi) {
          trace_rec(pl.trace, 29, sgi, iss == 0 && lane32 == 0);
          if (!ready) wait_ss(ss, sph, us, uph);
          ready = false;
          tc_fence_after();
          trace_rec(pl.trace, 16, sgi, iss == 0 && lane32 == 0);
          if (!(ABL(2))) {  // DEBUG timing ablation: skip the MMAs (commits still signal)
#pragma unroll
            for (int pos = 0; pos < KPS; ++pos) {
              const int kl = kl0 + pos;
              // each k-step's V slot is released by its own commit (one k-step of MMA time earlier
              // than a per-super-stage commit for the first k-step); padding k-steps commit too
              uint64_t* sfree = &st_empty[(sgi * KPS + pos) & (NSLOT - 1)];
              if (kl >= NKS) {
                if constexpr (PAIR) mma_commit2_warp(sfree);
                else mma_commit_warp(sfree);
                continue;
              }
              const uint64_t bk = bdesc0 + (uint64_t)((us * USBYTES + pos * UBYTES) >> 4);
              const uint32_t va = tbase + VCOL + (ss * KPS + pos) * GP * 16;
              // product order lo*hi, hi*lo, hi*hi (small terms first), points innermost
              constexpr int PROD0 = P1 ? 2 : 0;  // 1xTF32: the hi*hi product only
#pragma unroll
              for (int prod = PROD0; prod < 3; ++prod) {
#pragma unroll
                for (int pi = 0; pi < PPI; ++pi) {
                  const int tl = iss * PPI + pi;
                  const uint32_t a = va + tl * 16 + (prod == 0 ? 8 : 0);
                  const uint64_t bd = bk + (uint64_t)(((tl * 2 + (prod == 1 ? 1 : 0)) * BROWS * 32) >> 4);
                  const uint32_t acc = (kl > 0 || prod > PROD0) ? 1u : 0u;
                  if constexpr (PAIR) mma2_tf32_ts_warp(tbase + tl * NT, a, bd, idesc, acc);
                  else mma_tf32_ts_warp(tbase + tl * NT, a, bd, idesc, acc);
                }
              }
              if constexpr (PAIR) mma_commit2_warp(sfree);
              else mma_commit_warp(sfree);
              if (LA && pos == 0 && kl0 + KPS < NKSP) {  // lookahead: the next super-stage of this pass
                const int s2 = ss + 1 == NSS ? 0 : ss + 1, sp2 = ss + 1 == NSS ? sph ^ 1 : sph;
                const int u2 = us + 1 == NUS ? 0 : us + 1, up2 = us + 1 == NUS ? uph ^ 1 : uph;
                wait_ss(s2, sp2, u2, up2);
                ready = true;
              }
            }
          } else {  // DEBUG ablation 2 (no MMAs): the slots are still released
#pragma unroll
            for (int pos = 0; pos < KPS; ++pos) {
              uint64_t* sfree = &st_empty[(sgi * KPS + pos) & (NSLOT - 1)];
              if constexpr (PAIR) mma_commit2_warp(sfree);
              else mma_commit_warp(sfree);
            }
          }
          trace_rec(pl.trace, 17, sgi, iss == 0 && lane32 == 0);
          if constexpr (PAIR) mma_commit2_warp(&u_empty[us]);
          else mma_commit_warp(&u_empty[us]);
          trace_rec(pl.trace, 18, sgi, iss == 0 && lane32 == 0);
          if (++ss == NSS) { ss = 0; sph ^= 1; }
          if (++us == NUS) { us = 0; uph ^= 1; }
        }
        if constexpr (PAIR) mma_commit2_warp(d_full);
        else mma_commit_warp(d_full);
      }
      }  // units
    } else if (PAIR && lane32 == 0 && rank == 1 && iss == 0) {
      // ===== pair peer: forward "my U half landed" to the leader's U slot =====
      // (off the critical path: the U ring runs several super-stages ahead; V readiness and the D
      // drain are signalled by the peer's transform warps themselves, remotely)
      const uint32_t lead_ufull = mapa_shared(u_full, 0);
      int us = 0, uph = 0;
      for (int it = unit0; it < NITEMS; it += ustride) {
      const Item I = item_at(it);
      for (int pass = I.pb; pass < I.pe; ++pass) {
        for (int kl0 = 0; kl0 < NKSP; kl0 += KPS) {
          mbar_wait(&u_full[us], uph);
          mbar_arrive_remote(lead_ufull + 8u * (uint32_t)us);
          if (++us == NUS) { us = 0; uph ^= 1; }
        }
      }
      }  // units
    }
    __syncwarp();
   }
  }

  tc_fence_before();
  if constexpr (PAIR) cluster_sync_all();
  else __syncthreads();
  if (warp == ISS_WARP0) {
    tc_fence_after();
    if constexpr (PAIR) tmem_dealloc2(tbase, Cfg::TMEM_COLS);
    else tmem_dealloc(tbase, Cfg::TMEM_COLS);
  }
}

// Persistent grid: one CTA (pair) per SM (pair of SMs), capped by the number of work units;
// I2CW_GRID=<n> overrides the CTA count (experiments).
inline int persistent_ctas(int units, int per) {
  static int nsm = 0;
  static const int forced = [] { const char* e = getenv("I2CW_GRID"); return e ? atoi(e) : 0; }();
  if (nsm == 0) {
    int dev = 0;
    cudaGetDevice(&dev);
    if (cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || nsm <= 0) nsm = 148;
  }
  const int cap = forced > 0 ? forced : nsm;
  const int slots = cap / per > 0 ? cap / per : 1;
  return (units < slots ? units : slots) * per;
}

template <int M, int RW, int NT, bool PAIR, bool VOL = false, bool P1 = false>
static cudaError_t launch_tc_t(const CUtensorMap& xmap, const CUtensorMap& ymap, const Plan& pl, const float* u,
                               cudaStream_t stream) {
  using Cfg = TcCfg<M, RW, NT, PAIR>;
  auto kern = fused_tc_kernel<M, RW, NT, PAIR, VOL, P1>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, pl.smem_bytes);
  if (e != cudaSuccess) return e;
  if constexpr (PAIR) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(persistent_ctas(pl.NITEMS, 2));
    cfg.blockDim = dim3(Cfg::NTHREADS);
    cfg.dynamicSmemBytes = pl.smem_bytes;
    cfg.stream = stream;
    cudaLaunchAttribute attr[2];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = 2;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[1].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 2;
    e = cudaLaunchKernelEx(&cfg, kern, xmap, ymap, pl, u);
    if (e != cudaSuccess) return e;
  } else {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(persistent_ctas(pl.NITEMS, 1));
    cfg.blockDim = dim3(Cfg::NTHREADS);
    cfg.dynamicSmemBytes = pl.smem_bytes;
    cfg.stream = stream;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;  // overlap the prologue
    attr[0].val.programmaticStreamSerializationAllowed = 1;            // with the previous kernel
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    e = cudaLaunchKernelEx(&cfg, kern, xmap, ymap, pl, u);
    if (e != cudaSuccess) return e;
  }
  return cudaGetLastError();
}

}  // namespace i2cw
