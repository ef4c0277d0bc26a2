// C ABI (include/i2cw.h): argument validation, the host planner, TMA tensor-map
// encoding, the stream-ordered workspace and the two launches per call
// (filter transform, fused kernel).
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstring>
#include <atomic>
#include <mutex>
#include <tuple>
#include <vector>

#include "../../include/i2cw.h"
#include "common.cuh"
#include "cook_toom.h"

namespace i2cw {
cudaError_t launch_filter_transform(const float* w, float* u, int C, int K, int R, int S, int is_deconv, int alpha,
                                    int NT, int NB, int NCC, int halves, const double* G, const UTag& tag,
                                    UTag* tag_dst, cudaStream_t stream);
cudaError_t launch_fused_tc(const CUtensorMap& xmap, const CUtensorMap& ymap, const Plan& pl, const float* u,
                            cudaStream_t stream);
struct alignas(64) YMaps { CUtensorMap m[4]; };  // fused_strip.cuh
cudaError_t launch_fused_strip_a8(const CUtensorMap& xmap, const YMaps& ym, const Plan& pl, const float* u,
                                  cudaStream_t stream);
cudaError_t launch_zero_tail(float* y, size_t count, bool wait_first, cudaStream_t stream);
cudaError_t launch_transpose(const float* in, float* out, int B, int rows, int cols, cudaStream_t stream);
cudaError_t launch_ksum(float* y, const float* slices, int nslices, size_t count, size_t stride, cudaStream_t stream);
cudaError_t launch_fused_simt(const Plan& pl, const float* x, const float* u, float* y, cudaStream_t stream);

namespace {


constexpr int kSmemBudget = 225 * 1024;
constexpr int kStripLanes = 32;  // input rows per strip (one TMEM subpartition), fused_strip.cuh

// Longest accumulation in one TMEM accumulator, in k-steps (8 channels x 1 filter row each).
// The tcgen05 fp32 accumulator rounds toward zero once per MMA (3 MMAs per k-step in 3xTF32),
// so the error grows ~linearly with the k-steps summed in TMEM. Measured on B200 with
// all-positive U[1,2] inputs (the worst case, profiles/r02_accuracy_table.md): max |err| / sum|x||w|
// ~1.4e-7 per k-step for alpha = 8 and ~2.8e-7 for alpha = 12 (the larger transform
// amplification). Longer K loops are split into K-chunks whose partial results are added into y
// by the fp32 round-to-nearest TMA reduce-add; the caps below keep that worst case at ~3.6e-5,
// a ~2.8x margin under the 1e-4 bound, for any C.
// i2cw_debug_set_kchunk (test hook) overrides the cap so small parity cases exercise chunking.
int kchunk_default(int alpha) { return alpha <= 8 ? 256 : (alpha <= 12 ? 128 : 64); }
std::atomic<int> g_kchunk_max{0};  // 0: kchunk_default(alpha)
// Cap on concurrent K slices for small grids (run_fused); -1: default (4, or I2CW_KSLICES).
std::atomic<int> g_kslices_max{-1};
constexpr int kMaxKSlices = 8;
int kslices_cap() {
  static const int env = [] { const char* e = getenv("I2CW_KSLICES"); return e ? std::max(1, atoi(e)) : 4; }();
  const int v = g_kslices_max.load();
  return std::min(kMaxKSlices, v > 0 ? v : env);
}

// Per filter width S: F(m, S) and the point set. r = 2..7 follow the paper's
// Gamma_8 choices (Table 2). For r = 8, 9 the paper uses
// Gamma_16; on B200 the tcgen05 fp32 accumulation measured max err/bound 1.1e-4
// with alpha = 16 (alt points) > the 5e-5 acceptance of DESIGN.md reading R7,
// so r = 8, 9 use alpha = 12 (F(5,8), F(4,9); paper point order). Setting
// I2CW_ALPHA16=1 selects alpha = 16 (alt points) for r = 7..9 (ablation only).
struct Choice { int m, alpha, point_set; };
bool alpha16_override() {
  static const bool on = [] { const char* e = getenv("I2CW_ALPHA16"); return e && e[0] == '1'; }();
  return on;
}
// Per (S, C) choice of F(m, S) -- a function of the filter only, so a pre-transformed U fits
// every call with that filter. r = 4..7 follow the paper's Gamma_8 choices (Table 2,
// PAPER.md:3968-3984); r = 8, 9 use alpha = 12 (reading R7). For S = 2 and S = 3 the
// paper's Gamma_4 variants were measured against Gamma_8 on B200
// (profiles/r02_variant_sweep.txt): F(3,2) alpha = 4 beats F(7,2) alpha = 8 by 31% (cfg3-r2), and
// F(2,3) alpha = 4 beats F(6,3) alpha = 8 by ~6% at C >= 256 (cfg5b c256/c512, with CTA pairs)
// but loses 15% on cfg2 and 2.5% at C = 128: one pass (no reduce-add of a second point group)
// against 1.5x the tensor work. I2CW_ALPHA=4 / 8 forces the alpha = 4 / 8 variant for S = 2, 3.
int alpha_env() {
  static const int v = [] { const char* e = getenv("I2CW_ALPHA"); return e ? atoi(e) : 0; }();
  return v;
}
bool strip_enabled() {
  static const bool on = [] { const char* e = getenv("I2CW_STRIP"); return !(e && e[0] == '0'); }();
  return on;
}
bool choose(int S, int C, Choice* c) {
  if (alpha16_override() && S >= 7 && S <= 9) { *c = {17 - S, 16, 1}; return true; }
  if (S == 2 || S == 3) {
    // r = 3 at C >= 256: the strip kernel (alpha = 8 only) with F(6,3) beats the base kernel's best
    // alpha = 4 plan by ~21% on cfg5b c256 / c512 (profiles/r02_strip_sweep.txt)
    const bool a4 = alpha_env() == 4 || (alpha_env() != 8 && (S == 2 || (C >= 256 && !strip_enabled())));
    *c = a4 ? Choice{5 - S, 4, 0} : Choice{9 - S, 8, 0};
    return true;
  }
  switch (S) {
    case 4: *c = {5, 8, 0}; return true;
    case 5: *c = {4, 8, 0}; return true;
    case 6: *c = {3, 8, 0}; return true;
    case 7: *c = {2, 8, 0}; return true;
    case 8: *c = {5, 12, 0}; return true;
    case 9: *c = {4, 12, 0}; return true;
    default: return false;
  }
}

inline int cdiv(int a, int b) { return (a + b - 1) / b; }

// lane -> (image, row, tile) permutation. Every 8 consecutive lanes form one quarter-warp
// shared-memory wavefront for two access patterns:
//  * input reads (LDS.128 of 16-byte columns): bank group (inrow*WBOX + tw*m) mod 8,
//    inrow = img*HBOX + row (images stacked in the staged box);
//  * staged output writes (swizzled 64B rows r = (img*ROWS + row)*TS + tw): (r >> 1) & 3 etc.
// Greedy: fill each group with the tile adding the fewest repeated residues.
// Returns the summed conflict degree (0 = both conflict-free).
int assign_lanes(int NI, int ROWS, int HBOX, int TS, int WBOX, int m, unsigned char* lrow, unsigned short* lin,
                 unsigned char* ltw) {
  struct Tile { int vr, in, t, bin, bout; };
  std::vector<Tile> pool;
  for (int i = 0; i < NI; ++i)
    for (int r = 0; r < ROWS; ++r)
      for (int t = 0; t < TS; ++t) {
        const int vr = i * ROWS + r, in = i * HBOX + r;
        pool.push_back({vr, in, t, (in * WBOX + t * m) % 8, (vr * TS + t) & 7});
      }
  std::fill(lrow, lrow + kMaxLanes, 0xFF);
  std::fill(lin, lin + kMaxLanes, 0);
  std::fill(ltw, ltw + kMaxLanes, 0);
  int lane = 0, cost = 0;
  std::vector<char> used(pool.size(), 0);
  while (lane < (int)pool.size()) {
    int cin[8] = {0}, cout_[8] = {0};
    for (int k = 0; k < 8 && lane < (int)pool.size(); ++k) {
      int best = -1, bestc = 1 << 30;
      for (size_t i = 0; i < pool.size(); ++i) {
        if (used[i]) continue;
        const int c = 2 * cin[pool[i].bin] + cout_[pool[i].bout];
        if (c < bestc) { bestc = c; best = (int)i; }
        if (c == 0) break;
      }
      used[best] = 1;
      cin[pool[best].bin]++;
      cout_[pool[best].bout]++;
      lrow[lane] = (unsigned char)pool[best].vr;
      lin[lane] = (unsigned short)pool[best].in;
      ltw[lane] = (unsigned char)pool[best].t;
      ++lane;
    }
    int mi = 0, mo = 0;
    for (int i = 0; i < 8; ++i) { mi = std::max(mi, cin[i]); mo = std::max(mo, cout_[i]); }
    cost += (mi - 1) + (mo - 1);
  }
  return cost;
}

int num_sms() {
  int dev = 0, nsm = 0;
  if (cudaGetDevice(&dev) != cudaSuccess ||
      cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || nsm <= 0) {
    cudaGetLastError();  // no device (host-only planning): assume a B200
    nsm = 148;
  }
  return nsm;
}

}  // namespace

// Strip kernel (fused_strip.cuh): one input-row transform per 8-channel chunk
// serves all R filter rows through TMEM row shifts. A strip = one tile column of up to
// 33 - R output rows (+ R - 1 halo input rows) in the 32 lanes of a TMEM subpartition; a unit =
// 4 consecutive strips in (n, row block, tw) order. Used for the 2D 3xTF32 alpha = 8 single-CTA
// plans (the U layout of the pair plans differs) when its lane use is not much worse than the
// base block shape's. I2CW_STRIP=0/1 disables / forces it (experiments).
void plan_strip(Plan* plp, int nsm, bool nopair) {
  Plan& pl = *plp;
  static const int env = [] { const char* e = getenv("I2CW_STRIP"); return e ? atoi(e) : -1; }();
  pl.strip = 0;
  if (env == 0 || pl.vol || pl.prec || pl.alpha != 8 || pl.NT != 64 || pl.R > 24) return;
  // CTA pairs (M = 256, each SM streams half of U): I2CW_STRIP_PAIR=0/1 (default on)
  static const int pair_env = [] { const char* e = getenv("I2CW_STRIP_PAIR"); return e ? atoi(e) : 1; }();
  const int rbmax = 33 - pl.R;
  const int pb = cdiv(pl.P, rbmax), rb = cdiv(pl.P, pb);
  const long long nstrip = (long long)pl.N * pb * pl.T_r;
  if (nstrip > (1 << 30)) return;
  const int sgroups = (int)cdiv((int)nstrip, 4);
  // lanes doing useful output work: strip plan vs the base plan's tile blocks
  const double useful = (double)pl.N * pl.P * pl.T_r;
  const double util_strip = useful / ((double)sgroups * kMaxLanes);
  const double util_base = useful / ((double)pl.tile_blocks * kMaxLanes);
  // measured on B200 (profiles/r02_strip_sweep.txt): the strip kernel wins from a lane-use ratio
  // of 0.8 (cfg5a +2.5%, cfg2 +10%, cfg5b +14..21%) and loses below 0.7 (P = 32 images: cfg3)
  if (env != 1 && util_strip < 0.75 * util_base) return;
  const int spair = pair_env != 0 && !nopair && sgroups >= 2 ? 1 : 0;
  const int kUB = 4 * 2 * (spair ? 32 : 64) * 32;  // this CTA's U k-step (alpha = 8, GP = 4)
  constexpr int kStage = 4 * 9 * 32 * 32;           // 4 strip boxes (alpha = 8)
  const int osb = 4 * 2048, ostride = osb;  // 4 strips x 32 rows x 16 channels per output buffer
  // U ring: one k-step per slot. One slot per chunk (KU = R: one barrier wait and commit per
  // chunk instead of R) fits only 2 slots and measured 4-5% slower on cfg2 / c128 (the U stream's
  // latency shows through one chunk of lookahead); I2CW_STRIP_KU=2 selects it (experiments).
  // Candidates: (U slots, input stages, output buffers >= 2).
  static int kSD[][3] = {{6, 2, 3}, {5, 2, 3}, {5, 2, 2}, {4, 2, 2}, {3, 2, 2}, {2, 2, 2}};
  static int kSDc[][3] = {{3, 2, 3}, {2, 2, 3}, {3, 2, 2}, {2, 2, 2}};
  static const bool sd_env = [] {  // I2CW_STRIP_DEPTHS=u,i,o (experiments): try these first
    const char* e = getenv("I2CW_STRIP_DEPTHS");
    int a, b, c;
    if (e && sscanf(e, "%d,%d,%d", &a, &b, &c) == 3 && b >= 1 && c >= 2) {
      kSD[0][0] = a; kSD[0][1] = b; kSD[0][2] = c;
      kSDc[0][0] = a; kSDc[0][1] = b; kSDc[0][2] = c;
    }
    return e != nullptr;
  }();
  (void)sd_env;
  static const int ku_env = [] { const char* e = getenv("I2CW_STRIP_KU"); return e ? atoi(e) : 0; }();
  int sel = -1, smem = 0, ku = 1;
  for (int pass = 0; pass < 2 && sel < 0; ++pass) {
    ku = pass == 0 ? pl.R : 1;
    if (pass == 0 && (ku_env < 2 || pl.R == 1)) continue;
    const int(*cand)[3] = pass == 0 ? kSDc : kSD;
    const int ncand = pass == 0 ? 4 : 6;
    for (int d = 0; d < ncand; ++d) {
      const int bar_bytes = 8 * (4 + cand[d][1] + 10 + 2 * cand[d][0]) + 32 + 4 * 4 * 16;  // + slot, op table
      smem = cand[d][0] * ku * kUB + cand[d][1] * kStage + 4 * cand[d][2] * ostride + bar_bytes;
      if (smem <= kSmemBudget) { sel = d; break; }
    }
  }
  if (sel < 0) return;
  const int(*kSel)[3] = ku > 1 ? kSDc : kSD;
  pl.strip = 1;
  pl.pair = spair;
  pl.NSTRIP = (int)nstrip;
  pl.ROWS = rb;
  pl.PB = pb;
  pl.TS = 4;
  pl.NI = 1;
  pl.SEGS = 1;
  pl.HBOX = kStripLanes;
  pl.WBOX = pl.alpha;
  pl.tile_blocks = sgroups;
  pl.KU = ku;
  pl.NUS = kSel[sel][0];
  pl.NIS = kSel[sel][1];
  pl.NOB = kSel[sel][2];
  pl.OSB = osb;
  pl.OSTRIDE = ostride;
  pl.BOXB = kStage;
  pl.PLANE = kStage / 2;
  pl.smem_bytes = smem;
  std::fill(pl.lane_row, pl.lane_row + kMaxLanes, 0);
  std::fill(pl.lane_in, pl.lane_in + kMaxLanes, 0);
  std::fill(pl.lane_tw, pl.lane_tw + kMaxLanes, 0);
  const int units = (spair ? cdiv(sgroups, 2) : sgroups) * pl.NB;
  const int G = spair ? std::max(1, nsm / 2) : nsm;
  const int tail = units % G;
  const char* st = getenv("I2CW_SPLIT_TAIL");
  static const bool allsplit = [] { const char* e = getenv("I2CW_STRIP_ALLSPLIT"); return e && e[0] == '1'; }();
  if (pl.NPASS == 2 && allsplit) {  // experiments: every unit as two one-pass items
    pl.NFULL = 0;
    pl.NITEMS = 2 * units;
  } else if (pl.NPASS == 2 && !(st && st[0] == '0') && tail > 0 && 2 * tail <= G) {
    pl.NFULL = units - tail;
    pl.NITEMS = pl.NFULL + 2 * tail;
  } else {
    pl.NFULL = pl.NITEMS = units;
  }
  const int item_ksteps = pl.NKS * (pl.NFULL > 0 ? pl.NPASS : 1);
  pl.KSL = 1;
  const int ctas = spair ? 2 * pl.NITEMS : pl.NITEMS;
  if (pl.NKC == 1 && pl.NCC >= 2 && 2 * ctas <= nsm)
    pl.KSL = std::max(1, std::min({kslices_cap(), pl.NCC, nsm / std::max(1, ctas), item_ksteps / 64}));
  if (pl.KSL > 1) pl.KSL = cdiv(pl.NCC, cdiv(pl.NCC, pl.KSL));
}

// Build the launch plan. Returns I2CW_OK or an error code.
// vol = 1: 3D convolution (D, T, pad_d); 2D calls pass D = T = 1, pad_d = 0, vol = 0.
int make_plan_uncached(int N, int D, int H, int W, int C, int K, int T, int R, int S, int pad_d, int pad_h, int pad_w,
                       int is_deconv, int vol, int prec, Plan* out) {
  Plan pl;
  std::memset(&pl, 0, sizeof(pl));
  if (N <= 0 || D <= 0 || H <= 0 || W <= 0 || C <= 0 || K <= 0 || T <= 0 || R <= 0 || S <= 0 || pad_d < 0 ||
      pad_h < 0 || pad_w < 0)
    return I2CW_EINVAL;
  if (!vol && (D != 1 || T != 1 || pad_d != 0)) return I2CW_EINVAL;
  const int nostrip = prec & 2, strip_nopair = prec & 4;
  prec &= 1;
  if (prec && vol) return I2CW_EUNSUPPORTED;  // 1xTF32 kernels: 2D only
  Choice ch;
  if (!choose(S, C, &ch)) return I2CW_EUNSUPPORTED;
  // the 3D and 1xTF32 kernels are instantiated for the default alpha = 8 / 12 families only
  if ((vol || prec) && ch.alpha != 8 && ch.alpha != 12) ch = Choice{S <= 7 ? 9 - S : 13 - S, S <= 7 ? 8 : 12, 0};
  if (C % 4 != 0 || K % 4 != 0) return I2CW_EUNSUPPORTED;
  pl.N = N; pl.H = H; pl.W = W; pl.C = C; pl.K = K; pl.R = R; pl.S = S;
  pl.vol = vol; pl.D = D; pl.T = T; pl.prec = prec;
  pl.is_deconv = is_deconv;
  if (is_deconv) {  // deconv(x, w, pad) == conv(x, rot180(w)^T, R-1-pad) (3D: rotate all three taps)
    pl.pad_d = T - 1 - pad_d;
    pl.pad_h = R - 1 - pad_h;
    pl.pad_w = S - 1 - pad_w;
  } else {
    pl.pad_d = pad_d;
    pl.pad_h = pad_h;
    pl.pad_w = pad_w;
  }
  pl.OD = D + 2 * pl.pad_d - T + 1;
  pl.P = H + 2 * pl.pad_h - R + 1;
  pl.Q = W + 2 * pl.pad_w - S + 1;
  if (pl.OD < 1 || pl.P < 1 || pl.Q < 1) return I2CW_EINVAL;
  pl.m = ch.m;
  pl.alpha = ch.alpha;
  // Output channels per CTA (UMMA N): 64 (4 points per pass, 4 V slots of 64 columns) for
  // K > 32, else 32. NT = 128 (2 points per pass, 8 V slots of 32 columns: a V ring twice as
  // long in MMA time) is implemented and parity-tested but measured 10-60% slower on every
  // K >= 128 config (twice the passes: 4 y writes per output, shallower U ring;
  // profiles/r01f_nt128.txt), so it is opt-in: I2CW_NT=<32|64|128> overrides (experiments).
  static const int nt_env = [] { const char* e = getenv("I2CW_NT"); return e ? atoi(e) : 0; }();
  pl.NT = K > 32 ? 64 : 32;
  if (nt_env == 32 || nt_env == 64 || (nt_env == 128 && ch.alpha >= 8 && ch.alpha <= 12)) pl.NT = nt_env;
  pl.GP = gp_for(pl.alpha, pl.NT);
  pl.NPASS = pl.alpha / pl.GP;
  pl.NB = cdiv(K, pl.NT);
  pl.NCC = cdiv(C, 8) * T;  // 3D: virtual chunks (channel chunk, depth tap)
  pl.NKS = pl.NCC * R;
  {
    const int kset = g_kchunk_max.load();
    const int kmax = std::max(R, kset > 0 ? kset : kchunk_default(pl.alpha));
    const int cpc_max = std::max(1, kmax / R);
    pl.NKC = cdiv(pl.NCC, cpc_max);
    pl.CPC = cdiv(pl.NCC, pl.NKC);  // balanced chunks
    pl.CC0 = 0;
    pl.CC1 = pl.NCC;
    pl.ACCUM = 0;
  }
  pl.T_r = cdiv(pl.Q, pl.m);
  // WBOX <= 256 (TMA box limit), leave 7 columns of slack for the bank search
  const int ts_max = std::min(kMaxLanes, (256 - 7 - (S - 1)) / pl.m);
  if (ts_max < 1) return I2CW_EUNSUPPORTED;
  pl.TS = std::min(pl.T_r, ts_max);
  pl.SEGS = cdiv(pl.T_r, pl.TS);
  // CTA pairs (clusters of 2, tcgen05.mma.cta_group::2 with M = 256, each CTA stages half of
  // U): halves the per-SM filter stream and B-operand reads but adds a cross-CTA relay per
  // super-stage. Measured on B200 (profiles/r01d_pair_sweep.txt, profiles/r01i_pair_rule.txt):
  // +5..12% at NKS = C/8 * R >= 128 (r8, r9, cfg4 r5/r7, c512) or >= 4 output-channel blocks
  // (c256 +11%), -2..-18% otherwise (cfg2, r2-r7, c64, c128). I2CW_PAIR=1/0 forces it.
  static const int pair_env = [] { const char* e = getenv("I2CW_PAIR"); return e ? (e[0] == '1' ? 1 : 0) : -1; }();
  pl.pair = pair_env >= 0 ? pair_env : ((pl.NKS >= 128 || pl.NB >= 4) ? 1 : 0);
  if (vol || prec) pl.pair = 0;  // 3D and 1xTF32 kernels: single-CTA instantiations only
  // DEBUG timing ablation (never set in production; results are wrong when non-zero)
  static const int ablate = [] { const char* e = getenv("I2CW_ABLATE"); return e ? atoi(e) : 0; }();
  pl.ablate = ablate;
  const int ubytes = pl.GP * 2 * pl.NT * 32 / (pl.pair ? 2 : 1);
  const int NS = ns_for(pl.alpha, pl.NT);
  const int kps = kps_for(pl.alpha, pl.NT);  // k-steps per U super-slot
  const int wmin = pl.TS * pl.m + S - 1;
  // ring depths, most preferred first: U slots hide the L2 latency of the filter
  // stream (~1-2K cycles), input stages that of the row boxes, 2 output buffers
  // overlap the TMA store of one output column with the next column's math.
  static int kDepths[][3] = {{8, 3, 3}, {8, 3, 2}, {6, 3, 3}, {6, 3, 2}, {6, 2, 2}, {4, 3, 2}, {4, 2, 2},
                             {3, 2, 2}, {2, 2, 2}};
  constexpr int kNumDepths = sizeof(kDepths) / sizeof(kDepths[0]);
  // I2CW_DEPTHS=u,i,o (experiments only): try this (U k-steps, input stages, output buffers)
  // first
  static const bool depth_env = [] {
    const char* e = getenv("I2CW_DEPTHS");
    int a, b, c;
    if (e && sscanf(e, "%d,%d,%d", &a, &b, &c) == 3) { kDepths[0][0] = a; kDepths[0][1] = b; kDepths[0][2] = c; }
    return e != nullptr;
  }();
  (void)depth_env;
  // Tile blocks = NI images x ROWS output rows x TS tiles (<= 128 UMMA lanes). Candidates are
  // ranked by (1) persistent rounds ceil(units / #CTAs) -- the makespan, (2) ring depth that
  // fits in shared memory, (3) staged input rows per unit NI * (ROWS + R - 1), (4) units.
  // Small images pack several per block (28x28 with m = 6: 5 tiles per row; one image per
  // block would use 70 of 128 lanes, NI = 6 x 4 rows uses 120).
  const int nsm = num_sms();
  // Split tail (Plan::NFULL / NITEMS, applied after the block shape is chosen): with 2 passes
  // (single CTAs or CTA pairs), the last T = units mod G units run as 2T one-pass items when 2T <= G, so
  // they cost half a unit time (cfg2 +4%, r7 +10%). Ranking block shapes by half-unit rounds
  // instead picked more images per block and measured slower (r2 -24%, c128 -7%), so the
  // ranking keeps whole rounds. I2CW_SPLIT_TAIL=0 disables the split.
  const bool split_ok = pl.NPASS == 2 && [] {
    const char* e = getenv("I2CW_SPLIT_TAIL");
    return !(e && e[0] == '0');
  }();
  const int cpw = pl.NT / nwg_for(pl.NT);  // epilogue channels per warpgroup (staging row = cpw * 4 B)
  struct Cand { int rounds, depth, inrows, units, NI, rows, pb; };
  bool have = false;
  Cand best{};
  // I2CW_NI=<n> (tests only) forces n images per block (even n > N: a ragged last group),
  // so small parity cases exercise multi-image blocks
  static const int force_ni = [] { const char* e = getenv("I2CW_NI"); return e ? atoi(e) : 0; }();
  const int ni_lo = force_ni > 0 ? std::min(force_ni, kMaxLanes / pl.TS) : 1;
  // 2D: NI consecutive images per block; 3D: NI consecutive output depths of one image
  const int stack_extent = vol ? pl.OD : N;
  const int ni_max = force_ni > 0 ? ni_lo : std::min(stack_extent, kMaxLanes / pl.TS);
  for (int ni = ni_lo; ni <= ni_max; ++ni) {
    int rmax = std::min({kMaxLanes / (ni * pl.TS), pl.P, 256 - (R - 1)});
    if (pl.SEGS > 1) rmax = std::min(rmax, 1);
    int last_bal = -1;
    for (int r = rmax; r >= 1; --r) {
      const int pb = cdiv(pl.P, r), rb = cdiv(pl.P, pb);  // balanced rows over the row blocks
      if (rb == last_bal) continue;
      last_bal = rb;
      const int hbox = rb + R - 1;
      const int plane = (ni * hbox * (wmin + 7) * 32 + 1023) / 1024 * 512;  // half stage, upper bound (WBOX <= wmin + 7)
      const int ostride = (ni * rb * pl.TS * cpw * 4 + 1023) / 1024 * 1024;
      int depth = -1;
      for (int d = 0; d < kNumDepths; ++d) {
        const int nus = std::max(kDepths[d][0] / kps, 2);
        const int bar_bytes = 8 * (2 * kDepths[d][1] + NS + 2 * (NS / kps) + 2 + 2 * nus) + 16;
        const int sm = nus * kps * ubytes + kDepths[d][1] * 2 * plane + nwg_for(pl.NT) * kDepths[d][2] * ostride +
                       bar_bytes;
        if (sm <= kSmemBudget) { depth = d; break; }
      }
      if (depth < 0 || ni * hbox > 256) continue;
      const int blocks = (vol ? N * cdiv(pl.OD, ni) : cdiv(N, ni)) * pb * pl.SEGS;
      const int units = (pl.pair ? cdiv(blocks, 2) : blocks) * pl.NB;
      const int G = pl.pair ? std::max(1, nsm / 2) : nsm;
      const Cand c{cdiv(units, G), depth, ni * hbox, units, ni, rb, pb};
      auto key = [](const Cand& x) { return std::make_tuple(x.rounds, x.depth, x.inrows, x.units, x.NI); };
      if (!have || key(c) < key(best)) { best = c; have = true; }
    }
  }
  if (!have) return I2CW_EUNSUPPORTED;
  pl.NI = best.NI;
  pl.ROWS = best.rows;
  pl.PB = best.pb;
  pl.HBOX = pl.ROWS + R - 1;
  {
    int bc = -1, bestw = wmin;
    for (int wb = wmin; wb <= std::min(256, wmin + 7); ++wb) {
      unsigned char lr[kMaxLanes], lt[kMaxLanes];
      unsigned short li[kMaxLanes];
      const int c = assign_lanes(pl.NI, pl.ROWS, pl.HBOX, pl.TS, wb, pl.m, lr, li, lt);
      if (bc < 0 || c < bc) { bc = c; bestw = wb; }
    }
    pl.WBOX = bestw;
  }
  pl.BOXB = pl.NI * pl.HBOX * pl.WBOX * 32;  // one 8-channel box per input stage
  pl.PLANE = (pl.BOXB + 1023) / 1024 * 512;   // half a stage; stages stay 1024-aligned (TMA swizzle)
  // Output staging: one output column i of every tile for one warpgroup's 16 channels (one
  // 64-byte swizzled row per tile), stored by TMA with Q stride m.
  pl.OSB = pl.NI * pl.ROWS * pl.TS * cpw * 4;
  pl.OSTRIDE = (pl.OSB + 1023) / 1024 * 1024;
  pl.NUS = std::max(kDepths[best.depth][0] / kps, 2);  // U super-slots
  pl.NIS = kDepths[best.depth][1];
  pl.NOB = kDepths[best.depth][2];
  const int bar_bytes = 8 * (2 * pl.NIS + NS + 2 * (NS / kps) + 2 + 2 * pl.NUS) + 16;
  pl.smem_bytes = pl.NUS * kps * ubytes + pl.NIS * 2 * pl.PLANE + nwg_for(pl.NT) * pl.NOB * pl.OSTRIDE + bar_bytes;
  if (pl.smem_bytes > kSmemBudget) return I2CW_EUNSUPPORTED;
  assign_lanes(pl.NI, pl.ROWS, pl.HBOX, pl.TS, pl.WBOX, pl.m, pl.lane_row, pl.lane_in, pl.lane_tw);
  pl.DB = vol ? cdiv(pl.OD, pl.NI) : 1;
  pl.tile_blocks = (vol ? N * pl.DB : cdiv(N, pl.NI)) * pl.PB * pl.SEGS;
  {
    const int units = (pl.pair ? cdiv(pl.tile_blocks, 2) : pl.tile_blocks) * pl.NB;
    const int G = pl.pair ? std::max(1, nsm / 2) : nsm;
    const int tail = units % G;
    if (split_ok && tail > 0 && 2 * tail <= G) {
      pl.NFULL = units - tail;
      pl.NITEMS = pl.NFULL + 2 * tail;
    } else {
      pl.NFULL = pl.NITEMS = units;
    }
  }
  // K slices (run_fused): when the work items fill at most half of the SMs and the K loop is
  // one chunk, up to kslices_cap() slices of the channel chunks run concurrently, each item
  // keeping >= 64 k-step passes (shorter slices save less device time than the extra launches
  // cost on the host: measured on B200, profiles/r02_kslice_ab.txt)
  {
    const int ctas = pl.pair ? 2 * pl.NITEMS : pl.NITEMS;
    const int item_ksteps = pl.NKS * (pl.NFULL > 0 ? pl.NPASS : 1);
    pl.KSL = 1;
    if (pl.NKC == 1 && pl.NCC >= 2 && 2 * ctas <= nsm)
      pl.KSL = std::max(1, std::min({kslices_cap(), pl.NCC, nsm / std::max(1, ctas), item_ksteps / 64}));
    if (pl.KSL > 1) pl.KSL = cdiv(pl.NCC, cdiv(pl.NCC, pl.KSL));  // no empty slice
  }
  // prec bit 1: base plan only (the SIMT stepping stone, filter-only plans); bit 2: no CTA pairs
  // in the strip plan (a pre-transformed U in the single-CTA layout)
  if (!nostrip) plan_strip(&pl, nsm, strip_nopair != 0);
  *out = pl;
  return I2CW_OK;
}

// Plans are pure functions of the call's dimensions (and the device's SM count): memoised,
// so repeated calls skip the block-shape search and the lane permutation.
int make_plan3(int N, int D, int H, int W, int C, int K, int T, int R, int S, int pad_d, int pad_h, int pad_w,
               int is_deconv, int vol, Plan* out, int prec = 0) {
  struct Key { int v[18]; };
  static std::mutex mu;
  static std::vector<std::pair<Key, Plan>> memo;
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) { cudaGetLastError(); dev = -1; }
  const Key k{{N, D, H, W, C, K, T, R, S, pad_d, pad_h, pad_w, is_deconv, vol, prec, dev, g_kchunk_max.load(), kslices_cap()}};
  {
    std::lock_guard<std::mutex> lk(mu);
    for (auto& e : memo)
      if (std::memcmp(e.first.v, k.v, sizeof(k.v)) == 0) { *out = e.second; return I2CW_OK; }
  }
  Plan pl;
  const int rc = make_plan_uncached(N, D, H, W, C, K, T, R, S, pad_d, pad_h, pad_w, is_deconv, vol, prec, &pl);
  if (rc != I2CW_OK) return rc;
  std::lock_guard<std::mutex> lk(mu);
  if (memo.size() >= 256) memo.erase(memo.begin());
  memo.push_back({k, pl});
  *out = pl;
  return I2CW_OK;
}

int make_plan(int N, int H, int W, int C, int K, int R, int S, int pad_h, int pad_w, int is_deconv, Plan* out) {
  return make_plan3(N, 1, H, W, C, K, 1, R, S, 0, pad_h, pad_w, is_deconv, 0, out);
}

namespace {

typedef CUresult (*PFN_encodeTiled_t)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                      const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                      CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

PFN_encodeTiled_t get_encode() {
  static PFN_encodeTiled_t fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_encodeTiled_t>(p);
  });
  return fn;
}

// x: [N][H][W][C] fp32; box = 8 channels (32 B, 32B-swizzled) x WBOX columns x HBOX rows x NI images
int encode_x_map(const Plan& pl, const float* x, CUtensorMap* map) {
  PFN_encodeTiled_t enc = get_encode();
  if (!enc) return I2CW_ECUDA;
  if (pl.vol) {  // [N][D][H][W][C]: box = 8 channels x WBOX x HBOX x NI depths x 1 image
    cuuint64_t dims[5] = {(cuuint64_t)pl.C, (cuuint64_t)pl.W, (cuuint64_t)pl.H, (cuuint64_t)pl.D, (cuuint64_t)pl.N};
    const cuuint64_t sw = (cuuint64_t)pl.C * 4, sh = sw * pl.W, sd = sh * pl.H, sn = sd * pl.D;
    cuuint64_t strides[4] = {sw, sh, sd, sn};
    cuuint32_t box[5] = {8, (cuuint32_t)pl.WBOX, (cuuint32_t)pl.HBOX, (cuuint32_t)pl.NI, 1};
    cuuint32_t es[5] = {1, 1, 1, 1, 1};
    CUresult r = enc(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 5, const_cast<float*>(x), dims, strides, box, es,
                     CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_32B, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
                     CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS ? I2CW_OK : I2CW_EUNSUPPORTED;
  }
  cuuint64_t dims[4] = {(cuuint64_t)pl.C, (cuuint64_t)pl.W, (cuuint64_t)pl.H, (cuuint64_t)pl.N};
  cuuint64_t strides[3] = {(cuuint64_t)pl.C * 4, (cuuint64_t)pl.W * pl.C * 4, (cuuint64_t)pl.H * pl.W * pl.C * 4};
  cuuint32_t box[4] = {8, (cuuint32_t)pl.WBOX, (cuuint32_t)pl.HBOX, (cuuint32_t)pl.NI};
  cuuint32_t es[4] = {1, 1, 1, 1};
  CUresult r = enc(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, const_cast<float*>(x), dims, strides, box, es,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_32B, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS ? I2CW_OK : I2CW_EUNSUPPORTED;
}

// strip kernel: x box = 8 channels x (alpha + 1) columns x 32 rows, 32B swizzle: the 288-byte
// row stride puts the 8 rows a quarter-warp reads in 8 distinct 16-byte bank groups
// (tools/tma_view_test.cu checks the layout; a (C, H, W, N) view with non-monotonic strides
// encodes but faults in the TMA unit)
int encode_x_map_strip(const Plan& pl, const float* x, CUtensorMap* map) {
  PFN_encodeTiled_t enc = get_encode();
  if (!enc) return I2CW_ECUDA;
  cuuint64_t dims[4] = {(cuuint64_t)pl.C, (cuuint64_t)pl.W, (cuuint64_t)pl.H, (cuuint64_t)pl.N};
  cuuint64_t strides[3] = {(cuuint64_t)pl.C * 4, (cuuint64_t)pl.W * pl.C * 4, (cuuint64_t)pl.H * pl.W * pl.C * 4};
  cuuint32_t box[4] = {8, (cuuint32_t)(pl.alpha + 1), (cuuint32_t)kStripLanes, 1};
  cuuint32_t es[4] = {1, 1, 1, 1};
  CUresult r = enc(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, const_cast<float*>(x), dims, strides, box, es,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_32B, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS ? I2CW_OK : I2CW_EUNSUPPORTED;
}

// strip kernel: y store box for a run of L strips = 16 channels x L tiles (element stride m) x ROWS
// rows x 1 image; swizzle 64B for L = 3, else 128B (the staging writes of a warp -- 8 rows of one
// tile -- are then conflict-free or 2-way, fused_strip.cuh). A box that starts at a negative
// column faults (tools/tma_view_test.cu), hence one map per run length.
int encode_y_map_strip(const Plan& pl, float* y, int L, CUtensorMap* map) {
  PFN_encodeTiled_t enc = get_encode();
  if (!enc) return I2CW_ECUDA;
  cuuint64_t dims[4] = {(cuuint64_t)pl.K, (cuuint64_t)pl.Q, (cuuint64_t)pl.P, (cuuint64_t)pl.N};
  cuuint64_t strides[3] = {(cuuint64_t)pl.K * 4, (cuuint64_t)pl.Q * pl.K * 4, (cuuint64_t)pl.P * pl.Q * pl.K * 4};
  // L = 2 is the warp-pair store box of the strip kernel (I2CW_STRIP_PAIRSTORE): 32 channels x 1
  // column x ROWS rows, 128B swizzle (128-byte staging rows); L = 1: the per-warp 16-channel box
  const bool pairbox = L == 2;
  cuuint32_t box[4] = {pairbox ? 32u : 16u, pairbox ? 1u : (cuuint32_t)(L * pl.m), (cuuint32_t)pl.ROWS, 1};
  cuuint32_t es[4] = {1, pairbox ? 1u : (cuuint32_t)pl.m, 1, 1};
  CUresult r = enc(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, y, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   pairbox ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_64B, CU_TENSOR_MAP_L2_PROMOTION_NONE,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS ? I2CW_OK : I2CW_EUNSUPPORTED;
}

// y: [N][P][Q][K] fp32; store box = NT/4 channels x (TS*m columns walked with element
// stride m, i.e. TS positions q0 + i) x ROWS rows x NI images, 64B / 128B swizzled.
// Elements outside [0,K) x [0,Q) x [0,P) are clipped by the TMA unit (the in-kernel boundary).
int encode_y_map(const Plan& pl, float* y, CUtensorMap* map) {
  PFN_encodeTiled_t enc = get_encode();
  if (!enc) return I2CW_ECUDA;
  if (pl.vol) {  // [N][OD][P][Q][K]: box = cpw channels x TS positions (stride m) x ROWS x NI depths x 1
    const int cpw = pl.NT / nwg_for(pl.NT);
    cuuint64_t dims[5] = {(cuuint64_t)pl.K, (cuuint64_t)pl.Q, (cuuint64_t)pl.P, (cuuint64_t)pl.OD, (cuuint64_t)pl.N};
    const cuuint64_t sq = (cuuint64_t)pl.K * 4, sp = sq * pl.Q, sd = sp * pl.P, sn = sd * pl.OD;
    cuuint64_t strides[4] = {sq, sp, sd, sn};
    cuuint32_t box[5] = {(cuuint32_t)cpw, (cuuint32_t)(pl.TS * pl.m), (cuuint32_t)pl.ROWS, (cuuint32_t)pl.NI, 1};
    cuuint32_t es[5] = {1, (cuuint32_t)pl.m, 1, 1, 1};
    CUresult r = enc(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 5, y, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                     (cpw == 16 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_128B),
                     CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS ? I2CW_OK : I2CW_EUNSUPPORTED;
  }
  cuuint64_t dims[4] = {(cuuint64_t)pl.K, (cuuint64_t)pl.Q, (cuuint64_t)pl.P, (cuuint64_t)pl.N};
  cuuint64_t strides[3] = {(cuuint64_t)pl.K * 4, (cuuint64_t)pl.Q * pl.K * 4, (cuuint64_t)pl.P * pl.Q * pl.K * 4};
  const int cpw = pl.NT / nwg_for(pl.NT);  // one warpgroup's channels: 64 B or 128 B rows
  cuuint32_t box[4] = {(cuuint32_t)cpw, (cuuint32_t)(pl.TS * pl.m), (cuuint32_t)pl.ROWS, (cuuint32_t)pl.NI};
  cuuint32_t es[4] = {1, (cuuint32_t)pl.m, 1, 1};
  if (I2CW_ABLATION && (pl.ablate & 128)) {  // DEBUG timing ablation: contiguous (unstrided) boxes, results wrong
    box[1] = (cuuint32_t)pl.TS;
    es[1] = 1;
  }
  CUresult r = enc(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, y, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   (cpw == 16 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_128B),
                   CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS ? I2CW_OK : I2CW_EUNSUPPORTED;
}

void ensure_pool(int dev) {
  static std::mutex mu;
  static bool done[64] = {false};
  std::lock_guard<std::mutex> lk(mu);
  if (dev < 0 || dev >= 64 || done[dev]) return;
  cudaMemPool_t pool;
  if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) {
    uint64_t thr = UINT64_MAX;
    cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
  }
  done[dev] = true;
}

// Our statically linked runtime keeps its own "current device": follow the
// device that owns the caller's pointer (multi-GPU ranks use device != 0).
int bind_device_of(const void* p) {
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) { cudaGetLastError(); return I2CW_EINVAL; }
  if (a.type != cudaMemoryTypeDevice && a.type != cudaMemoryTypeManaged) return I2CW_EINVAL;
  int cur = -1;
  cudaGetDevice(&cur);
  if (cur != a.device && cudaSetDevice(a.device) != cudaSuccess) return I2CW_ECUDA;
  ensure_pool(a.device);
  return I2CW_OK;
}

// Host-side copy of the tags written by i2cw_filter_transform, so the
// pre-transformed calls can validate u without a device-to-host sync.
std::mutex g_reg_mu;
std::vector<std::pair<const void*, UTag>> g_registry;
void registry_put(const void* u, const UTag& t) {
  std::lock_guard<std::mutex> lk(g_reg_mu);
  for (auto& e : g_registry)
    if (e.first == u) { e.second = t; return; }
  if (g_registry.size() >= 4096) g_registry.erase(g_registry.begin());
  g_registry.push_back({u, t});
}
bool registry_lookup(const void* u, UTag* t) {
  std::lock_guard<std::mutex> lk(g_reg_mu);
  for (auto& e : g_registry)
    if (e.first == u) { *t = e.second; return true; }
  return false;
}

inline bool aligned16(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }

// exact G of F(m, S), rows permuted to the internal point order, as doubles
void g_internal(const Plan& pl, int point_set, std::vector<double>* G) {
  Transforms T = cook_toom(pl.m, pl.S, point_set);
  G->assign((size_t)pl.alpha * pl.S, 0.0);
  for (int idx = 0; idx < pl.alpha; ++idx)
    for (int s = 0; s < pl.S; ++s) (*G)[(size_t)idx * pl.S + s] = T.G[(size_t)point_of(idx, pl.alpha) * pl.S + s].to_double();
}

// the 256-byte header in front of U: what the filter was transformed for
UTag make_tag(const Plan& pl, int is_deconv) {
  UTag t;
  std::memset(&t, 0, sizeof(t));
  t.magic = kUMagic; t.alpha = pl.alpha; t.m = pl.m; t.is_deconv = is_deconv;
  t.C = pl.C; t.K = pl.K; t.R = pl.R; t.S = pl.S; t.NT = pl.NT; t.NB = pl.NB; t.NCC = pl.NCC;
  t.halves = pl.pair ? 2 : 1;
  t.T = pl.T;
  return t;
}

size_t u_data_bytes(const Plan& pl) { return (size_t)pl.NB * pl.NKS * pl.alpha * 2 * pl.NT * 8 * 4; }

// exact G tables are generated once per (m, S, point set) and kept (host memo). Returned BY
// VALUE (at most 16 x 9 doubles): a reference into the memo could be invalidated by another
// thread's insertion while the caller still reads it.
std::vector<double> g_cached(const Plan& pl, int point_set) {
  static std::mutex mu;
  static std::vector<std::pair<int, std::vector<double>>> memo;
  const int key = (pl.m * 16 + pl.S) * 2 + point_set;
  std::lock_guard<std::mutex> lk(mu);
  for (auto& e : memo)
    if (e.first == key) return e.second;
  std::vector<double> G;
  g_internal(pl, point_set, &G);
  memo.push_back({key, G});
  return G;
}

int transform_into(const Plan& pl, int is_deconv, const float* w, void* u, cudaStream_t stream) {
  const std::vector<double> G = g_cached(pl, pl.alpha == 16 ? 1 : 0);  // alt alpha = 16 points (R7)
  const UTag tag = make_tag(pl, is_deconv);
  static_assert(sizeof(UTag) <= kUTagBytes, "tag");
  float* ud = reinterpret_cast<float*>(static_cast<uint8_t*>(u) + kUTagBytes);
  // 3D: the [K][T][R][S][C] filter is the 2D filter [K][T*R][S][C] (and the deconv rotation of the
  // combined T*R axis is the rotation of both), with ceil(C/8) channel chunks
  if (launch_filter_transform(w, ud, pl.C, pl.K, pl.R * pl.T, pl.S, is_deconv, pl.alpha, pl.NT, pl.NB, pl.NCC / pl.T,
                              pl.pair ? 2 : 1, G.data(), tag, static_cast<UTag*>(u), stream) != cudaSuccess)
    return I2CW_ECUDA;
  return I2CW_OK;
}

// after_own_ft: the previous kernel in the stream is this library's filter transform (which
// never touches y), so the zeroing kernel may overlap it through programmatic dependent launch;
// otherwise (pre-transformed path: the caller's last kernel is unknown) the zeroing kernel
// waits for the previous grid before its first store.
// A failed CUDA call on the launch path: clears the error, logs it with I2CW_VERBOSE=1.
int cuda_fail(const char* what) {
  static const bool verbose = [] { const char* e = getenv("I2CW_VERBOSE"); return e && e[0] == '1'; }();
  const cudaError_t e = cudaGetLastError();
  if (verbose) fprintf(stderr, "i2cw: %s failed: %s\n", what, cudaGetErrorString(e));
  return I2CW_ECUDA;
}

// One fused launch sequence (K-chunks in order, split-tail zeroing first) writing y.
int run_fused_into(const Plan& pl, const float* x, const void* u, float* y, bool after_own_ft, cudaStream_t stream) {
  CUtensorMap map, ymap;
  if (pl.NITEMS != pl.NFULL) {
    // split tail: both passes of a tail unit reduce-add into y, so y is zeroed from the first
    // image the tail touches (earlier rows of that image are overwritten by whole-unit stores)
    const int tb0 = (pl.pair ? 2 : 1) * (pl.NFULL / pl.NB);  // first tile block of the tail
    const int ib = tb0 / pl.SEGS / pl.PB;  // image block of the first tail unit
    size_t n0 = pl.vol ? (size_t)(ib / pl.DB) : (size_t)ib * pl.NI;
    if (pl.strip) n0 = (size_t)((long long)tb0 * 4 / pl.T_r / pl.PB);  // image of the tail's first strip
    const size_t img = (size_t)pl.OD * pl.P * pl.Q * pl.K;
    if (n0 < (size_t)pl.N &&
        launch_zero_tail(y + n0 * img, ((size_t)pl.N - n0) * img, !after_own_ft, stream) != cudaSuccess)
      return cuda_fail("zero tail");
  }
  YMaps ym;
  int rc = pl.strip ? encode_x_map_strip(pl, x, &map) : encode_x_map(pl, x, &map);
  if (rc != I2CW_OK) return rc;
  if (pl.strip) {
    for (int L = 1; L <= 4; ++L)
      if ((rc = encode_y_map_strip(pl, y, L, &ym.m[L - 1])) != I2CW_OK) return rc;
  } else if ((rc = encode_y_map(pl, y, &ymap)) != I2CW_OK) {
    return rc;
  }
  const float* ud = reinterpret_cast<const float*>(static_cast<const uint8_t*>(u) + kUTagBytes);
  // K-chunks: one launch per chunk of <= CPC channel chunks, in order on the
  // stream; the first stores y (its split tail reduce-adds into the zeroed region), later ones
  // add every pass. Sequential launches keep the fp32 summation order fixed.
  for (int kc = 0; kc < pl.NKC; ++kc) {
    Plan pk = pl;
    pk.CC0 = pl.CC0 + kc * pl.CPC;
    pk.CC1 = std::min(pl.CC1, pk.CC0 + pl.CPC);
    pk.ACCUM = kc > 0;
    // the split tail's two one-pass items per unit add in either order: exact only onto y = 0
    // (0 + a + b), so later chunks (y != 0) run every unit whole, its passes in order
    if (kc > 0) pk.NFULL = pk.NITEMS = pl.NFULL + (pl.NITEMS - pl.NFULL) / 2;
    const cudaError_t e = pl.strip ? (pl.alpha == 8 ? launch_fused_strip_a8(map, ym, pk, ud, stream) : cudaErrorInvalidValue)
                                   : launch_fused_tc(map, ymap, pk, ud, stream);
    if (e != cudaSuccess) return cuda_fail("fused launch");
  }
  return I2CW_OK;
}

// Small grids (SURVEY.md §7 hard part 7, §8(e): a per-GPU shard of a few images leaves most
// SMs idle, and one work unit's latency sets the time): the K loop is split into S slices
// launched CONCURRENTLY on forked streams, each into its own y-sized workspace (slice 0 into
// y), and a combine kernel sums the slices in a fixed order -- deterministic, and each slice's
// accumulation is shorter (more accurate). The planner sets S = Plan::KSL (make_plan_uncached).
// Per-device fork/join resources, created once: the slice streams and events. The mutex is
// held while a call issues its fork/join (host side, a few microseconds), so concurrent host
// threads never interleave records of the shared events.
struct ForkCtx {
  std::mutex mu;
  bool ready = false;
  cudaStream_t st[kMaxKSlices - 1] = {};
  cudaEvent_t ev[kMaxKSlices] = {};
};

ForkCtx* fork_ctx(int dev) {
  static ForkCtx ctx[64];
  return dev >= 0 && dev < 64 ? &ctx[dev] : nullptr;
}

int run_fused(const Plan& pl, const float* x, const void* u, float* y, bool after_own_ft, cudaStream_t stream) {
  const int S = pl.KSL;
  if (S <= 1) return run_fused_into(pl, x, u, y, after_own_ft, stream);
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) return cuda_fail("device");
  ForkCtx* fc = fork_ctx(dev);
  if (!fc) return I2CW_EINVAL;
  std::lock_guard<std::mutex> lk(fc->mu);
  if (!fc->ready) {
    for (auto& st : fc->st)
      if (cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking) != cudaSuccess) return cuda_fail("stream");
    for (auto& e : fc->ev)
      if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess) return cuda_fail("event");
    fc->ready = true;
  }
  const size_t ycount = (size_t)pl.N * pl.OD * pl.P * pl.Q * pl.K;
  const size_t ystride = (ycount + 63) / 64 * 64;  // 256-byte aligned slices (TMA base alignment)
  float* ws = nullptr;
  if (cudaMallocAsync(&ws, (size_t)(S - 1) * ystride * 4, stream) != cudaSuccess) return cuda_fail("alloc");
  const int per = cdiv(pl.NCC, S);
  int rc = I2CW_OK;
  if (cudaEventRecord(fc->ev[0], stream) != cudaSuccess) rc = cuda_fail("record");  // after U, workspace
  for (int s = 0; s < S && rc == I2CW_OK; ++s) {
    Plan ps = pl;
    ps.CC0 = s * per;
    ps.CC1 = std::min(pl.NCC, ps.CC0 + per);
    ps.CPC = ps.CC1 - ps.CC0;
    ps.NKC = 1;
    ps.KSL = 1;
    if (ps.CC0 >= ps.CC1) break;
    cudaStream_t st = s == 0 ? stream : fc->st[s - 1];
    if (s > 0 && cudaStreamWaitEvent(st, fc->ev[0], 0) != cudaSuccess) { rc = cuda_fail("fork"); break; }
    rc = run_fused_into(ps, x, u, s == 0 ? y : ws + (size_t)(s - 1) * ystride, s == 0 && after_own_ft, st);
    if (rc == I2CW_OK && s > 0 &&
        (cudaEventRecord(fc->ev[s], st) != cudaSuccess || cudaStreamWaitEvent(stream, fc->ev[s], 0) != cudaSuccess))
      rc = cuda_fail("join");
  }
  if (rc == I2CW_OK && launch_ksum(y, ws, S - 1, ycount, ystride, stream) != cudaSuccess) rc = cuda_fail("ksum");
  cudaFreeAsync(ws, stream);
  return rc;
}

int conv_plan(const Plan& plan, int is_deconv, const float* x, const float* w, float* y, cudaStream_t stream, bool simt,
              unsigned long long* trace);

int conv_common(int is_deconv, int N, int H, int W, int C, int K, int R, int S, int pad_h, int pad_w, const float* x,
                const float* w, float* y, cudaStream_t stream, bool simt, unsigned long long* trace = nullptr) {
  if (!x || !w || !y) return I2CW_EINVAL;
  if (!aligned16(x) || !aligned16(w) || !aligned16(y)) return I2CW_EINVAL;
  Plan pl;
  // the SIMT stepping stone reads the base plan's block shape
  int rc = simt ? make_plan3(N, 1, H, W, C, K, 1, R, S, 0, pad_h, pad_w, is_deconv, 0, &pl, 2)
                : make_plan(N, H, W, C, K, R, S, pad_h, pad_w, is_deconv, &pl);
  if (rc != I2CW_OK) return rc;
  return conv_plan(pl, is_deconv, x, w, y, stream, simt, trace);
}

// 3D convolution / deconvolution: NDHWC x, KTRSC (deconv: CTRSK) w, NDHWC y
int conv3_common(int is_deconv, int N, int D, int H, int W, int C, int K, int T, int R, int S, int pad_d, int pad_h,
                 int pad_w, const float* x, const float* w, float* y, cudaStream_t stream) {
  if (!x || !w || !y) return I2CW_EINVAL;
  if (!aligned16(x) || !aligned16(w) || !aligned16(y)) return I2CW_EINVAL;
  Plan pl;
  int rc = make_plan3(N, D, H, W, C, K, T, R, S, pad_d, pad_h, pad_w, is_deconv, 1, &pl);
  if (rc != I2CW_OK) return rc;
  return conv_plan(pl, is_deconv, x, w, y, stream, false, nullptr);
}

int conv_plan(const Plan& plan, int is_deconv, const float* x, const float* w, float* y, cudaStream_t stream, bool simt,
              unsigned long long* trace) {
  Plan pl = plan;
  int rc = I2CW_OK;
  pl.trace = trace;
  if (simt) pl.pair = 0;  // the SIMT stepping stone reads the single-CTA U layout
  if ((rc = bind_device_of(x)) != I2CW_OK) return rc;
  void* u = nullptr;
  const size_t ub = kUTagBytes + u_data_bytes(pl);
  if (cudaMallocAsync(&u, ub, stream) != cudaSuccess) { cudaGetLastError(); return I2CW_ECUDA; }
  rc = transform_into(pl, is_deconv, w, u, stream);
  if (rc == I2CW_OK) {
    if (simt)
      rc = launch_fused_simt(pl, x, reinterpret_cast<const float*>(static_cast<uint8_t*>(u) + kUTagBytes), y, stream) ==
                   cudaSuccess
               ? I2CW_OK
               : I2CW_ECUDA;
    else
      rc = run_fused(pl, x, u, y, /*after_own_ft=*/true, stream);
  }
  cudaFreeAsync(u, stream);
  if (rc != I2CW_OK) cudaGetLastError();
  return rc;
}

int pretransformed_common(int is_deconv, int N, int H, int W, int C, int K, int R, int S, int pad_h, int pad_w,
                          const float* x, const void* u, float* y, cudaStream_t stream) {
  if (!x || !u || !y) return I2CW_EINVAL;
  if (!aligned16(x) || !aligned16(u) || !aligned16(y)) return I2CW_EINVAL;
  Plan pl;
  int rc = make_plan(N, H, W, C, K, R, S, pad_h, pad_w, is_deconv, &pl);
  if (rc != I2CW_OK) return rc;
  if (pl.strip) {  // u has the filter-only (base) plan's layout (i2cw_filter_transform)
    Plan pb;
    if ((rc = make_plan3(N, 1, H, W, C, K, 1, R, S, 0, pad_h, pad_w, is_deconv, 0, &pb, 2)) != I2CW_OK) return rc;
    if (pl.pair && !pb.pair) {
      // the single-CTA strip kernel reads that layout and sums in the same order (bitwise equal)
      if ((rc = make_plan3(N, 1, H, W, C, K, 1, R, S, 0, pad_h, pad_w, is_deconv, 0, &pl, 4)) != I2CW_OK) return rc;
    } else if (!pl.pair && pb.pair) {
      pl = pb;  // a strip plan too small for CTA pairs: the base kernel reads the pair layout
    }
  }
  if ((rc = bind_device_of(x)) != I2CW_OK) return rc;
  auto matches = [&](const UTag& t) {
    return t.magic == kUMagic && (int)t.is_deconv == is_deconv && (int)t.C == C && (int)t.K == K && (int)t.R == R &&
           (int)t.S == S && (int)t.alpha == pl.alpha && (int)t.m == pl.m && (int)t.NT == pl.NT &&
           (int)t.halves == (pl.pair ? 2 : 1);
  };
  // Host copy of the tag (written by i2cw_filter_transform for this address) when it matches;
  // otherwise -- an unknown u, or a host entry that disagrees (the address may have been freed
  // and reused) -- the device tag decides (one small synchronous read). The fused kernel checks
  // the device tag again and traps on a mismatch, so a stale host entry cannot pass silently.
  UTag tag;
  if (!registry_lookup(u, &tag) || !matches(tag)) {
    if (cudaMemcpyAsync(&tag, u, sizeof(tag), cudaMemcpyDeviceToHost, stream) != cudaSuccess ||
        cudaStreamSynchronize(stream) != cudaSuccess) {
      cudaGetLastError();
      return I2CW_ECUDA;
    }
    if (!matches(tag)) return I2CW_EINVAL;
    registry_put(u, tag);
  }
  rc = run_fused(pl, x, u, y, /*after_own_ft=*/false, stream);
  if (rc != I2CW_OK) cudaGetLastError();
  return rc;
}

}  // namespace
}  // namespace i2cw

using namespace i2cw;

extern "C" {

const char* i2cw_status_string(int s) {
  switch (s) {
    case I2CW_OK: return "ok";
    case I2CW_EINVAL: return "invalid argument";
    case I2CW_EUNSUPPORTED: return "unsupported shape";
    case I2CW_ECUDA: return "CUDA error";
    default: return "unknown status";
  }
}

int i2cw_version(void) { return 20000; }

int i2cw_conv2d_nhwc(int N, int H, int W, int C, int K, int R, int S, int pad_h, int pad_w, const float* x,
                     const float* w, float* y, i2cw_stream_t stream) {
  return conv_common(0, N, H, W, C, K, R, S, pad_h, pad_w, x, w, y, (cudaStream_t)stream, false);
}

int i2cw_deconv2d_nhwc(int N, int H, int W, int C, int K, int R, int S, int pad_h, int pad_w, const float* x,
                       const float* w, float* y, i2cw_stream_t stream) {
  return conv_common(1, N, H, W, C, K, R, S, pad_h, pad_w, x, w, y, (cudaStream_t)stream, false);
}

// NCHW adapter (f4): transpose x (NCHW -> NHWC) and the filter (OIHW -> KRSC, or for the
// deconv the [C][K][R][S] conv_transpose weight -> CRSK) into pooled workspaces, run the NHWC
// call, transpose y back. Costs one extra read + write of x, y and w in HBM.
static int nchw_common(int is_deconv, int N, int C, int H, int W, int K, int R, int S, int pad_h, int pad_w,
                       const float* x, const float* w, float* y, cudaStream_t stream) {
  if (!x || !w || !y) return I2CW_EINVAL;
  if (!aligned16(x) || !aligned16(w) || !aligned16(y)) return I2CW_EINVAL;
  Plan pl;
  int rc = make_plan(N, H, W, C, K, R, S, pad_h, pad_w, is_deconv, &pl);
  if (rc != I2CW_OK) return rc;
  if ((rc = bind_device_of(x)) != I2CW_OK) return rc;
  const size_t nx = (size_t)N * C * H * W, nw = (size_t)K * C * R * S, ny = (size_t)N * K * pl.P * pl.Q;
  float *xt = nullptr, *wt = nullptr, *yt = nullptr;
  if (cudaMallocAsync(&xt, nx * 4, stream) != cudaSuccess || cudaMallocAsync(&wt, nw * 4, stream) != cudaSuccess ||
      cudaMallocAsync(&yt, ny * 4, stream) != cudaSuccess) {
    cudaGetLastError();
    if (xt) cudaFreeAsync(xt, stream);
    if (wt) cudaFreeAsync(wt, stream);
    return I2CW_ECUDA;
  }
  if (launch_transpose(x, xt, N, C, H * W, stream) != cudaSuccess ||
      // conv: OIHW [K][C][R*S] -> [K][R*S][C]; deconv: [C][K][R*S] -> [C][R*S][K]
      launch_transpose(w, wt, is_deconv ? C : K, is_deconv ? K : C, R * S, stream) != cudaSuccess)
    rc = I2CW_ECUDA;
  if (rc == I2CW_OK) rc = conv_common(is_deconv, N, H, W, C, K, R, S, pad_h, pad_w, xt, wt, yt, stream, false);
  if (rc == I2CW_OK && launch_transpose(yt, y, N, pl.P * pl.Q, K, stream) != cudaSuccess) rc = I2CW_ECUDA;
  cudaFreeAsync(xt, stream);
  cudaFreeAsync(wt, stream);
  cudaFreeAsync(yt, stream);
  if (rc != I2CW_OK) cudaGetLastError();
  return rc;
}

int i2cw_conv2d_nchw(int N, int C, int H, int W, int K, int R, int S, int pad_h, int pad_w, const float* x,
                     const float* w, float* y, i2cw_stream_t stream) {
  return nchw_common(0, N, C, H, W, K, R, S, pad_h, pad_w, x, w, y, (cudaStream_t)stream);
}

int i2cw_deconv2d_nchw(int N, int C, int H, int W, int K, int R, int S, int pad_h, int pad_w, const float* x,
                       const float* w, float* y, i2cw_stream_t stream) {
  return nchw_common(1, N, C, H, W, K, R, S, pad_h, pad_w, x, w, y, (cudaStream_t)stream);
}

int i2cw_conv2d_nhwc_prec(int precision, int is_deconv, int N, int H, int W, int C, int K, int R, int S, int pad_h,
                          int pad_w, const float* x, const float* w, float* y, i2cw_stream_t stream) {
  if (precision == I2CW_PREC_3XTF32)
    return conv_common(is_deconv ? 1 : 0, N, H, W, C, K, R, S, pad_h, pad_w, x, w, y, (cudaStream_t)stream, false);
  if (precision != I2CW_PREC_1XTF32 || (is_deconv != 0 && is_deconv != 1)) return I2CW_EINVAL;
  if (!x || !w || !y) return I2CW_EINVAL;
  if (!aligned16(x) || !aligned16(w) || !aligned16(y)) return I2CW_EINVAL;
  Plan pl;
  int rc = make_plan3(N, 1, H, W, C, K, 1, R, S, 0, pad_h, pad_w, is_deconv, 0, &pl, 1);
  if (rc != I2CW_OK) return rc;
  return conv_plan(pl, is_deconv, x, w, y, (cudaStream_t)stream, false, nullptr);
}

int i2cw_conv3d_ndhwc(int N, int D, int H, int W, int C, int K, int T, int R, int S, int pad_d, int pad_h, int pad_w,
                      const float* x, const float* w, float* y, i2cw_stream_t stream) {
  return conv3_common(0, N, D, H, W, C, K, T, R, S, pad_d, pad_h, pad_w, x, w, y, (cudaStream_t)stream);
}

int i2cw_deconv3d_ndhwc(int N, int D, int H, int W, int C, int K, int T, int R, int S, int pad_d, int pad_h, int pad_w,
                        const float* x, const float* w, float* y, i2cw_stream_t stream) {
  return conv3_common(1, N, D, H, W, C, K, T, R, S, pad_d, pad_h, pad_w, x, w, y, (cudaStream_t)stream);
}

size_t i2cw_filter_bytes(int K, int C, int R, int S) {
  Plan pl;
  // the filter-side plan fields do not depend on N, H, W or pad: plan a 1 x R x S map (base
  // kernel layout; a call whose plan would use the strip kernel's CTA-pair layout instead runs
  // the base kernel on a pre-transformed U, pretransformed_common)
  if (make_plan3(1, 1, R, S, C, K, 1, R, S, 0, 0, 0, 0, 0, &pl, 2) != I2CW_OK) return 0;
  return kUTagBytes + u_data_bytes(pl);
}

int i2cw_filter_transform(int K, int C, int R, int S, int is_deconv, const float* w, void* u, i2cw_stream_t stream) {
  if (!w || !u || !aligned16(w) || !aligned16(u) || (is_deconv != 0 && is_deconv != 1)) return I2CW_EINVAL;
  Plan pl;
  int rc = make_plan3(1, 1, R, S, C, K, 1, R, S, 0, 0, 0, is_deconv, 0, &pl, 2);
  if (rc != I2CW_OK) return rc;
  if ((rc = bind_device_of(w)) != I2CW_OK) return rc;
  rc = transform_into(pl, is_deconv, w, u, (cudaStream_t)stream);
  if (rc != I2CW_OK) {
    cudaGetLastError();
    return rc;
  }
  // host copy of the caller-owned u's tag (internal workspaces are never registered)
  const UTag tag = make_tag(pl, is_deconv);
  registry_put(u, tag);
  return rc;
}

int i2cw_conv2d_nhwc_pretransformed(int N, int H, int W, int C, int K, int R, int S, int pad_h, int pad_w,
                                    const float* x, const void* u, float* y, i2cw_stream_t stream) {
  return pretransformed_common(0, N, H, W, C, K, R, S, pad_h, pad_w, x, u, y, (cudaStream_t)stream);
}

int i2cw_deconv2d_nhwc_pretransformed(int N, int H, int W, int C, int K, int R, int S, int pad_h, int pad_w,
                                      const float* x, const void* u, float* y, i2cw_stream_t stream) {
  return pretransformed_common(1, N, H, W, C, K, R, S, pad_h, pad_w, x, u, y, (cudaStream_t)stream);
}

int i2cw_set_device(int device) {
  if (cudaSetDevice(device) != cudaSuccess) { cudaGetLastError(); return I2CW_ECUDA; }
  ensure_pool(device);
  return I2CW_OK;
}

int i2cw_conv2d_nhwc_host(int is_deconv, int N, int H, int W, int C, int K, int R, int S, int pad_h, int pad_w,
                          const float* x_host, const float* w_host, float* y_host, i2cw_stream_t stream_) {
  if (!x_host || !w_host || !y_host || (is_deconv != 0 && is_deconv != 1)) return I2CW_EINVAL;
  cudaStream_t stream = (cudaStream_t)stream_;
  Plan pl;
  int rc = make_plan(N, H, W, C, K, R, S, pad_h, pad_w, is_deconv, &pl);
  if (rc != I2CW_OK) return rc;
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) { cudaGetLastError(); return I2CW_ECUDA; }
  ensure_pool(dev);
  // Pipelined over image chunks: the host->device copy of chunk c+1 and the device->host copy
  // of chunk c-1 run on two copy streams while chunk c computes on `stream` (PCIe is full
  // duplex; the copies, not the kernel, bound this call). The filter is transformed once.
  // I2CW_HOST_CHUNKS=<n> (experiments): chunk count; 8 measured best on cfg2
  static const int chunks_env = [] { const char* e = getenv("I2CW_HOST_CHUNKS"); return e ? atoi(e) : 0; }();
  const int nchunk = std::max(1, std::min(N, chunks_env > 0 ? chunks_env : 8));
  const size_t img_x = (size_t)H * W * C, img_y = (size_t)pl.P * pl.Q * K;
  const size_t xb = (size_t)N * img_x * 4, wb = (size_t)K * R * S * C * 4, yb = (size_t)N * img_y * 4;
  static cudaStream_t s_in[64] = {}, s_out[64] = {};
  static std::mutex mu;
  {
    std::lock_guard<std::mutex> lk(mu);
    if (dev < 0 || dev >= 64) return I2CW_ECUDA;
    if (!s_in[dev] && (cudaStreamCreateWithFlags(&s_in[dev], cudaStreamNonBlocking) != cudaSuccess ||
                       cudaStreamCreateWithFlags(&s_out[dev], cudaStreamNonBlocking) != cudaSuccess)) {
      cudaGetLastError();
      return I2CW_ECUDA;
    }
  }
  cudaStream_t si = s_in[dev], so = s_out[dev];
  float *xd = nullptr, *wd = nullptr, *yd = nullptr;
  void* u = nullptr;
  const size_t ub = kUTagBytes + u_data_bytes(pl);
  if (cudaMallocAsync(&xd, xb, stream) != cudaSuccess || cudaMallocAsync(&wd, wb, stream) != cudaSuccess ||
      cudaMallocAsync(&yd, yb, stream) != cudaSuccess || cudaMallocAsync(&u, ub, stream) != cudaSuccess) {
    cudaGetLastError();
    if (xd) cudaFreeAsync(xd, stream);
    if (wd) cudaFreeAsync(wd, stream);
    if (yd) cudaFreeAsync(yd, stream);
    return I2CW_ECUDA;
  }
  std::vector<cudaEvent_t> ev(2 * nchunk + 1, nullptr);
  for (auto& e : ev)
    if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess) rc = I2CW_ECUDA;
  // the copy streams start after the allocations (and all earlier work) on `stream`
  if (rc == I2CW_OK && (cudaEventRecord(ev[2 * nchunk], stream) != cudaSuccess ||
                        cudaStreamWaitEvent(si, ev[2 * nchunk], 0) != cudaSuccess ||
                        cudaStreamWaitEvent(so, ev[2 * nchunk], 0) != cudaSuccess))
    rc = I2CW_ECUDA;
  if (rc == I2CW_OK && cudaMemcpyAsync(wd, w_host, wb, cudaMemcpyHostToDevice, stream) != cudaSuccess) rc = I2CW_ECUDA;
  if (rc == I2CW_OK) rc = transform_into(pl, is_deconv, wd, u, stream);
  int n0 = 0;
  for (int c = 0; c < nchunk && rc == I2CW_OK; ++c) {
    const int nc = N / nchunk + (c < N % nchunk ? 1 : 0);
    Plan pc;
    if ((rc = make_plan(nc, H, W, C, K, R, S, pad_h, pad_w, is_deconv, &pc)) != I2CW_OK) break;
    float* xdc = xd + (size_t)n0 * img_x;
    float* ydc = yd + (size_t)n0 * img_y;
    if (cudaMemcpyAsync(xdc, x_host + (size_t)n0 * img_x, (size_t)nc * img_x * 4, cudaMemcpyHostToDevice, si) !=
            cudaSuccess ||
        cudaEventRecord(ev[2 * c], si) != cudaSuccess || cudaStreamWaitEvent(stream, ev[2 * c], 0) != cudaSuccess) {
      rc = I2CW_ECUDA;
      break;
    }
    if ((rc = run_fused(pc, xdc, u, ydc, /*after_own_ft=*/c == 0, stream)) != I2CW_OK) break;
    if (cudaEventRecord(ev[2 * c + 1], stream) != cudaSuccess || cudaStreamWaitEvent(so, ev[2 * c + 1], 0) != cudaSuccess ||
        cudaMemcpyAsync(y_host + (size_t)n0 * img_y, ydc, (size_t)nc * img_y * 4, cudaMemcpyDeviceToHost, so) !=
            cudaSuccess) {
      rc = I2CW_ECUDA;
      break;
    }
    n0 += nc;
  }
  // the buffers are freed on `stream` after the last device->host copy
  cudaEvent_t done = nullptr;
  if (cudaEventCreateWithFlags(&done, cudaEventDisableTiming) == cudaSuccess) {
    cudaEventRecord(done, so);
    cudaStreamWaitEvent(stream, done, 0);
  }
  cudaFreeAsync(xd, stream);
  cudaFreeAsync(wd, stream);
  cudaFreeAsync(yd, stream);
  cudaFreeAsync(u, stream);
  if (cudaStreamSynchronize(stream) != cudaSuccess) rc = I2CW_ECUDA;
  for (auto& e : ev)
    if (e) cudaEventDestroy(e);
  if (done) cudaEventDestroy(done);
  if (rc != I2CW_OK) cudaGetLastError();
  return rc;
}

int i2cw_plan(int S, int C, int* m, int* alpha, int* point_set) {
  Choice c;
  if (C <= 0) return I2CW_EINVAL;
  if (!choose(S, C, &c)) return I2CW_EUNSUPPORTED;
  if (m) *m = c.m;
  if (alpha) *alpha = c.alpha;
  if (point_set) *point_set = c.point_set;
  return I2CW_OK;
}

int i2cw_transform_matrices_rational(int m, int r, int point_set, int64_t* at_num, int64_t* at_den, int64_t* g_num,
                                     int64_t* g_den, int64_t* bt_num, int64_t* bt_den) {
  if (m < 1 || r < 1 || m + r - 1 > 16 || m + r - 1 < 2 || (point_set != 0 && point_set != 1)) return I2CW_EINVAL;
  if (point_set == 1 && m + r - 1 != 16) return I2CW_EINVAL;
  if (!at_num || !at_den || !g_num || !g_den || !bt_num || !bt_den) return I2CW_EINVAL;
  Transforms T;
  try {
    T = cook_toom(m, r, point_set);
  } catch (...) {
    return I2CW_EUNSUPPORTED;
  }
  const i128 lim = (i128)INT64_MAX;
  auto put = [&](const std::vector<Rat>& v, int64_t* num, int64_t* den) {
    for (size_t i = 0; i < v.size(); ++i) {
      if (v[i].n > lim || v[i].n < -lim || v[i].d > lim) return false;
      num[i] = (int64_t)v[i].n;
      den[i] = (int64_t)v[i].d;
    }
    return true;
  };
  if (!put(T.AT, at_num, at_den) || !put(T.G, g_num, g_den) || !put(T.BT, bt_num, bt_den)) return I2CW_EUNSUPPORTED;
  return I2CW_OK;
}

// ---- not part of the public header: test hooks (csrc/debug_api.h) ----
I2CW_API int i2cw_debug_conv_simt(int is_deconv, int N, int H, int W, int C, int K, int R, int S, int pad_h, int pad_w,
                         const float* x, const float* w, float* y, i2cw_stream_t stream) {
  return conv_common(is_deconv, N, H, W, C, K, R, S, pad_h, pad_w, x, w, y, (cudaStream_t)stream, true);
}

// Longest TMEM accumulation in k-steps (0 restores the per-alpha default); returns the previous
// setting (0 = default).
I2CW_API int i2cw_debug_set_kchunk(int ksteps) { return g_kchunk_max.exchange(ksteps > 0 ? ksteps : 0); }
I2CW_API int i2cw_debug_set_kslices(int n) { return g_kslices_max.exchange(n > 0 ? n : -1); }

// Runs the product path with CTA 0's event timeline recorded into trace (device,
// 32 kinds x 512 uint64 clock64 stamps; see trace_rec in common.cuh).
I2CW_API int i2cw_debug_trace(int is_deconv, int N, int H, int W, int C, int K, int R, int S, int pad_h, int pad_w,
                              const float* x, const float* w, float* y, unsigned long long* trace,
                              i2cw_stream_t stream) {
  return conv_common(is_deconv, N, H, W, C, K, R, S, pad_h, pad_w, x, w, y, (cudaStream_t)stream, false, trace);
}

I2CW_API int i2cw_debug_plan(int is_deconv, int N, int H, int W, int C, int K, int R, int S, int pad_h, int pad_w,
                    int* out /* 40 ints */) {
  Plan pl;
  int rc = make_plan(N, H, W, C, K, R, S, pad_h, pad_w, is_deconv, &pl);
  if (rc != I2CW_OK) return rc;
  int v[] = {pl.P, pl.Q, pl.m, pl.alpha, pl.NT, pl.NB, pl.NCC, pl.NKS, pl.T_r, pl.TS, pl.SEGS, pl.ROWS, pl.PB,
             pl.WBOX, pl.HBOX, pl.tile_blocks, pl.GP, pl.NPASS, pl.NUS, pl.smem_bytes, pl.pad_h, pl.pad_w, pl.NI,
             pl.NFULL, pl.NITEMS, pl.pair, pl.NKC, pl.CPC, pl.KSL, pl.NIS, pl.NOB, pl.PLANE, pl.strip, pl.NSTRIP};
  for (int i = 0; i < 40; ++i) out[i] = i < (int)(sizeof(v) / sizeof(v[0])) ? v[i] : 0;
  return I2CW_OK;
}

}  // extern "C"
