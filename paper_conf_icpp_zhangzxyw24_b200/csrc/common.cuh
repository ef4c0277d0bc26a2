// Shared definitions for the i2cw CUDA path: the launch plan (host-computed,
// passed by value) and thin inline-PTX wrappers for sm_100a mbarrier, TMA /
// bulk copies and tcgen05 (TMEM alloc, MMA, ld/st, commit, fences).
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <cstdio>

#ifndef I2CW_ABLATION
#define I2CW_ABLATION 0  // 1: timing-ablation branches compiled in (make ABLATION=1; tools only)
#endif

namespace i2cw {

constexpr int kMaxLanes = 128;  // UMMA M = 128 Winograd tiles per CTA (one TMEM lane each)

// Everything the kernels need about one call; built by make_plan() in api.cu.
struct Plan {
  int N, H, W, C, K, R, S;
  int is_deconv;        // 1: deconvolution (U holds the rotated, channel-transposed filter)
  int vol;              // 1: 3D convolution (x NDHWC, filter KTRSC): D, T, pad_d, OD, DB below
  int D, T, pad_d, OD;  // input depth, filter depth taps, depth padding (kernel's view), output depth
  int DB;               // 3D: depth blocks per image = ceil(OD / NI) (a tile block stacks NI output depths)
  int pad_h, pad_w;     // conv padding as seen by the kernel (deconv: R-1-pad, may be < 0)
  int P, Q;             // output height / width
  int m, alpha;         // F(m, S), alpha = m + S - 1
  int NT;               // output channels per CTA (UMMA N)
  int NB;               // ceil(K / NT)
  int NCC;              // chunks of the K loop: ceil(C / 8) channel chunks (8 fp32 = one tf32 UMMA K
                        // step), times T depth taps in 3D (virtual chunk vc = cc * T + fd)
  int NKS;              // k-steps = NCC * R  (ks = vc * R + fh)
  int T_r;              // Winograd tiles per output row = ceil(Q / m)
  int TS;               // tiles per row segment handled by one CTA
  int SEGS;             // segments per row = ceil(T_r / TS)
  int ROWS;             // output rows per CTA
  int PB;               // row blocks per image = ceil(P / ROWS)
  int NI;               // images per tile block (the block's lanes are NI x ROWS x TS tiles)
  int WBOX, HBOX;       // staged input box (columns, rows = ROWS + R - 1)
  int BOXB;             // bytes of one TMA input box (8 channels) = NI*HBOX*WBOX*32
  int PLANE;            // half an input stage (BOXB rounded up to 1024, halved)
  int tile_blocks;      // ceil(N / NI) * PB * SEGS
  int NFULL, NITEMS;    // work items: [0, NFULL) whole units; then 2 per tail unit (one per pass)
  int GP, NPASS;        // points per pass (TMEM budget), point groups = alpha / GP
  int NKC, CPC;         // K-chunks (launches) of the K loop, channel chunks per K-chunk (bounded accumulation)
  int CC0, CC1;         // this launch's channel chunks [CC0, CC1) (set per K-chunk launch)
  int ACCUM;            // 1: every pass adds into y (a K-chunk after the first)
  int KSL;              // concurrent K-slice launches (small grids, api.cu run_fused); 1: none
  int prec;             // 0: 3xTF32 (default, fp32 accuracy); 1: 1xTF32 (looser tolerance, f4)
  int NUS;              // U ring super-slots (KPS k-steps of GP points each)
  int OSB;              // bytes of one output staging buffer = NI*ROWS*TS*16*4 (TMA store box, 16 channels)
  int OSTRIDE;          // OSB rounded up to 1024 (swizzled TMA boxes need 1024-byte alignment)
  int NOB;              // output staging buffers per warpgroup (1..4)
  int NIS;              // input (x row box) stages
  int smem_bytes;
  int pair;             // 1: CTA pairs (cluster of 2) with tcgen05.mma.cta_group::2, U split by N halves
  int strip;            // 1: strip kernel (fused_strip.cuh): one input-row transform per chunk, TMEM row
                        // shifts between filter rows; ROWS = valid rows per strip, TS = 4 strips per unit
  int NSTRIP;           // strip kernel: strips = N * PB * T_r (tile column tw fastest)
  int KU;               // strip kernel: k-steps per U ring slot (R: one barrier round trip per chunk, or 1)
  int ablate;           // DEBUG timing ablation (I2CW_ABLATE, results wrong): 1 no transform math,
                        // 2 no MMAs, 4 no epilogue math/stores; 0 in production
  unsigned long long* trace;  // debug timeline of CTA 0 (nullptr = off), see i2cw_debug_trace
  unsigned char lane_row[kMaxLanes];  // lane -> virtual row img*ROWS + row within block (0xFF = idle lane)
  unsigned short lane_in[kMaxLanes];  // lane -> first input row in the staged box, img*HBOX + row
  unsigned char lane_tw[kMaxLanes];   // lane -> tile within segment
};

// Points per TMEM pass: GP * NT = 256 accumulator columns (GP even, dividing alpha; the
// other 256 columns hold the V slots).
__host__ __device__ constexpr int gp_for(int alpha, int NT) {
  return alpha <= 4 ? alpha : (NT == 128 ? 2 : (NT == 64 ? 4 : (alpha % 8 == 0 ? 8 : 6)));
}
// V slots (one k-step of GP points, hi + lo, each) next to the accumulators:
// NS * GP * 16 <= 512 - GP * NT. NT = 128: 8 slots of 32 columns (two per warpgroup);
// NT = 64: 4 of 64; NT = 32: 2 of 128.
__host__ __device__ constexpr int ns_for(int alpha, int NT) {
  return NT == 128 ? 8
                   : (((512 - gp_for(alpha, NT) * NT) / (gp_for(alpha, NT) * 16)) >= 4
                          ? 4
                          : (((512 - gp_for(alpha, NT) * NT) / (gp_for(alpha, NT) * 16)) / 2) * 2);
}
// k-steps per super-stage (one barrier round trip + one U slot): 2 when 4 V slots fit
#ifndef I2CW_KPS_MAX
#define I2CW_KPS_MAX 2
#endif
__host__ __device__ constexpr int kps_for(int alpha, int NT) { return ns_for(alpha, NT) >= 4 ? I2CW_KPS_MAX : 1; }
// MMA-issuing warps: each owns whole accumulators (deterministic accumulation order). Two
// warps, each issuing warp-uniformly (elect.sync inside the asm), keep up with 32-cycle UMMAs.
__host__ __device__ constexpr int niss_for(int GP) { return GP % 2 == 0 ? 2 : 1; }
// Transform / epilogue warpgroups: the input transform of one k-step by one
// warpgroup (one warp per SMSP) is latency-bound, so NT=64 (4 stages) uses 4
// warpgroups, each owning one stage and 16 output channels in the epilogue.
__host__ __device__ constexpr int nwg_for(int NT) { return NT >= 64 ? 4 : 2; }
__host__ __device__ constexpr int tc_threads(int GP, int NT) { return nwg_for(NT) * 128 + 64 + niss_for(GP) * 32; }

// Internal Winograd point order: singles {0, alpha-1} first, then the ± pairs
// (1,2), (3,4), ... so that every pass of GP (even) points holds whole pairs
// (PAPER.md:595-603 pair structure).
__host__ __device__ constexpr int point_of(int idx, int alpha) {
  return idx == 0 ? 0 : (idx == 1 ? alpha - 1 : idx - 1);
}

// U (transformed filter) layout, fp32 words:
//   U[nb][ks][idx][hl][kc][n][e],  idx = internal point index, hl = 0 hi / 1 lo,
//   kc = 16-byte half of the 8-channel k-step, n < NT, e < 4  (channel = cc*8 + kc*4 + e)
// i.e. one k-step's image for one (point, hl) is the UMMA K-major SWIZZLE_NONE
// canonical layout of an NT x 8 tf32 tile with SBO = 128 B, LBO = NT * 16 B.
__host__ __device__ inline size_t u_offset(int NT, int alpha, int nb, int NKS, int ks, int idx, int hl) {
  return ((((size_t)nb * NKS + ks) * alpha + idx) * 2 + hl) * (size_t)NT * 8;
}

// CTA-pair layout (Plan::pair): the N rows of every image are split in two halves owned
// by the two CTAs of a cluster; per (nb, ks) the halves are outermost so one CTA's share of
// a pass is one contiguous run:  U[nb][ks][h][idx][hl][kc][n'][e],  n' < NT/2.
// Returns the offset of image (nb, ks, h, idx, hl = 0); hl = 1 follows at + (NT/2)*8.
__host__ __device__ inline size_t u_offset_pair(int NT, int alpha, int nb, int NKS, int ks, int h, int idx) {
  return (((((size_t)nb * NKS + ks) * 2 + h) * alpha + idx) * 2) * (size_t)(NT / 2) * 8;
}

constexpr int kUTagBytes = 256;
constexpr uint32_t kUMagic = 0x49324357u;  // "I2CW"
struct UTag {
  uint32_t magic, alpha, m, is_deconv, C, K, R, S, NT, NB, NCC, halves, T;  // T: depth taps (2D: 1)
};

#if defined(__CUDACC__)
// Debug timeline: CTA b < 2, kind k, entry i -> trace[(b * 32 + k) * 512 + i] = clock64 of the
// SM (cycles; not comparable across the two SMs of a CTA pair). The "memory" clobber keeps
// the compiler from moving loads/stores across a trace point.
// Timeline tracing (tools/trace_run.py) is compiled in only with `make TRACE=1`
// (-DI2CW_TRACE=1): in the product build trace_rec() is empty and costs no issue slots.
#ifndef I2CW_TRACE
#define I2CW_TRACE 0
#endif
__device__ __forceinline__ void trace_rec(unsigned long long* tr, int kind, int i, bool on = true) {
#if I2CW_TRACE
  if (on && tr != nullptr && blockIdx.x < 2 && i < 512) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%clock64;" : "=l"(t)::"memory");
    tr[(blockIdx.x * 32 + kind) * 512 + i] = t;
  }
#else
  (void)tr; (void)kind; (void)i; (void)on;
#endif
}
// ----------------------------------------------------------------------------
// PTX helpers
// ----------------------------------------------------------------------------
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ uint64_t globaltimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
// I2CW_WAITMODE (build-time experiment switch): 0 = try_wait (HW-chosen suspend time),
// 1 = test_wait polling (never suspends), 2 = try_wait with an explicit 32 ns suspend hint.
#ifndef I2CW_WAITMODE
#define I2CW_WAITMODE 0
#endif
__device__ __forceinline__ bool mbar_try_wait(uint64_t* bar, uint32_t parity) {
  uint32_t ok;
#if I2CW_WAITMODE == 1
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "mbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
      "selp.u32 %0, 1, 0, p;\n\t}"
      : "=r"(ok)
      : "r"(smem_u32(bar)), "r"(parity)
      : "memory");
#elif I2CW_WAITMODE == 2
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\t"
      "selp.u32 %0, 1, 0, p;\n\t}"
      : "=r"(ok)
      : "r"(smem_u32(bar)), "r"(parity), "r"(32u)
      : "memory");
#else
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
      "selp.u32 %0, 1, 0, p;\n\t}"
      : "=r"(ok)
      : "r"(smem_u32(bar)), "r"(parity)
      : "memory");
#endif
  return ok != 0;
}
// Blocking wait with a watchdog: a protocol bug traps (launch error) after ~4 s
// instead of hanging the GPU.
#ifndef I2CW_WATCHDOG_PRINT
#define I2CW_WATCHDOG_PRINT 0  // debug builds: report the stuck barrier before trapping
#endif
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  if (mbar_try_wait(bar, parity)) return;
  const uint64_t t0 = globaltimer();
  while (!mbar_try_wait(bar, parity)) {
    if (globaltimer() - t0 > 4000000000ull) {
#if I2CW_WATCHDOG_PRINT
      printf("i2cw watchdog: block %d thread %d smem bar 0x%x parity %u\n", blockIdx.x, threadIdx.x, smem_u32(bar), parity);
#endif
      __trap();
    }
  }
}

// TMA: 4D tiled tensor load global -> shared, completes on an mbarrier (tx bytes)
__device__ __forceinline__ void tma_load_4d(void* smem_dst, const CUtensorMap* map, uint64_t* bar, int c0, int c1,
                                            int c2, int c3) {
  asm volatile(
      "cp.async.bulk.tensor.4d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%2, %3, %4, %5}], [%6];" ::"r"(smem_u32(smem_dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "r"(smem_u32(bar))
      : "memory");
}
// TMA: 4D tiled tensor store shared -> global (OOB elements of the box are not written)
// 5D variants (3D convolution: C, W, H, D, N)
__device__ __forceinline__ void tma_load_5d(void* smem_dst, const CUtensorMap* map, uint64_t* bar, int c0, int c1,
                                            int c2, int c3, int c4) {
  asm volatile(
      "cp.async.bulk.tensor.5d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%2, %3, %4, %5, %6}], [%7];" ::"r"(smem_u32(smem_dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "r"(c4), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void tma_store_5d(const CUtensorMap* map, const void* smem_src, int c0, int c1, int c2,
                                             int c3, int c4) {
  asm volatile("cp.async.bulk.tensor.5d.global.shared::cta.tile.bulk_group [%0, {%2, %3, %4, %5, %6}], [%1];" ::"l"(
                   reinterpret_cast<uint64_t>(map)),
               "r"(smem_u32(smem_src)), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "r"(c4)
               : "memory");
}
__device__ __forceinline__ void tma_reduce_add_5d(const CUtensorMap* map, const void* smem_src, int c0, int c1,
                                                  int c2, int c3, int c4) {
  asm volatile(
      "cp.reduce.async.bulk.tensor.5d.global.shared::cta.add.tile.bulk_group [%0, {%2, %3, %4, %5, %6}], [%1];" ::"l"(
          reinterpret_cast<uint64_t>(map)),
      "r"(smem_u32(smem_src)), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "r"(c4)
      : "memory");
}
__device__ __forceinline__ void tma_store_4d(const CUtensorMap* map, const void* smem_src, int c0, int c1, int c2,
                                             int c3) {
  asm volatile("cp.async.bulk.tensor.4d.global.shared::cta.tile.bulk_group [%0, {%2, %3, %4, %5}], [%1];" ::"l"(
                   reinterpret_cast<uint64_t>(map)),
               "r"(smem_u32(smem_src)), "r"(c0), "r"(c1), "r"(c2), "r"(c3)
               : "memory");
}
// TMA: 4D tiled reduce-add shared -> global (fp32 add performed at L2)
__device__ __forceinline__ void tma_reduce_add_4d(const CUtensorMap* map, const void* smem_src, int c0, int c1,
                                                  int c2, int c3) {
  asm volatile(
      "cp.reduce.async.bulk.tensor.4d.global.shared::cta.add.tile.bulk_group [%0, {%2, %3, %4, %5}], [%1];" ::"l"(
          reinterpret_cast<uint64_t>(map)),
      "r"(smem_u32(smem_src)), "r"(c0), "r"(c1), "r"(c2), "r"(c3)
      : "memory");
}
__device__ __forceinline__ void bulk_commit_group() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void bulk_wait_group_read() {
  asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
// wait until at most n (runtime, <= 3; n < 0 waits for all) bulk groups are still reading smem
__device__ __forceinline__ void bulk_wait_group_read_dyn(int n) {
  if (n >= 3) bulk_wait_group_read<3>();
  else if (n == 2) bulk_wait_group_read<2>();
  else if (n == 1) bulk_wait_group_read<1>();
  else bulk_wait_group_read<0>();
}
__device__ __forceinline__ void bulk_wait_group_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
// generic-proxy shared-memory writes -> visible to the async proxy (TMA store reads)
__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void named_bar_sync(int id, int nthreads) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}

__device__ __forceinline__ void tma_prefetch_desc(const CUtensorMap* map) {
  asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(map)) : "memory");
}
// 1D bulk copy global -> shared (16-byte multiple), completes on an mbarrier
__device__ __forceinline__ void bulk_load(void* smem_dst, const void* gsrc, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(smem_dst)),
      "l"(gsrc), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}

// ---- clusters (CTA pairs for cta_group::2) ---------------------------------
__device__ __forceinline__ uint32_t cluster_ctarank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ void cluster_sync_all() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
// shared::cluster address of the same shared variable in CTA `rank` of the cluster
__device__ __forceinline__ uint32_t mapa_shared(const void* p, uint32_t rank) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(smem_u32(p)), "r"(rank));
  return r;
}
// Remote arrive on the peer CTA's barrier. Relaxed: every use forwards the completion of
// work that is already complete and visible to the tensor core (tcgen05.wait::st by the
// writers, TMA complete_tx), observed through a local barrier wait; a release.cluster
// arrive measured ~600 ns per call and paced the whole CTA pair.
__device__ __forceinline__ void mbar_arrive_remote(uint32_t cluster_addr) {
  asm volatile("mbarrier.arrive.relaxed.cluster.shared::cluster.b64 _, [%0];" ::"r"(cluster_addr) : "memory");
}
// parity wait with cluster-scope acquire, for barriers completed by the other CTA of a pair
// (remote mbarrier arrives, multicast tcgen05.commit). Measured: a suspended try_wait is
// not woken promptly by remote arrivals (waits of 2.5-4 us instead of ~0.1), so the
// suspend time is capped with an explicit 64 ns hint.
__device__ __forceinline__ bool mbar_try_wait_cluster(uint64_t* bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 p, [%1], %2, %3;\n\t"
      "selp.u32 %0, 1, 0, p;\n\t}"
      : "=r"(ok)
      : "r"(smem_u32(bar)), "r"(parity), "r"(64u)
      : "memory");
  return ok != 0;
}
__device__ __forceinline__ void mbar_wait_cluster(uint64_t* bar, uint32_t parity) {
  if (mbar_try_wait_cluster(bar, parity)) return;
  const uint64_t t0 = globaltimer();
  while (!mbar_try_wait_cluster(bar, parity)) {
    if (globaltimer() - t0 > 4000000000ull) __trap();
  }
}

// Wait on a barrier completed by tcgen05.commit: CTA-scope acquire for a lone CTA (the
// cluster-scope form compiles to an L1 invalidate, CCTL.IVALL, on every successful wait),
// cluster scope when the commit comes from the CTA pair's leader.
template <bool CLUSTER>
__device__ __forceinline__ void mbar_wait_tc(uint64_t* bar, uint32_t parity) {
  if constexpr (CLUSTER) mbar_wait_cluster(bar, parity);
  else mbar_wait(bar, parity);
}

// warpgroup register reallocation (all threads of the warpgroup execute it)
template <int N>
__device__ __forceinline__ void setmaxnreg_inc() {
  asm volatile("setmaxnreg.inc.sync.aligned.u32 %0;" ::"n"(N));
}
template <int N>
__device__ __forceinline__ void setmaxnreg_dec() {
  asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" ::"n"(N));
}

// ---- tcgen05 --------------------------------------------------------------
__device__ __forceinline__ void tmem_alloc2(uint32_t* smem_dst, uint32_t ncols) {
  asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(smem_dst)),
               "r"(ncols)
               : "memory");
}
__device__ __forceinline__ void tmem_relinquish2() {
  asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
}
__device__ __forceinline__ void tmem_dealloc2(uint32_t taddr, uint32_t ncols) {
  asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(taddr), "r"(ncols) : "memory");
}
// D[tmem] (+)= A[tmem] * B[smem]^T over a CTA pair: M = 256 (128 rows per CTA, A and D
// at the same TMEM address in both), B split along N (N/2 rows per CTA, same smem offset)
__device__ __forceinline__ void mma2_tf32_ts(uint32_t d_tmem, uint32_t a_tmem, uint64_t b_desc, uint32_t idesc,
                                             uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::2.kind::tf32 [%0], [%1], %2, %3, p;\n\t}" ::"r"(d_tmem),
      "r"(a_tmem), "l"(b_desc), "r"(idesc), "r"(accumulate)
      : "memory");
}
// commit of this thread's prior cta_group::2 MMAs to the barrier at the same smem
// offset in both CTAs of the pair
__device__ __forceinline__ void mma_commit2(uint64_t* bar) {
  asm volatile(
      "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
          smem_u32(bar)),
      "h"((uint16_t)0x3)
      : "memory");
}
__device__ __forceinline__ void tmem_alloc(uint32_t* smem_dst, uint32_t ncols) {
  asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(smem_dst)),
               "r"(ncols)
               : "memory");
}
__device__ __forceinline__ void tmem_relinquish() {
  asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
}
__device__ __forceinline__ void tmem_dealloc(uint32_t taddr, uint32_t ncols) {
  asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(taddr), "r"(ncols) : "memory");
}
__device__ __forceinline__ void tc_fence_before() {
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void tc_fence_after() {
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
}
// Warp-collective forms (all 32 lanes call with warp-uniform operands; one elected lane issues):
// uniform operands stay in uniform registers instead of a per-call elect/broadcast loop.
__device__ __forceinline__ void mma_tf32_ts_warp(uint32_t d_tmem, uint32_t a_tmem, uint64_t b_desc, uint32_t idesc,
                                                 uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p, e;\n\t"
      "elect.sync _|e, 0xffffffff;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::tf32 [%0], [%1], %2, %3, p;\n\t}" ::"r"(d_tmem),
      "r"(a_tmem), "l"(b_desc), "r"(idesc), "r"(accumulate)
      : "memory");
}
__device__ __forceinline__ void mma2_tf32_ts_warp(uint32_t d_tmem, uint32_t a_tmem, uint64_t b_desc, uint32_t idesc,
                                                  uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p, e;\n\t"
      "elect.sync _|e, 0xffffffff;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "@e tcgen05.mma.cta_group::2.kind::tf32 [%0], [%1], %2, %3, p;\n\t}" ::"r"(d_tmem),
      "r"(a_tmem), "l"(b_desc), "r"(idesc), "r"(accumulate)
      : "memory");
}
__device__ __forceinline__ void mma_commit_warp(uint64_t* bar) {
  asm volatile(
      "{\n\t.reg .pred e;\n\t"
      "elect.sync _|e, 0xffffffff;\n\t"
      "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t}" ::"r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void mma_commit2_warp(uint64_t* bar) {
  asm volatile(
      "{\n\t.reg .pred e;\n\t"
      "elect.sync _|e, 0xffffffff;\n\t"
      "@e tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;\n\t}" ::"r"(
          smem_u32(bar)),
      "h"((uint16_t)0x3)
      : "memory");
}
// D[tmem] (+)= A[tmem] * B[smem]^T, kind::tf32, M=128, N from idesc, K=8
__device__ __forceinline__ void mma_tf32_ts(uint32_t d_tmem, uint32_t a_tmem, uint64_t b_desc, uint32_t idesc,
                                            uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::tf32 [%0], [%1], %2, %3, p;\n\t}" ::"r"(d_tmem),
      "r"(a_tmem), "l"(b_desc), "r"(idesc), "r"(accumulate)
      : "memory");
}
// D[tmem] (+)= A[smem] * B[smem]^T
__device__ __forceinline__ void mma_tf32_ss(uint32_t d_tmem, uint64_t a_desc, uint64_t b_desc, uint32_t idesc,
                                            uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
      "l"(a_desc), "l"(b_desc), "r"(idesc), "r"(accumulate)
      : "memory");
}
__device__ __forceinline__ void mma_commit(uint64_t* bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(bar))
               : "memory");
}
__device__ __forceinline__ void tmem_st_x4(uint32_t taddr, float a, float b, float c, float d) {
  asm volatile("tcgen05.st.sync.aligned.32x32b.x4.b32 [%0], {%1, %2, %3, %4};" ::"r"(taddr), "r"(__float_as_uint(a)),
               "r"(__float_as_uint(b)), "r"(__float_as_uint(c)), "r"(__float_as_uint(d))
               : "memory");
}
__device__ __forceinline__ void tmem_st_x8(uint32_t taddr, const float (&v)[8]) {
  asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8};" ::"r"(taddr),
               "r"(__float_as_uint(v[0])), "r"(__float_as_uint(v[1])), "r"(__float_as_uint(v[2])),
               "r"(__float_as_uint(v[3])), "r"(__float_as_uint(v[4])), "r"(__float_as_uint(v[5])),
               "r"(__float_as_uint(v[6])), "r"(__float_as_uint(v[7]))
               : "memory");
}
// 16 consecutive columns of this thread's lane
__device__ __forceinline__ void tmem_st_x16(uint32_t taddr, const float (&v)[16]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, "
      "%15, %16};" ::"r"(taddr),
      "r"(__float_as_uint(v[0])), "r"(__float_as_uint(v[1])), "r"(__float_as_uint(v[2])), "r"(__float_as_uint(v[3])),
      "r"(__float_as_uint(v[4])), "r"(__float_as_uint(v[5])), "r"(__float_as_uint(v[6])), "r"(__float_as_uint(v[7])),
      "r"(__float_as_uint(v[8])), "r"(__float_as_uint(v[9])), "r"(__float_as_uint(v[10])), "r"(__float_as_uint(v[11])),
      "r"(__float_as_uint(v[12])), "r"(__float_as_uint(v[13])), "r"(__float_as_uint(v[14])), "r"(__float_as_uint(v[15]))
      : "memory");
}
__device__ __forceinline__ void tmem_wait_st() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }
__device__ __forceinline__ void tmem_ld_x8(uint32_t taddr, float* v) {
  uint32_t r[8];
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
               : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7])
               : "r"(taddr)
               : "memory");
#pragma unroll
  for (int i = 0; i < 8; ++i) v[i] = __uint_as_float(r[i]);
}
__device__ __forceinline__ void tmem_ld_x16(uint32_t taddr, float* v) {
  uint32_t r[16];
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, "
      "%15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]), "=r"(r[8]),
        "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
      : "r"(taddr)
      : "memory");
#pragma unroll
  for (int i = 0; i < 16; ++i) v[i] = __uint_as_float(r[i]);
}
__device__ __forceinline__ void tmem_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }

// tf32 round-to-nearest (ties away): the hi part of the 3xTF32 split
__device__ __forceinline__ float tf32_rna(float x) {
  uint32_t r;
  asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(r) : "f"(x));
  return __uint_as_float(r);
}
// 3xTF32 split on the ALU pipe: hi = x rounded to 10 mantissa bits (half away from
// zero on the magnitude bits, == cvt.rna for finite x), lo = x - hi exactly in fp32
// (the tensor core reads lo's top 19 bits; the dropped part is < 2^-21 |x|).
__device__ __forceinline__ void split_tf32(float x, float& hi, float& lo) {
  hi = __uint_as_float((__float_as_uint(x) + 0x1000u) & 0xFFFFE000u);
  lo = x - hi;
}

// UMMA shared-memory descriptor, K-major, SWIZZLE_NONE (canonical interleaved
// layout: 8-row x 16-byte core matrices; SBO = byte stride between 8-row
// groups, LBO = byte stride between the two 16-byte K halves).
__device__ __forceinline__ uint64_t umma_desc_kmajor_noswizzle(uint32_t smem_addr, uint32_t lbo, uint32_t sbo) {
  uint64_t d = 0;
  d |= (uint64_t)((smem_addr >> 4) & 0x3FFFu);
  d |= (uint64_t)((lbo >> 4) & 0x3FFFu) << 16;
  d |= (uint64_t)((sbo >> 4) & 0x3FFFu) << 32;
  d |= (uint64_t)1 << 46;  // descriptor version (sm_100)
  return d;                // base offset 0, lbo mode 0, layout type 0 (no swizzle)
}
// Instruction descriptor for kind::tf32: D f32, A/B tf32, both K-major, M=128
__host__ __device__ constexpr uint32_t idesc_tf32(int M, int N) {
  return (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}
#endif  // __CUDACC__

}  // namespace i2cw
