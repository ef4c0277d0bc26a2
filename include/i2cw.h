/*
 * i2cw.h — C ABI of the B200-native fused Im2col-Winograd convolution
 * (Zhang, Zhang, Xu, Yan, Wang, "Im2col-Winograd: An Efficient and Flexible
 * Fused-Winograd Convolution for NHWC Format on GPUs", ICPP '24 = PAPER.md).
 *
 * Operation (§4.1, Table 1): a unit-stride
 * 2D convolution of an fp32 NHWC input X[N][H][W][C] ("ifms", IH=H, IW=W, IC=C)
 * with fp32 filters W[K][R][S][C] (OC=K, FH=R, FW=S), symmetric zero padding
 * (pad_h, pad_w; implicit), giving Y[N][P][Q][K]:
 *
 *   y[n][p][q][k] = sum_{r<R} sum_{s<S} sum_{c<C} x[n][p-pad_h+r][q-pad_w+s][c] * w[k][r][s][c]
 *   P = H + 2*pad_h - R + 1,   Q = W + 2*pad_w - S + 1       (cross-correlation)
 *
 * computed as Gamma_alpha(m, S): per filter row r and channel c a 1D Winograd
 * F(m, S) along W, accumulated over (r, c) in the Winograd
 * domain and output-transformed once (A^T applied after the sum, by linearity).
 * Filter widths S = 2..9 are supported; R >= 1 is
 * unrestricted (the method restricts only FW).
 *
 * Conventions for every entry point:
 *  - Pointers x, w, u, y are DEVICE pointers unless the name ends in _host;
 *    caller-owned, dense (NHWC / KRSC as documented), 16-byte aligned.
 *  - Asynchronous: work is enqueued on `stream` (a cudaStream_t; NULL = legacy
 *    default stream) and the call returns without a host sync; kernel faults
 *    surface at the caller's next synchronisation.
 *  - The library keeps no global mutable state except a lazily created
 *    stream-ordered workspace pool (see i2cw_conv2d_nhwc), a memo of launch plans
 *    and transform tables (pure functions of the dimensions), and two copy streams
 *    per device for i2cw_conv2d_nhwc_host.
 *  - A conv/deconv call enqueues the filter transform, then one fused launch per
 *    K-chunk (a K loop longer than 256 k-steps for alpha <= 8 / 128 for alpha = 12,
 *    one k-step = 8 channels x 1 filter row, runs as several launches whose partial
 *    sums are added into y in order: the tcgen05 fp32 accumulator truncates once per
 *    MMA, so bounding the accumulation length bounds the error for any C), and may
 *    enqueue a small zeroing kernel on part of y before the first fused launch (the
 *    "split tail" of the persistent schedule, whose two Winograd passes both
 *    reduce-add into y). The zeroing kernel is a programmatic dependent of the
 *    previous kernel and touches y only after that kernel's grid has completed unless
 *    that kernel is the library's own filter transform. Results are bitwise
 *    deterministic run to run.
 *  - fp32 in / fp32 out. The per-point channel contraction runs on the tcgen05
 *    tensor cores in 3xTF32 (hi*hi + hi*lo + lo*hi, V split to nearest tf32), which
 *    keeps |y - y_exact| <= 1e-4 * sum|x|*|w| per element (BASELINE.json north_star);
 *    i2cw_conv2d_nhwc_prec offers a 1xTF32 mode with a looser stated bound.
 *  - No CPU fallback: on a machine without a B200 the calls return I2CW_ECUDA.
 *
 * Return codes (i2cw_status): 0 on success, negative on error; nothing is
 * enqueued when an error is returned before launch.
 *   I2CW_EINVAL       null pointer, a dimension <= 0, pad < 0, P or Q < 1,
 *                     misaligned pointer, tag mismatch on a pre-transformed filter.
 *   I2CW_EUNSUPPORTED S outside [2, 9]; C % 4 != 0 or K % 4 != 0 (TMA global strides
 *                     and 16-byte vector stores need 16-byte rows); a shape whose
 *                     tile plan exceeds the on-chip budget or a TMA box limit.
 *   I2CW_ECUDA        a CUDA runtime error (no device, launch failure, OOM).
 */
#ifndef I2CW_H_
#define I2CW_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#if defined(__GNUC__)
#define I2CW_API __attribute__((visibility("default")))
#else
#define I2CW_API
#endif

typedef struct CUstream_st* i2cw_stream_t; /* == cudaStream_t */

typedef enum {
  I2CW_OK = 0,
  I2CW_EINVAL = -1,
  I2CW_EUNSUPPORTED = -2,
  I2CW_ECUDA = -3
} i2cw_status;

/* Human-readable text for a status code (static storage). */
I2CW_API const char* i2cw_status_string(int status);

/* Library/ABI version: major*10000 + minor*100 + patch. */
I2CW_API int i2cw_version(void);

/*
 * Forward convolution (see the definition above).
 *   x: [N][H][W][C] fp32, w: [K][R][S][C] fp32 (KRSC, the paper's OC x FH x FW x IC),
 *   y: [N][P][Q][K] fp32 (written, never read).
 * The filter transform U = G w runs as a first launch
 * into a filter-sized workspace taken from a stream-ordered pool
 * (cudaMallocAsync on `stream`, cached after first use); the fused kernel itself
 * uses no Winograd-domain workspace.
 */
I2CW_API int i2cw_conv2d_nhwc(int N, int H, int W, int C, int K, int R, int S, int pad_h, int pad_w,
                     const float* x, const float* w, float* y, i2cw_stream_t stream);

/*
 * Unit-stride deconvolution (transposed convolution, the backward-data pass of
 * the conv whose filter is w): the 180-degree filter rotation
 * is folded into the filter transform, w is used without rearrangement.
 *   x: [N][H][W][C] fp32, w: [C][R][S][K] fp32 (the KRSC filter of the forward
 *   conv with K'=C outputs and C'=K inputs), y: [N][P][Q][K] fp32,
 *   y[n][p][q][k] = sum_{c<C,r<R,s<S} x[n][p+pad_h-r][q+pad_w-s][c] * w[c][r][s][k]
 *   P = H + R - 1 - 2*pad_h,  Q = W + S - 1 - 2*pad_w.
 * Equals torch conv_transpose2d(x, w.permute(0,3,1,2), padding=pad) in NHWC, and
 * conv(x, w', R-1-pad) with w'[k][r][s][c] = w[c][R-1-r][S-1-s][k].
 */
I2CW_API int i2cw_deconv2d_nhwc(int N, int H, int W, int C, int K, int R, int S, int pad_h, int pad_w,
                       const float* x, const float* w, float* y, i2cw_stream_t stream);

/*
 * Precision modes ("1xTF32 with looser tolerance").
 *   I2CW_PREC_3XTF32 (default of every other call): hi*hi + hi*lo + lo*hi tf32 products,
 *     |y - y_exact| <= 1e-4 * sum|x||w| per element.
 *   I2CW_PREC_1XTF32: one tf32 product per Winograd point (V and U rounded to nearest tf32,
 *     a third of the tensor work); tolerance |y - y_exact| <= 1e-2 * sum|x||w| (each product's
 *     relative error <= 2^-10, amplified <= ~10x by the alpha <= 12 transforms; measured max
 *     3.1e-3, profiles/r02_precision.txt; reading R17).
 * i2cw_conv2d_nhwc_prec: the 2D conv (is_deconv = 0, w KRSC) or deconv (is_deconv = 1, w CRSK)
 * with the given precision; otherwise as i2cw_conv2d_nhwc / i2cw_deconv2d_nhwc.
 * EINVAL for an unknown precision.
 */
#define I2CW_PREC_3XTF32 0
#define I2CW_PREC_1XTF32 1
I2CW_API int i2cw_conv2d_nhwc_prec(int precision, int is_deconv, int N, int H, int W, int C, int K, int R, int S,
                                   int pad_h, int pad_w, const float* x, const float* w, float* y,
                                   i2cw_stream_t stream);

/*
 * 3D convolution (Im2col-Winograd "can be applied to ND convolution, by
 * expanding Stage1 Im2col to ND, while remaining Stage2 unchanged"): the 1D F(m, S) Winograd
 * runs along W exactly as in 2D; the K loop of the channel contraction runs over (c, depth tap
 * t, filter row r).
 *   x: [N][D][H][W][C] fp32, w: [K][T][R][S][C] fp32, y: [N][OD][P][Q][K] fp32,
 *   y[n][od][p][q][k] = sum_{t<T,r<R,s<S,c<C} x[n][od-pad_d+t][p-pad_h+r][q-pad_w+s][c] * w[k][t][r][s][c]
 *   OD = D + 2*pad_d - T + 1 (P, Q as in 2D), zero padding.
 * i2cw_deconv3d_ndhwc: the unit-stride transposed 3D conv, w: [C][T][R][S][K],
 *   y[n][od][p][q][k] = sum_{c,t,r,s} x[n][od+pad_d-t][p+pad_h-r][q+pad_w-s][c] * w[c][t][r][s][k],
 *   OD = D + T - 1 - 2*pad_d (rotation of all three taps folded into the filter transform).
 * Same conventions, errors and tolerance as the 2D calls; S in [2, 9], T, R >= 1; the 3D path
 * always uses the default alpha = 8 (S <= 7) / 12 (S = 8, 9) transforms.
 */
I2CW_API int i2cw_conv3d_ndhwc(int N, int D, int H, int W, int C, int K, int T, int R, int S, int pad_d, int pad_h,
                               int pad_w, const float* x, const float* w, float* y, i2cw_stream_t stream);
I2CW_API int i2cw_deconv3d_ndhwc(int N, int D, int H, int W, int C, int K, int T, int R, int S, int pad_d, int pad_h,
                                 int pad_w, const float* x, const float* w, float* y, i2cw_stream_t stream);

/*
 * NCHW layout adapters: PyTorch's default layouts.
 *   i2cw_conv2d_nchw:   x [N][C][H][W], w [K][C][R][S] (OIHW), y [N][K][P][Q]
 *   i2cw_deconv2d_nchw: x [N][C][H][W], w [C][K][R][S] (conv_transpose2d weight), y [N][K][P][Q]
 * Same operation, padding, errors and tolerance as the NHWC calls. x, w are transposed to
 * NHWC / KRSC (CRSK) into stream-ordered pool workspaces by a tiled transpose kernel, the NHWC
 * path runs, and y is transposed back: one extra HBM read + write of x, w and y per call.
 */
I2CW_API int i2cw_conv2d_nchw(int N, int C, int H, int W, int K, int R, int S, int pad_h, int pad_w, const float* x,
                              const float* w, float* y, i2cw_stream_t stream);
I2CW_API int i2cw_deconv2d_nchw(int N, int C, int H, int W, int K, int R, int S, int pad_h, int pad_w,
                                const float* x, const float* w, float* y, i2cw_stream_t stream);

/*
 * Pre-transformed filters (the paper's '*' variant, PAPER.md:3951-3952, 4001-4004:
 * transform once, reuse across calls).
 * Argument order (K, C, R, S) follows SURVEY.md §8(b): K = output channels, C = input
 * channels of the call the filter is for (for a deconvolution: the K and C passed to
 * i2cw_deconv2d_nhwc, i.e. w is [C][R][S][K]).
 * i2cw_filter_bytes: bytes of the transformed filter u for these dims
 *   (a 256-byte tag + 2 * alpha(S) * ceil(K/NT)*NT * R * ceil8(C) * 4), or 0 if the
 *   shape is unsupported.
 * i2cw_filter_transform: u = tag || U_hi/U_lo in the fused kernel's staging layout.
 *   is_deconv = 0: w is [K][R][S][C]; is_deconv = 1: w is [C][R][S][K].
 * The _pretransformed calls take u instead of w; a u produced for other dims or
 * the other is_deconv value is rejected with I2CW_EINVAL. Validation: a host-side copy of
 * the tag is kept for every u written by i2cw_filter_transform in this process; any other
 * u (cloned, loaded, another process) or a registry mismatch has its device tag read with a
 * small device-to-host copy on `stream` (which synchronises that stream). The fused kernel
 * also checks the device tag itself and traps (a launch failure at the next sync) if it
 * disagrees with the call, so a stale host copy can never run a mismatched u silently.
 * u must stay alive and unmodified until the calls that read it have completed.
 */
I2CW_API size_t i2cw_filter_bytes(int K, int C, int R, int S);
I2CW_API int i2cw_filter_transform(int K, int C, int R, int S, int is_deconv, const float* w, void* u,
                          i2cw_stream_t stream);
I2CW_API int i2cw_conv2d_nhwc_pretransformed(int N, int H, int W, int C, int K, int R, int S, int pad_h, int pad_w,
                                    const float* x, const void* u, float* y, i2cw_stream_t stream);
I2CW_API int i2cw_deconv2d_nhwc_pretransformed(int N, int H, int W, int C, int K, int R, int S, int pad_h,
                                      int pad_w, const float* x, const void* u, float* y,
                                      i2cw_stream_t stream);

/*
 * End-to-end call with HOST buffers (pinned or pageable): copies x and w to the
 * device, runs the conv (is_deconv = 0) or deconv (is_deconv = 1) on `stream`,
 * copies y back, and synchronises `stream` before returning. Device buffers come
 * from the stream-ordered pool. Same shapes and semantics as the device calls.
 * The batch is processed in up to 8 image chunks: host->device copies (one internal
 * non-blocking stream) and device->host copies (another) overlap the chunks'
 * kernels on `stream`; with pinned buffers both PCIe directions run concurrently.
 */
I2CW_API int i2cw_conv2d_nhwc_host(int is_deconv, int N, int H, int W, int C, int K, int R, int S, int pad_h,
                          int pad_w, const float* x_host, const float* w_host, float* y_host,
                          i2cw_stream_t stream);

/* Select the device used by i2cw_conv2d_nhwc_host (the device-pointer calls
 * follow the device that owns x). Returns I2CW_ECUDA for an invalid device. */
I2CW_API int i2cw_set_device(int device);

/*
 * Host-side introspection (no GPU needed).
 * i2cw_plan: the Winograd choice for filter width S and C input channels: m outputs,
 *   alpha = m+S-1 states, and the alpha = 16 point set (0 paper, 1 alt; reading R7).
 *   S = 2: Gamma4(3,2); S = 3: Gamma8(6,3) (Gamma4(2,3) for C >= 256 only when the strip kernel
 *   is disabled with I2CW_STRIP=0); S = 4..7: Gamma8; S = 8, 9: alpha = 12 (measured selection,
 *   DESIGN.md reading R8). The 3D and 1xTF32 calls use alpha = 8 for S = 2, 3. The planner runs
 *   the strip kernel or the base kernel for a call; both read the same U layout
 *   produced by i2cw_filter_transform and give results within the same bound. Returns
 *   I2CW_EUNSUPPORTED for S outside [2, 9], EINVAL for C <= 0.
 * i2cw_transform_matrices_rational: the exact Cook-Toom matrices of F(m, r)
 *   (§5.3, Figure 5) as int64 numerator/denominator
 *   pairs, row-major: AT (m x alpha), G (alpha x r), BT (alpha x alpha), with
 *   alpha = m + r - 1 <= 16 and point_set 0 (paper) or 1 (alt, alpha = 16 only).
 *   Each output array must hold the matrix's element count; returns I2CW_EINVAL
 *   on bad arguments and I2CW_EUNSUPPORTED if an entry does not fit in int64.
 */
I2CW_API int i2cw_plan(int S, int C, int* m, int* alpha, int* point_set);
I2CW_API int i2cw_transform_matrices_rational(int m, int r, int point_set, int64_t* at_num, int64_t* at_den,
                                     int64_t* g_num, int64_t* g_den, int64_t* bt_num, int64_t* bt_den);

#ifdef __cplusplus
}
#endif
#endif /* I2CW_H_ */
