/*
 * qconv.h -- C ABI of the B200 (sm_100a) 4/8-bit quantized convolution library
 * (libqconv.so, built from paper_conf_icpp_hanhyylhgwwlq20_b200/csrc).
 *
 * The hot path of Han, Hu et al., "Extremely Low-bit Convolution Optimization
 * for Quantized Neural Network on Modern Computer Architectures" (ICPP'20),
 * section 4: quantization, implicit-GEMM convolution on tensor cores
 * (Alg.2) with bias + re-quantization fused into the
 * epilogue (P:L223 l.15) and ReLU folded into the truncation range
 * (P:L265).  "P:Lnnn" = line nnn of the paper text; "Zn"/"R1" are
 * the readings listed in DESIGN.md section 3.
 *
 * Conventions for every entry point
 *  - Plain pointers and sizes only.  "device" pointers are CUDA device
 *    allocations owned by the caller; "host" pointers are host memory owned by
 *    the caller.  The library never allocates device memory and never frees a
 *    caller buffer.
 *  - `stream` is a cudaStream_t passed as void* (NULL = legacy default
 *    stream).  Device work is enqueued asynchronously on it; the call returns
 *    after enqueueing.  Argument errors are detected on the host and returned
 *    synchronously before anything is enqueued; a failed launch returns
 *    QC_ERR_CUDA (qconv_last_cuda_error() gives the CUDA error code).
 *  - No call throws; all calls are reentrant and thread-safe (the only global
 *    state is a lazily resolved driver entry point).
 *  - Layouts: activations NHWC (C contiguous), weights KRSC (R*S*C
 *    contiguous per output channel), outputs NHWC [N,P,Q,K].  4-bit tensors
 *    pack two elements per byte, element 2j in the low nibble of byte j of the
 *    row (reading Z7); signed 4-bit values are two's complement nibbles.
 *  - P = (H + 2*pad_h - dil_h*(R-1) - 1)/stride_h + 1, Q likewise.
 */
#ifndef QCONV_H_
#define QCONV_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    QC_OK = 0,
    QC_ERR_INVALID_ARG = 1,    /* malformed shape / dtype / range / NULL pointer */
    QC_ERR_UNSUPPORTED = 2,    /* well-formed but outside what the GPU path implements */
    QC_ERR_OVERFLOW_RISK = 3,  /* int32 accumulation could overflow for this shape/dtype */
    QC_ERR_MISALIGNED = 4,     /* a device pointer is not 16-byte aligned */
    QC_ERR_WORKSPACE = 5,      /* workspace missing or smaller than qconv2d_workspace_size */
    QC_ERR_CUDA = 6            /* a CUDA driver/runtime call failed */
} qc_status;

/* QC_F32_OUT / QC_BF16_OUT: dequantized outputs of qconv2d_forward_dequant only. */
typedef enum { QC_U4 = 0, QC_S4 = 1, QC_U8 = 2, QC_S8 = 3, QC_S32 = 4, QC_F32_OUT = 5,
               QC_BF16_OUT = 6 } qc_dtype;
typedef enum { QC_F32 = 0, QC_BF16 = 1 } qc_ftype;

/* Re-quantization rounding (qconv_desc.rounding).
 *  QC_ROUND_SINGLE (reading Z3): t = floor((acc*m + 2^(n-1)) / 2^n), one rounding, ties
 *                   toward +inf.
 *  QC_ROUND_TFLITE (reading Z15; the gemmlowp/TFLite scheme, "same quantization
 *                   scheme", gemmlowp [14] P:L45): with ls = max(0, 31-n), rs = max(0, n-31),
 *                   a = sat32(acc * 2^ls), h = SaturatingRoundingDoublingHighMul(a, m)
 *                   = floor((a*m + 2^30) / 2^31) (INT32_MAX for a = m = INT32_MIN),
 *                   t = RoundingDivideByPOT(h, rs) (nearest, ties away from zero). */
typedef enum { QC_ROUND_SINGLE = 0, QC_ROUND_TFLITE = 1 } qc_rounding;

/*
 * qconv_quantize_pack -- quantization step of the QNN layer sequence,
 * reading Z4: for every element, q = clamp(rne(x * fl32(1/scale)) + zero_point,
 * qmin(yt), qmax(yt)), computed as one IEEE fp32 multiply then round-to-
 * nearest-even (matches torch.quantize_per_tensor); NaN -> zero_point.
 *   x          device, [npix, c] fp32 or bf16 (xt), npix = N*H*W
 *   y          device, [npix, c_pad] packed yt in {U4,S4,U8,S8}; channels
 *              c..c_pad-1 are written with zero_point (channel padding)
 *   scale      > 0 and finite; zero_point inside the yt range
 * Errors: INVALID_ARG (npix < 0, c < 1, c_pad < c, 4-bit with odd c_pad, bad
 * scale/zero point/dtype, NULL), MISALIGNED (x or y not 16-byte aligned).
 */
qc_status qconv_quantize_pack(const void *x, qc_ftype xt, int64_t npix, int32_t c,
                              int32_t c_pad, float scale, int32_t zero_point, qc_dtype yt,
                              void *y, void *stream);

/*
 * qconv_requant_params -- host only, synchronous, deterministic (reading R1;
 * the paper only says "re-quantize").  For k output channels:
 *   M_k = fl64(fl64(in_scale) * fl64(w_scale[k])) / fl64(out_scale);
 *   (f, e) = frexp(M_k); m = round-half-up(f * 2^31); if m == 2^31 {m = 2^30; e++}
 *   multiplier[k] = m in [2^30, 2^31), shift[k] = 31 - e in [1, 62];
 *   M_k == 0 gives (0, 31).
 *   w_scale, multiplier, shift: host arrays of length k.
 * Errors: INVALID_ARG (non-positive / non-finite scales, k < 1, NULL, or a
 * shift outside [1, 62]).
 */
qc_status qconv_requant_params(float in_scale, const float *w_scale, float out_scale,
                               int32_t k, int32_t *multiplier, int32_t *shift);

/* Convolution descriptor (host struct, read during the call only). */
typedef struct {
    int32_t n, h, w, c, k, r, s;          /* X: [n,h,w,c] NHWC; W: [k,r,s,c] KRSC */
    int32_t stride_h, stride_w;           /* 1..8 */
    int32_t pad_h, pad_w;                 /* >= 0 (zero padding = real zero, Z2) */
    int32_t dil_h, dil_w;                 /* >= 1 */
    qc_dtype x_t, w_t, y_t;               /* x_t, w_t in {U4,S4,U8,S8}: equal bit widths, or
                                             8-bit activations with 4-bit weights (A8W4);
                                             y_t in {U4,S4,U8,S8,S32} (qconv2d_forward) or
                                             {F32_OUT,BF16_OUT} (qconv2d_forward_dequant) */
    int32_t x_zero;                       /* per-tensor activation zero point (Z1) */
    const int32_t *w_zero;                /* device int32 [k] per-output-channel weight zero
                                             points (Z1), or NULL (= 0).  Read by the device
                                             only: any values inside the w_t range */
    int32_t w_prepared;                   /* 1: `w` is the output of qconv_prepare_weights */
    int32_t y_zero;                       /* output zero point (integer outputs except S32) */
    int32_t clamp_lo, clamp_hi;           /* truncation range inside the y_t range; ReLU:
                                             clamp_lo = max(qmin, y_zero) (Z5);
                                             ignored for S32 / float outputs */
    int32_t rounding;                     /* qc_rounding (requantized outputs) */
    int32_t relu;                         /* float outputs: y = (y > 0 ? y : +0) */
} qconv_desc;

/*
 * Channel counts the kernels take directly: c % 32 == 0 (any width), or c == 16 at 8 bits
 * (two filter taps per 32-byte K step).  Any other c is handled inside the library, with no
 * change of the result (the same products, regrouped or padded with zero terms):
 *  - stride 2, dilation 1 and 4*c <= 16 (the C = 3 / C = 4 image stems): the 2x2
 *    space-to-depth form  X2[n,i,j,(2b+b')*c+cc] = x[n, 2i+b-pad_h, 2j+b'-pad_w, cc]
 *    (x_zero outside), W2[k,a,a',(2b+b')*c+cc] = w[k, 2a+b, 2a'+b', cc] (0 beyond r, s):
 *    a stride-1, unpadded ceil(r/2) x ceil(s/2) conv over 16 byte-coded channels;
 *  - otherwise the channels are padded to 16 (8-bit, c < 16) or to a multiple of 32 with
 *    x_zero activation codes and zero weights.
 * The rearranged activations go to the workspace (qconv2d_workspace_size) on every call; the
 * rearranged weights are what qconv_prepare_weights produces for such a descriptor.
 */

/*
 * qconv_prepare_weights -- once-per-layer weight preparation (the paper's
 * "pre-processing"): KRSC weights of dtype d->w_t are brought to the
 * kernel's operand layout (sm_100 tensor cores have no 4-bit integer MMA).
 *  - 8-bit weights, c % 32 == 0 or c == 16: copied (k*r*s*c bytes).
 *  - 4-bit weights with 4-bit activations: "nibble-plane" int8 KRSC -- within each
 *    32-channel group of a (k,r,s) row the 16 even channels come first as 16*w, then the
 *    16 odd channels as w, matching the kernel's on-chip activation widening -- followed,
 *    16-byte aligned, by int32 wsum[k] = sum over (r,s,c) of w (the correction of signed
 *    4-bit activations).
 *  - 4-bit weights with 8-bit activations (A8W4): sign/zero-extended int8 KRSC.
 *  - other channel counts: the space-to-depth or channel-padded weights (see above),
 *    then as before.
 * The layout is opaque to callers: only qconv2d_forward / qconv2d_forward_dequant with
 * w_prepared = 1 read it.  qconv_prepared_weight_bytes(d) gives its size.
 *   w       device, packed KRSC (d->w_t)
 *   w_prep  device, >= qconv_prepared_weight_bytes(d) bytes
 * Errors: INVALID_ARG, UNSUPPORTED, MISALIGNED, CUDA.
 */
size_t qconv_prepared_weight_bytes(const qconv_desc *d);
qc_status qconv_prepare_weights(const qconv_desc *d, const void *w, void *w_prep, void *stream);

/*
 * qconv2d_workspace_size -- device workspace bytes qconv2d_forward needs for this
 * descriptor (0 for the plain 4/8-bit layers of ResNet-50 / VGG with prepared or 8-bit
 * weights).  Non-zero for: unprepared weights that need preparation (4-bit, A8W4, other
 * channel counts), rearranged activations (c not taken directly, see above), x_zero != 0
 * (zero-point border table, k*(r+1)*(s+1) int32) and w_zero != NULL (per-pixel activation
 * sums).  Returns 0 for an invalid descriptor.
 */
size_t qconv2d_workspace_size(const qconv_desc *d);

/*
 * qconv2d_forward -- y = requant(conv(x - x_zero, w - w_zero) + bias) (Alg.2).
 * Per output (n,p,q,k), with acc = sum over in-bounds taps (r,s) and c of
 * (x[n, p*sh-ph+r*dh, q*sw-pw+s*dw, c] - x_zero) * (w[k,r,s,c] - w_zero[k]) + bias[k]:
 *   y_t == S32 : y = acc
 *   otherwise  : t = rounding(acc, multiplier[k], shift[k])   (qc_rounding, Z3 / Z15)
 *                y = min(clamp_hi, max(clamp_lo, t + y_zero))  (Z5)
 * Domain of the per-channel device data: multiplier any int32 (qconv_requant_params gives
 * [2^30, 2^31) or 0), shift in [1, 62]; a shift outside [1, 62] gives undefined bytes.
 * Contract (the paper's 32-bit accumulator): |acc| < 2^31 for every output.
 * The host checks the dtype-range bound r*s*c*max|x-x_zero|*max|w| < 2^31 (else
 * OVERFLOW_RISK) -- for 4-bit activations, whose on-chip widening accumulates 16x the
 * sum, r*s*c*15*max|w| < 2^26 -- and keeping acc + bias (and the w_zero terms) inside int32
 * is the caller's duty (device data is not read on the host).  Every supported
 * configuration gives the same bytes (the integer result is unique); which kernel runs
 * (im2col, CTA-pair, halo, channel-major; see qconv_debug_plan) is an internal choice.
 *   x          device, packed NHWC (d->x_t)
 *   w          device, packed KRSC (d->w_t) or prepared (d->w_prepared = 1)
 *   bias       device int32 [k] or NULL (= 0)
 *   multiplier, shift   device int32 [k]; may be NULL only for y_t == S32
 *   y          device, NHWC [n,p,q,k] packed y_t
 *   workspace  device, >= qconv2d_workspace_size(d) bytes (NULL if 0)
 * Errors: INVALID_ARG (also a float y_t: use qconv2d_forward_dequant), UNSUPPORTED
 * (4-bit activations with 8-bit weights; 4-bit y_t with odd k; pad/dilation beyond the
 * TMA im2col corner range; stride > 8), OVERFLOW_RISK, MISALIGNED, WORKSPACE, CUDA.
 */
qc_status qconv2d_forward(const qconv_desc *d, const void *x, const void *w,
                          const int32_t *bias, const int32_t *multiplier, const int32_t *shift,
                          void *y, void *workspace, size_t ws_bytes, void *stream);

/*
 * qconv2d_forward_dequant -- fusion of convolution and dequantization (section
 * 4.4; reading Z16): the int32 result is converted to fp32 in the epilogue, with no
 * integer store.  With acc as in qconv2d_forward (bias included):
 *   y = fl32(fl32(acc) * scale[k])            (int32 -> fp32 and the product both RNE)
 *   d->relu: y = (y > 0 ? y : +0)              (ReLU fusion)
 *   d->y_t == QC_BF16_OUT: y rounded to bfloat16, nearest even.
 *   scale   device float [k], normally fl32(s_x * s_w[k])
 *   y       device, NHWC [n,p,q,k] fp32 or bf16
 * Other arguments and errors as qconv2d_forward (y_t must be F32_OUT or BF16_OUT).
 */
qc_status qconv2d_forward_dequant(const qconv_desc *d, const void *x, const void *w,
                                  const int32_t *bias, const float *scale, void *y,
                                  void *workspace, size_t ws_bytes, void *stream);

/*
 * qconv2d_forward_quantize -- the quantization step fused with the convolution (P:L257,
 * P:L263): float activations in, y = qconv2d_forward(d, q(x), ...) out, where q quantizes
 * every element with reading Z4 (one fp32 multiply by fl32(1/in_scale), round to nearest even,
 * + d->x_zero, clamp to the d->x_t code range; NaN -> x_zero).
 *   x         device, fp32 or bf16 (xt) NHWC [n, h, w, c] with the true channel count
 *   in_scale  > 0 and finite
 *   other arguments as qconv2d_forward; workspace >= qconv2d_quantize_workspace_size(d, xt)
 * The image stem (stride 2, dilation 1, 4*c <= 16, fp32, x_zero = 0, no w_zero, w*c % 4 == 0,
 * w*c <= 1024: the ResNet / VGG C = 3 stem) runs as ONE kernel: the TMA loads the fp32 rows and
 * the kernel's converter warps quantize them straight into its space-to-depth operand tile
 * (no code tensor in global memory).  Any other descriptor quantizes into the workspace and
 * then runs qconv2d_forward (two launches, same bytes).
 * Errors: as qconv2d_forward; UNSUPPORTED also for 4-bit x_t with odd c outside the fused case.
 */
size_t qconv2d_quantize_workspace_size(const qconv_desc *d, qc_ftype xt);
qc_status qconv2d_forward_quantize(const qconv_desc *d, const void *x, qc_ftype xt, float in_scale,
                                   const void *w, const int32_t *bias, const int32_t *multiplier,
                                   const int32_t *shift, void *y, void *workspace, size_t ws_bytes,
                                   void *stream);

/*
 * Launch plans and the per-shape tile search (the paper's "auto-search ... choose the
 * best ones through profile runs", section 5.1).
 *   kernel : QC_KERNEL_IM2COL   im2col implicit GEMM, one CTA per 128-pixel tile
 *            QC_KERNEL_PAIR     im2col on a 2-CTA cluster (tcgen05 cta_group::2, M = 256)
 *            QC_KERNEL_HALO     stride-1 halo tiles, weights resident in shared memory
 *            QC_KERNEL_CHANNEL  1x1 convs, channel-major (output channels on TMEM lanes)
 *            QC_KERNEL_HALO_T   stride-1 halo tiles, channel-major (K = 64 output channels on
 *                               TMEM lanes, up to 256 pixels per tile)
 *   bn     : output channels per tile (IM2COL/PAIR: 16..256; CHANNEL: 64 or 128; HALO: K)
 * qconv_debug_plan fills every field of the plan qconv2d_forward would launch for `d`
 * (after any qconv_plan_set choice); the pre-kernels (weight preparation, activation
 * rearrangement, zero-point tables) are listed in `prologue` as a bit mask
 * (1 weights, 2 activations, 4 x_zero table, 8 w_zero sums).
 * qconv_plan_set records a choice (kernel, bn; other fields ignored) for descriptors equal
 * to `d` in every field (process-wide, thread-safe); an ineligible choice is rejected with
 * UNSUPPORTED.  choice == NULL removes it.  qconv_plan_clear() removes all choices.
 * qconv_plan_candidates writes up to `cap` eligible (kernel, bn) choices for `d` and
 * returns how many exist.
 * qconv_autotune times every candidate (`iters` launches each, CUDA events on `stream`,
 * synchronous), records the fastest with qconv_plan_set and returns it in `best` and its
 * mean time in `best_us`.  It writes `y` (every candidate gives the same bytes).
 */
typedef enum { QC_KERNEL_AUTO = 0, QC_KERNEL_IM2COL = 1, QC_KERNEL_PAIR = 2, QC_KERNEL_HALO = 3,
               QC_KERNEL_CHANNEL = 4, QC_KERNEL_HALO_T = 5 } qc_kernel;
typedef struct {
    int32_t kernel;           /* qc_kernel */
    int32_t bn;               /* output channels per tile */
    int32_t bm;               /* output pixels per tile (per CTA pair for PAIR) */
    int32_t stages;           /* shared-memory pipeline depth */
    int32_t grid, threads;    /* launch shape (CTAs, threads per CTA) */
    int32_t num_tiles;
    int32_t smem_bytes, tmem_cols;
    int32_t prologue;         /* pre-kernel mask, see above */
    int32_t epilogue_mode;    /* 0 fast, 1 mid, 2 general: the mode all channels can take */
    int32_t reserved[5];
} qconv_plan;

qc_status qconv_debug_plan(const qconv_desc *d, qconv_plan *out);
/* The plan qconv2d_forward_quantize launches (prologue bit 16: a separate quantize launch). */
qc_status qconv_debug_plan_quantize(const qconv_desc *d, qc_ftype xt, qconv_plan *out);
qc_status qconv_plan_set(const qconv_desc *d, const qconv_plan *choice);
void qconv_plan_clear(void);
int32_t qconv_plan_candidates(const qconv_desc *d, qconv_plan *out, int32_t cap);
qc_status qconv_autotune(const qconv_desc *d, const void *x, const void *w, const int32_t *bias,
                         const int32_t *multiplier, const int32_t *shift, void *y,
                         void *workspace, size_t ws_bytes, void *stream, int32_t iters,
                         qconv_plan *best, float *best_us);

/*
 * Space-to-depth form of a stride-2 convolution (the ResNet/VGG C=3 stem), exposed so the
 * fp32 quantization can write the rearranged codes directly.  qconv2d_forward applies the
 * same rearrangement internally (above); these calls let the caller fuse it with the
 * quantization step instead:
 *   qconv_s2d_desc          -> the transformed descriptor (x_t/w_t = byte containers,
 *                              w_prepared = 1); pass it to qconv2d_forward
 *   qconv_quantize_pack_s2d -> fused quantization (Z4, zero point d->x_zero, code range
 *                              of d->x_t) + rearrangement of fp32/bf16 NHWC x into X2
 *                              (device, qconv_s2d_desc(d).{n,h,w,c} bytes)
 *   qconv_prepare_weights_s2d -> W2 (device int8, qconv_prepared_weight_bytes_s2d bytes)
 * Codes are stored one per byte (4-bit codes sign/zero-extended) so C2 = 16 meets the
 * 16-byte TMA stride rule.
 * Errors: INVALID_ARG, UNSUPPORTED (stride != 2 or dilation != 1), MISALIGNED, CUDA.
 */
qc_status qconv_s2d_desc(const qconv_desc *d, qconv_desc *out);
qc_status qconv_quantize_pack_s2d(const qconv_desc *d, const void *x, qc_ftype xt, float scale,
                                  void *y, void *stream);
size_t qconv_prepared_weight_bytes_s2d(const qconv_desc *d);
qc_status qconv_prepare_weights_s2d(const qconv_desc *d, const void *w, void *w_prep, void *stream);

/* Human-readable status; static storage, never NULL. */
const char *qconv_status_string(qc_status s);

/* CUDA error code (cudaError_t as int) of the last QC_ERR_CUDA on this thread. */
int qconv_last_cuda_error(void);

/* Library version (major*10000 + minor*100 + patch). */
int qconv_version(void);

/*
 * Diagnostics (used by the parity tests, not on the hot path):
 * qconv_debug_im2col_tile loads one 128-pixel im2col tile of x for GEMM row
 * m0, filter tap (r, s) and channel byte offset c_byte (box = box_bytes bytes
 * per pixel) with the same TMA descriptor construction as qconv2d_forward but
 * without swizzle, and writes it to `out` (device, 128*box_bytes bytes).
 */
qc_status qconv_debug_im2col_tile(const qconv_desc *d, const void *x, int64_t m0, int32_t r,
                                  int32_t s, int32_t c_byte, int32_t box_bytes, void *out,
                                  void *stream);

#ifdef __cplusplus
}
#endif

#endif /* QCONV_H_ */
