/*
 * oracle.c -- CPU oracle for the 4/8-bit quantized convolution hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.
 * It shares no code, header, table or constant generator with the CUDA path
 * (paper_conf_icpp_hanhyylhgwwlq20_b200/csrc); it is deliberately plain and
 * slow: the textbook definition written out, int64/int128 arithmetic, no
 * blocking, no fusion, no reordering.
 *
 * Paper: Han, Hu et al., "Extremely Low-bit Convolution Optimization for
 * Quantized Neural Network on Modern Computer Architectures", ICPP'20.
 * Citations "P:Lnnn" are lines of /root/reference/PAPER.md; readings Z1..Z14 and R1
 * are listed in DESIGN.md section 3 (taken from SURVEY.md section 8(c)).
 *
 * Functions
 *   oracle_quantize       -- P:L257 (the "quantization" step of the QNN layer
 *                            sequence), reading Z4: q = clamp(rne(x*fl32(1/s))+z)
 *   oracle_requant_params -- reading R1 (the paper is silent on how the
 *                            re-quantization multiplier is derived)
 *   oracle_conv2d         -- P:L78 "direct convolution ... uses the definition
 *                            of convolution to calculate the output through
 *                            nested loops"; bias + re-quantization after the
 *                            full reduction (Alg.2 l.15, P:L253,
 *                            reading Z11), ReLU by the truncation range
 *                            (reading Z5), int4/int8/int32 output.
 *   oracle_conv2d_ex      -- the same convolution with the two NEXT epilogues
 *                            of SURVEY 8 row f1/f3:
 *                            * rounding = 1: gemmlowp/TFLite fixed-point
 *                              re-quantization (reading Z15; "same
 *                              quantization scheme", gemmlowp [14] P:L45):
 *                              SaturatingRoundingDoublingHighMul then
 *                              RoundingDivideByPOT, written as gemmlowp states
 *                              them (oracle_srdhm / oracle_rdbpot)
 *                            * yt = F32 / BF16: fusion of convolution and
 *                              dequantization (section 4.4, reading
 *                              Z16): y = fl32(fl32(acc) * scale[k]), acc incl.
 *                              bias, optional ReLU y = (y > 0 ? y : +0), bf16 =
 *                              round-to-nearest-even of the fp32 value.
 *
 * Parity pins: tests/test_oracle_pins.py (brute force, im2col+matmul,
 * 1x1==GEMM, identity/delta kernels, saturation, tie rule, requant params vs
 * exact rationals, quantize vs torch.quantize_per_tensor, invariants).
 */
#include <stdint.h>
#include <stddef.h>
#include <math.h>
#include <string.h>

/* dtype codes used by the oracle's own API (independent of include/qconv.h) */
enum { OR_U4 = 0, OR_S4 = 1, OR_U8 = 2, OR_S8 = 3, OR_S32 = 4, OR_F32 = 5, OR_BF16 = 6 };

static int dtype_bits(int t) {
    return (t == OR_U4 || t == OR_S4) ? 4 : ((t == OR_S32 || t == OR_F32) ? 32 : (t == OR_BF16 ? 16 : 8));
}
static int dtype_signed(int t) { return t == OR_S4 || t == OR_S8 || t == OR_S32; }
static int64_t dtype_min(int t) {
    switch (t) { case OR_U4: return 0; case OR_S4: return -8; case OR_U8: return 0;
                 case OR_S8: return -128; default: return INT32_MIN; }
}
static int64_t dtype_max(int t) {
    switch (t) { case OR_U4: return 15; case OR_S4: return 7; case OR_U8: return 255;
                 case OR_S8: return 127; default: return INT32_MAX; }
}

/* Read element `idx` of a packed row-major buffer of dtype t (reading Z7:
 * 4-bit element 2j is the low nibble of byte j, element 2j+1 the high nibble;
 * signed values are two's complement). */
static int64_t get_elem(const uint8_t *buf, int t, int64_t idx) {
    if (dtype_bits(t) == 4) {
        uint8_t b = buf[idx >> 1];
        int v = (idx & 1) ? (b >> 4) : (b & 0xF);
        if (t == OR_S4 && v >= 8) v -= 16;
        return v;
    }
    if (t == OR_S32) { int32_t v; memcpy(&v, buf + 4 * idx, 4); return v; }
    return t == OR_S8 ? (int64_t)(int8_t)buf[idx] : (int64_t)buf[idx];
}

static void put_elem(uint8_t *buf, int t, int64_t idx, int64_t v) {
    if (dtype_bits(t) == 4) {
        uint8_t nib = (uint8_t)(v & 0xF);
        uint8_t *b = &buf[idx >> 1];
        if (idx & 1) *b = (uint8_t)((*b & 0x0F) | (nib << 4));
        else         *b = (uint8_t)((*b & 0xF0) | nib);
        return;
    }
    if (t == OR_S32) { int32_t w = (int32_t)v; memcpy(buf + 4 * idx, &w, 4); return; }
    buf[idx] = (uint8_t)(v & 0xFF);
}

/* ------------------------------------------------------------------------ */
/* Quantization (reading Z4).
 * For every element: inv_s = fl32(1/s); t = fl32(x * inv_s) (one IEEE fp32
 * multiply, round-to-nearest-even); q = rne(t) + z clamped to the dtype range.
 * NaN -> z.  Channels c in [C, C_pad) are filled with z.
 * x is fp32 (xt = 0) or bf16 bit patterns (xt = 1, widened exactly). */
int oracle_quantize(const void *x, int xt, int64_t npix, int c, int c_pad,
                    float scale, int zero_point, int yt, uint8_t *y) {
    if (!(scale > 0.0f) || !isfinite(scale)) return 1;
    if (c_pad < c || (yt != OR_U4 && yt != OR_S4 && yt != OR_U8 && yt != OR_S8)) return 1;
    if (dtype_bits(yt) == 4 && (c_pad & 1)) return 1;
    if (zero_point < dtype_min(yt) || zero_point > dtype_max(yt)) return 1;
    const float inv_s = 1.0f / scale;
    const int64_t qmin = dtype_min(yt), qmax = dtype_max(yt);
    for (int64_t p = 0; p < npix; ++p) {
        for (int ch = 0; ch < c_pad; ++ch) {
            int64_t q;
            if (ch >= c) {
                q = zero_point;
            } else {
                float xv;
                if (xt == 0) {
                    xv = ((const float *)x)[p * c + ch];
                } else {
                    uint32_t bits = (uint32_t)((const uint16_t *)x)[p * c + ch] << 16;
                    memcpy(&xv, &bits, 4);
                }
                volatile float t = xv * inv_s;        /* single fp32 product */
                if (isnan(t)) {
                    q = zero_point;
                } else {
                    double r = rint((double)t);          /* RNE (default mode) */
                    double qd = r + (double)zero_point;
                    if (qd < (double)qmin) qd = (double)qmin;
                    if (qd > (double)qmax) qd = (double)qmax;
                    q = (int64_t)qd;
                }
            }
            put_elem(y, yt, p * c_pad + ch, q);
        }
    }
    return 0;
}

/* ------------------------------------------------------------------------ */
/* Re-quantization parameters (reading R1).
 * M_k = fl64(fl64(s_in) * fl64(s_w[k])) / fl64(s_out)  (exact product, one
 * RNE division).  (f, e) = frexp(M_k), f in [0.5, 1); m = round-half-up(f*2^31);
 * if m == 2^31 then m = 2^30, e += 1; shift = 31 - e, must lie in [1, 62].
 * M_k == 0 -> m = 0, shift = 31.  Returns 0 on success, 1 on invalid input. */
int oracle_requant_params(float in_scale, const float *w_scale, float out_scale, int k,
                          int32_t *mult, int32_t *shift) {
    if (!(in_scale > 0.0f) || !(out_scale > 0.0f) || !isfinite(in_scale) || !isfinite(out_scale))
        return 1;
    for (int i = 0; i < k; ++i) {
        if (!(w_scale[i] >= 0.0f) || !isfinite(w_scale[i])) return 1;
        double M = ((double)in_scale * (double)w_scale[i]) / (double)out_scale;
        if (M == 0.0) { mult[i] = 0; shift[i] = 31; continue; }
        int e;
        double f = frexp(M, &e);
        double scaled = ldexp(f, 31);                 /* exact */
        int64_t m = (int64_t)floor(scaled + 0.5);     /* half up (scaled > 0) */
        if (m == ((int64_t)1 << 31)) { m = (int64_t)1 << 30; e += 1; }
        int n = 31 - e;
        if (n < 1 || n > 62) return 1;
        mult[i] = (int32_t)m;
        shift[i] = n;
    }
    return 0;
}

/* ------------------------------------------------------------------------ */
/* gemmlowp fixed-point primitives (reading Z15), as gemmlowp defines them.
 * SaturatingRoundingDoublingHighMul(a, b): the high 32 bits of 2*a*b with
 * rounding: nudge = ab >= 0 ? 2^30 : 1 - 2^30, result = (ab + nudge) / 2^31
 * with C's truncating division; the one overflowing case a = b = INT32_MIN
 * saturates to INT32_MAX. */
int32_t oracle_srdhm(int32_t a, int32_t b) {
    if (a == INT32_MIN && b == INT32_MIN) return INT32_MAX;
    const int64_t ab = (int64_t)a * (int64_t)b;
    const int64_t nudge = ab >= 0 ? ((int64_t)1 << 30) : (1 - ((int64_t)1 << 30));
    return (int32_t)((ab + nudge) / ((int64_t)1 << 31));
}

/* RoundingDivideByPOT(x, e): mask = 2^e - 1, remainder = x & mask,
 * threshold = (mask >> 1) + (x < 0), result = (x >> e) + (remainder > threshold). */
int32_t oracle_rdbpot(int32_t x, int e) {
    const int32_t mask = (int32_t)(((int64_t)1 << e) - 1);
    const int32_t remainder = x & mask;
    const int32_t threshold = (mask >> 1) + (x < 0 ? 1 : 0);
    return (x >> e) + (remainder > threshold ? 1 : 0);
}

/* TFLite MultiplyByQuantizedMultiplier with our (multiplier, shift) pair:
 * the TFLite exponent is 31 - shift; a positive exponent is a left shift of
 * the accumulator first (saturated to int32, reading Z15), a negative one the
 * RoundingDivideByPOT after the high multiply. */
static int64_t requant_tflite(int64_t acc, int32_t m, int sh) {
    const int left = sh < 31 ? 31 - sh : 0;
    const int right = sh > 31 ? sh - 31 : 0;
    int64_t a = acc * ((int64_t)1 << left);
    if (a > INT32_MAX) a = INT32_MAX;
    if (a < INT32_MIN) a = INT32_MIN;
    return oracle_rdbpot(oracle_srdhm((int32_t)a, m), right);
}

/* fp32 -> bf16 bit pattern, round to nearest even (finite inputs; the
 * dequantized values are always finite). */
static uint16_t f32_to_bf16_rne(float f) {
    uint32_t u;
    memcpy(&u, &f, 4);
    const uint32_t lsb = (u >> 16) & 1u;
    u += 0x7FFFu + lsb;
    return (uint16_t)(u >> 16);
}

/* ------------------------------------------------------------------------ */
/* Direct convolution with the integer or float epilogue.
 *
 * for n,p,q,k:
 *   acc = bias[k] + sum_{r,s in bounds} sum_c (X[n,h,w,c]-zx) * (W[k,r,s,c]-zw[k])
 *        (out-of-bounds taps are a real zero: they contribute nothing, Z2)
 *   S32 output : y = acc
 *   F32 / BF16 : y = fl32(fl32(acc) * dq_scale[k]); relu: y = y > 0 ? y : +0 (Z16)
 *   else, rounding 0 : t = floor((acc*m[k] + 2^(sh[k]-1)) / 2^sh[k])   (Z3, exact int128)
 *         rounding 1 : t = requant_tflite(acc, m[k], sh[k])            (Z15)
 *               y = min(hi, max(lo, t + zy))                              (Z5)
 *
 * Returns the number of outputs whose acc lies outside int32 (the paper's
 * 32-bit accumulator: such an input is outside the method's
 * contract; the tests require 0).  Returns -1 on invalid arguments. */
int64_t oracle_conv2d_ex(int n_, int h_, int w_, int c_, int k_, int r_, int s_,
                         int stride_h, int stride_w, int pad_h, int pad_w, int dil_h, int dil_w,
                         int xt, int wt, int yt, int x_zero, const int32_t *w_zero,
                         int y_zero, int clamp_lo, int clamp_hi, int rounding,
                         const uint8_t *x, const uint8_t *w, const int32_t *bias,
                         const int32_t *mult, const int32_t *shift, const float *dq_scale,
                         int relu, uint8_t *y) {
    if (n_ < 0 || h_ <= 0 || w_ <= 0 || c_ <= 0 || k_ <= 0 || r_ <= 0 || s_ <= 0) return -1;
    if (stride_h <= 0 || stride_w <= 0 || dil_h <= 0 || dil_w <= 0 || pad_h < 0 || pad_w < 0) return -1;
    const int P = (h_ + 2 * pad_h - dil_h * (r_ - 1) - 1) / stride_h + 1;
    const int Q = (w_ + 2 * pad_w - dil_w * (s_ - 1) - 1) / stride_w + 1;
    if (P <= 0 || Q <= 0) return -1;
    const int is_float = yt == OR_F32 || yt == OR_BF16;
    if (is_float && !dq_scale) return -1;
    if (!is_float && yt != OR_S32 && (!mult || !shift)) return -1;
    if (rounding != 0 && rounding != 1) return -1;
    int64_t overflow = 0;
    #pragma omp parallel for collapse(2) schedule(static) reduction(+:overflow)
    for (int n = 0; n < n_; ++n) {
        for (int p = 0; p < P; ++p) {
            for (int q = 0; q < Q; ++q) {
                for (int k = 0; k < k_; ++k) {
                    int64_t acc = bias ? (int64_t)bias[k] : 0;
                    const int64_t zw = w_zero ? (int64_t)w_zero[k] : 0;
                    for (int r = 0; r < r_; ++r) {
                        const int hh = p * stride_h - pad_h + r * dil_h;
                        if (hh < 0 || hh >= h_) continue;
                        for (int s = 0; s < s_; ++s) {
                            const int ww = q * stride_w - pad_w + s * dil_w;
                            if (ww < 0 || ww >= w_) continue;
                            const int64_t xbase = (((int64_t)n * h_ + hh) * w_ + ww) * c_;
                            const int64_t wbase = (((int64_t)k * r_ + r) * s_ + s) * c_;
                            for (int c = 0; c < c_; ++c) {
                                const int64_t xv = get_elem(x, xt, xbase + c) - x_zero;
                                const int64_t wv = get_elem(w, wt, wbase + c) - zw;
                                acc += xv * wv;
                            }
                        }
                    }
                    if (acc > INT32_MAX || acc < INT32_MIN) overflow += 1;
                    const int64_t oidx = (((int64_t)n * P + p) * Q + q) * k_ + k;
                    if (yt == OR_S32) {
                        put_elem(y, yt, oidx, acc);
                    } else if (is_float) {
                        volatile float fa = (float)acc;              /* RNE int -> fp32 */
                        volatile float fy = fa * dq_scale[k];        /* one fp32 product */
                        float v = fy;
                        if (relu && !(v > 0.0f)) v = 0.0f;
                        if (yt == OR_F32) {
                            memcpy(y + 4 * oidx, &v, 4);
                        } else {
                            const uint16_t b = f32_to_bf16_rne(v);
                            memcpy(y + 2 * oidx, &b, 2);
                        }
                    } else {
                        const int sh = shift[k];
                        __int128 t;
                        if (rounding == 0) {
                            __int128 prod = (__int128)acc * (__int128)mult[k];
                            __int128 num = prod + ((__int128)1 << (sh - 1));
                            /* floor division by 2^sh (arithmetic shift of int128 = floor) */
                            t = num >> sh;
                        } else {
                            t = requant_tflite(acc, mult[k], sh);
                        }
                        __int128 v = t + y_zero;
                        if (v < clamp_lo) v = clamp_lo;
                        if (v > clamp_hi) v = clamp_hi;
                        put_elem(y, yt, oidx, (int64_t)v);
                    }
                }
            }
        }
    }
    return overflow;
}

/* The round-1 entry point: single rounding, integer outputs. */
int64_t oracle_conv2d(int n_, int h_, int w_, int c_, int k_, int r_, int s_,
                      int stride_h, int stride_w, int pad_h, int pad_w, int dil_h, int dil_w,
                      int xt, int wt, int yt, int x_zero, const int32_t *w_zero,
                      int y_zero, int clamp_lo, int clamp_hi,
                      const uint8_t *x, const uint8_t *w, const int32_t *bias,
                      const int32_t *mult, const int32_t *shift, uint8_t *y) {
    if (yt == OR_F32 || yt == OR_BF16) return -1;
    return oracle_conv2d_ex(n_, h_, w_, c_, k_, r_, s_, stride_h, stride_w, pad_h, pad_w, dil_h,
                            dil_w, xt, wt, yt, x_zero, w_zero, y_zero, clamp_lo, clamp_hi, 0, x, w,
                            bias, mult, shift, NULL, 0, y);
}

/* Smallest/largest representable values, exported for the Python wrapper. */
long long oracle_dtype_min(int t) { return dtype_min(t); }
long long oracle_dtype_max(int t) { return dtype_max(t); }
int oracle_dtype_bits(int t) { return dtype_bits(t); }
int oracle_dtype_signed(int t) { return dtype_signed(t); }
