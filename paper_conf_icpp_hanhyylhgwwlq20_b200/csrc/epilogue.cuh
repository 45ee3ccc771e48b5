// epilogue.cuh -- launch parameters shared by the conv kernels, the fused epilogue
// (bias, per-channel fixed-point re-quantization, ReLU/clamp, sub-byte packing, dequantized
// float outputs) and the int4 -> int8 operand widening.
//
// Paper mapping (Han, Hu et al., ICPP'20; P:Lnnn = PAPER.md line):
//   * in-register bias + re-quantization after the mma loop (P:L223 l.15),
//     ReLU by the truncation range, reading Z3 (single rounding) or Z15
//     (gemmlowp/TFLite double rounding);
//   * fusion of convolution and dequantization: int32 -> fp32 in the epilogue
//     (reading Z16);
//   * 4-bit operands (P:L92 used Turing's native m8n8k32 s4): sm_100 has no int4 MMA, so
//     packed tiles are widened on chip (widen_word below).
#pragma once
#include <cstdint>
#include <cuda_bf16.h>
#include "ptx.cuh"

namespace qc {

constexpr int kBM = 128;             // output pixels per tile (UMMA M)
constexpr int kMaxBN = 256;
constexpr int kWarpTMA = 0;
constexpr int kWarpMMA = 1;
constexpr int kNumProducers = 3;      // TMA issuers: lane 0 of warps 0, 2, 3
constexpr int kWarpEpi0 = 4;         // warps 4..11: epilogue (TMEM lane quarter = warp % 4)
constexpr int kNumEpiWarps = 8;
constexpr int kWarpCvt0 = 12;        // warps 12..15: int4 -> int8 converters (4-bit only)
constexpr int kNumCvtWarps = 4;

constexpr int kMaxYstg = 4;          // halo / channel-major kernels: output staging buffers (max)
constexpr int kHaloMaxMMA = 18;      // halo kernel: 3x3 taps x 2 plane pairs (C = 64), or the 4x4/2 stem pairs
// channel-major kernel: 16 epilogue warps (4 per SMSP: the re-quantization is latency- not
// issue-bound), then the 4 converter warps (4-bit)
constexpr int kTEpiWarps = 16;
#ifndef QC_TGROUPS
#define QC_TGROUPS 2
#endif
// channel-major epilogue: warp groups on round-robin tiles, one accumulator (kTBNp pixels) each
constexpr int kTGroups = QC_TGROUPS;
constexpr int kTBNp = kTGroups == 4 ? 128 : 256;
constexpr int kTProducers = 2;        // TMA issuers: lane 0 of warps 0 and 3 (warp 2: output storer)
constexpr int kTWarpCvt0 = kWarpEpi0 + kTEpiWarps;
constexpr int kTThreads8 = 32 * kTWarpCvt0;
constexpr int kTThreads4 = 32 * (kTWarpCvt0 + kNumCvtWarps);

enum OutKind { OUT_S32 = 0, OUT_U8 = 1, OUT_S8 = 2, OUT_U4 = 3, OUT_S4 = 4, OUT_F32 = 5, OUT_BF16 = 6 };

template <int OUT> struct OutTraits {
    static constexpr bool kInt4 = OUT == OUT_U4 || OUT == OUT_S4;
    static constexpr bool kPacked = OUT == OUT_U4 || OUT == OUT_S4 || OUT == OUT_U8 || OUT == OUT_S8;
    static constexpr bool kFloat = OUT == OUT_F32 || OUT == OUT_BF16;
};

// n / d by multiply-high for 0 <= n < 2^31, 1 <= d < 2^31: with l = ceil(log2 d) and
// p = 31 + l, mul = ceil(2^p / d) < 2^32 and n / d = umulhi(n, mul) >> (p - 32) (the round-up
// multiplier method; the producers' per-tile / per-stage index math is on the critical path of
// the TMA issue loop, where an integer division costs a long dependent chain).
struct FastDiv {
    uint32_t d, mul, shr;
    __device__ __forceinline__ int div(int n) const {
        return d == 1u ? n : static_cast<int>(__umulhi(static_cast<uint32_t>(n), mul) >> shr);
    }
};
inline FastDiv make_fastdiv(uint32_t d) {
    FastDiv f;
    f.d = d;
    if (d <= 1u) { f.d = 1u; f.mul = 0u; f.shr = 0u; return f; }
    const uint32_t l = 32u - static_cast<uint32_t>(__builtin_clz(d - 1u));
    const uint64_t p = 31u + l;
    f.mul = static_cast<uint32_t>(((uint64_t(1) << p) + d - 1u) / d);
    f.shr = static_cast<uint32_t>(p - 32u);
    return f;
}

struct ConvParams {
    // GEMM geometry
    int32_t M, P, Q, PQ, K;
    int32_t BN, n_tiles_n, num_tiles, num_kb, chunks, S;
    int32_t stride_h, stride_w, pad_h, pad_w, dil_h, dil_w;
    int32_t H, W, R, C8;              // C8 = channels (int8 bytes per pixel after widening)
    int32_t BK, bkp, stages, sw_layout, sw_mask;
    int32_t pair;                     // C8 == 16: one K-stage = 2 filter taps x 16 B, no swizzle
    int32_t y_tma;                    // epilogue stages the whole output tile in smem -> TMA store
    uint32_t off_ystg;                // staging: 2 buffers x n_ygroups x [128 rows x y_gw bytes], swizzled
    uint32_t ystg_bytes;              // one staging buffer
    int32_t n_ystg;                   // halo / channel-major: staging buffers in the ring (2..4)
    int32_t n_wide;                   // channel-major 4-bit: widened operand slots (2..4)
    // halo kernel with fused fp32 quantization of the space-to-depth stem (F32 instantiation):
    // quantize_one parameters and the original image geometry
    float q_inv_s, q_flo, q_fhi;
    int32_t q_z, q_qmin, q_qmax;
    int32_t f_w, f_c, f_pad_h, f_pad_w, f_rowbytes;
    int32_t bf16;                     // fused stem: the input image is bf16 (else fp32)
    int32_t a_tmem_col;           // > 0 (im2col, 4-bit): the widened A operand goes to TMEM here
    int32_t b_res;                    // channel-major: the CTA's weights resident at off_bres
    const uint8_t *x_lin;             // channel-major 4-bit, 1x1/s1/p0, one K chunk: activations read
                                      // as one contiguous bulk copy per tile (else null: im2col TMA)
    int32_t x_row_bytes;              // packed bytes per pixel (x_lin)
    int32_t y_gw, y_gmask, n_ygroups; // staging group width (32/64/128 B), swizzle mask, count
    int32_t cvt_shift;                // log2(16-byte packed chunks per pixel) for the converter
    int32_t need_clamp;               // clamp range narrower than the output dtype range
    unsigned long long *trace;        // QC_DEBUG builds: per-event timestamps of CTA 0, else null
    uint32_t idesc, tmem_cols;
    // halo mode (stride-1 convs; a tile = Rt whole padded output rows of width Wh)
    int32_t Wh, Rt, HR, tiles_per_img, nplanes, nk_planes, tap_pair;
    uint32_t h_plane_bytes, off_hx, off_hp, hx_stage_bytes, hp_stage_bytes, off_bres, b_res_bytes;
    uint32_t halo_tx;
    int32_t halo_flat;                // halo loaded as whole pixel rows (3-D int64 view): staged
                                      // pixel-major [HR][Wh][c_px bytes] instead of 16-byte planes
    int32_t c_px;                     // packed bytes per input pixel (halo_flat)
    int32_t stg_sw;                   // TMA swizzle mask of the packed 4-bit staging rows (0 none,
                                      // 1 32B, 3 64B, 7 128B): SWIZZLE_NONE loads move 16 B per
                                      // request and are several times slower than swizzled ones
    uint32_t off_mtab; int32_t n_mma;  // halo: number of MMAs per tile
    // shared memory carve-up (byte offsets from the 1024-aligned base)
    uint32_t off_a, off_b, off_stg, off_bar, off_par;
    uint32_t a_stage_bytes, b_stage_bytes, stg_stage_bytes;
    // epilogue
    int32_t y_zero, clamp_lo, clamp_hi, x_zero;
    int32_t round_tfl;                // 1: gemmlowp/TFLite double rounding (Z15), general mode only
    int32_t relu;                     // float outputs: y = y > 0 ? y : +0
    const int32_t *bias, *mult, *shift;
    const float *dq_scale;            // float outputs: per-channel dequantization scale
    const int32_t *zx_table;          // [K][(R+1)*(S+1)] inclusive 2-D prefix sums of sum_c w
    const int32_t *zw;                // [K] weight zero points, or null
    const int32_t *x1;                // [M] sum over in-bounds taps and c of (x - x_zero) (zw != 0)
    // 4-bit activations (nibble-plane widening, see widen_word): the accumulator holds
    // 2^acc_lg * (acc + 8*sum_w if x_sgn4) -- acc_lg = 4 for 4-bit inputs, 0 for 8-bit
    int32_t acc_lg, x_sgn4;
    const int32_t *wsum;              // [K] sum_{r,s,c} w (true values) when x_sgn4, else null
    void *y;
    int64_t y_row_bytes;
    // fast divisions by P*Q, Q, n_tiles_n, S*chunks, chunks, S, tiles_per_img (set at launch)
    FastDiv fd_pq, fd_q, fd_ntn, fd_tpr, fd_chunks, fd_s, fd_tpi;
};

#ifdef QC_DEBUG
__device__ __forceinline__ void trace_ev(const ConvParams &p, int ev, int seq) {
    if (p.trace != nullptr && blockIdx.x == 0 && seq < 1024) p.trace[ev * 1024 + seq] = clock64();   // SM cycles
}
#else
__device__ __forceinline__ void trace_ev(const ConvParams &, int, int) {}
#endif

// ------------------------------------------------------------------ epilogue helpers
// Per-column epilogue constants (16 B in smem).  Their meaning is chosen per
// 32-column chunk (warp-uniform branch, no per-element branches):
//   fast chunk  {m, sh, C_lo, C_hi}: 33 <= shift <= 52 for all 32 columns:
//       y = clamp(hi32(acc*m + C) >> sh),  C = b*m + 2^(n-1) + zy*2^n (int64), sh = n-32
//     exact for any int32 m: |(acc+b)*m| <= 2^62 under the int32 contract, so the int64 sum
//     is exact, and floor(P / 2^n) = floor(hi32(P) / 2^(n-32)) for n >= 32 (IMAD.HI + shift)
//   mid chunk   {b, m, k, vlim}: 20 <= shift <= 50 and |m| >= 2^30 or m == 0 for all 32
//     columns; T = max(33, max shift of the chunk), k = T-n, vlim = 2^(n-20); per chunk
//     rhiT = 2^(T-33) + zy*2^(T-32):
//       x = clamp(acc + b, -vlim, vlim) << k;  y = clamp((mulhi(x, m) + rhiT) >> (T-32))
//     exact: scaling numerator and denominator by 2^k gives the common shift T; with
//     |m| >= 2^30, |acc+b| > 2^(n-20) gives |t| >= 2^10, which saturates every 8-bit output
//     range on the same side, so the pre-clamp changes nothing and keeps |x << k| <= 2^30
//     (m == 0 gives t = 0 either way).  A chunk with any 0 < |m| < 2^30 takes the general mode.
//   general chunk {b, m, n, zw}: t = (int64(v)*m + 2^(n-1)) >> n (int64) or the TFLite
//     double rounding (round_tfl), clamp, + zy; zw = weight zero point (ZX kernels)
//   S32 output   {b, 0, 0, zw}:  y = acc + b
//   float output {b, scale bits, 0, zw}: y = fl32(fl32(acc + b) * scale)
struct __align__(16) EpiCol {
    int32_t b, m, c2, c3;
};

__device__ __forceinline__ int4 lds128(uint32_t addr) {
    int4 v;
    asm volatile("ld.shared.v4.s32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
                 : "r"(addr));
    return v;
}

// number of valid filter taps along one spatial dim for output coordinate o:
// taps t in [t0, t1) with 0 <= o*stride - pad + t*dil < extent
__device__ __forceinline__ void valid_tap_range(int o, int stride, int pad, int dil, int extent,
                                                int taps, int &t0, int &t1) {
    const int base = o * stride - pad;
    int lo = 0;
    if (base < 0) lo = (-base + dil - 1) / dil;
    int hi = taps;
    const int lim = extent - 1 - base;          // t*dil <= lim
    if (lim < 0) hi = 0;
    else hi = min(taps, lim / dil + 1);
    t0 = lo;
    t1 = max(lo, hi);
}

// gemmlowp/TFLite MultiplyByQuantizedMultiplier with our (m, n) pair (reading Z15): the
// TFLite exponent is 31 - n; ls = max(0, 31-n) left shift (saturated to int32) before the
// SaturatingRoundingDoublingHighMul, rs = max(0, n-31) RoundingDivideByPOT after it.
// The high multiply is written as floor((a*m + 2^30) / 2^31), which equals gemmlowp's
// nudge-and-truncate form for every operand pair (oracle pin P13).
__device__ __forceinline__ int64_t requant_tflite(int32_t x, int32_t m, int n) {
    const int ls = n < 31 ? 31 - n : 0;
    const int rs = n > 31 ? n - 31 : 0;
    int64_t a = static_cast<int64_t>(x) * (static_cast<int64_t>(1) << ls);
    a = a > INT32_MAX ? static_cast<int64_t>(INT32_MAX) : (a < INT32_MIN ? static_cast<int64_t>(INT32_MIN) : a);
    int64_t h;
    if (a == INT32_MIN && m == INT32_MIN) h = INT32_MAX;
    else h = (a * m + (static_cast<int64_t>(1) << 30)) >> 31;
    const int64_t mask = (static_cast<int64_t>(1) << rs) - 1;
    const int64_t rem = h & mask;
    const int64_t thr = (mask >> 1) + (h < 0 ? 1 : 0);
    return (h >> rs) + (rem > thr ? 1 : 0);
}

// Fast chunk: 32 columns, all constants from smem (broadcast LDS.128), no branches.
template <int H, bool CLAMP>
__device__ __forceinline__ void epi_fast16(uint32_t (&v)[32], uint32_t par_addr, int32_t lo,
                                           int32_t hi) {
#pragma unroll
    for (int j = H; j < H + 16; ++j) {
        const int4 pr = lds128(par_addr + 16u * j);
        const int64_t c64 = (static_cast<int64_t>(pr.w) << 32) | static_cast<uint32_t>(pr.z);
        const int64_t prod = static_cast<int64_t>(static_cast<int32_t>(v[j])) * pr.x + c64;
        const int32_t t = static_cast<int32_t>(prod >> 32) >> pr.y;
        v[j] = static_cast<uint32_t>(CLAMP ? min(hi, max(lo, t)) : t);
    }
}

template <int H, bool CLAMP>
__device__ __forceinline__ void epi_mid16(uint32_t (&v)[32], uint32_t par_addr, int32_t lo,
                                          int32_t hi, int32_t rhi, int32_t sh) {
#pragma unroll
    for (int j = H; j < H + 16; ++j) {
        const int4 pr = lds128(par_addr + 16u * j);
        int32_t x = static_cast<int32_t>(v[j]) + pr.x;
        x = min(pr.w, max(-pr.w, x)) << pr.z;
        const int32_t t = (__mulhi(x, pr.y) + rhi) >> sh;
        v[j] = static_cast<uint32_t>(CLAMP ? min(hi, max(lo, t)) : t);
    }
}

// General chunk (any shift, either rounding, optional x_zero / w_zero corrections, int32
// or float output).  x1v = sum over the row's in-bounds taps of (x - x_zero) (w_zero != 0).
// The corrections are computed modulo 2^32: under the int32 contract the corrected
// accumulator fits int32, so the wrapped arithmetic gives it exactly.
template <int OUT, bool ZX, int H>
__device__ __forceinline__ void epi_general16(const ConvParams &p, uint32_t (&v)[32],
                                              uint32_t par_addr, int kc, int zr0, int zr1,
                                              int zs0, int zs1, int32_t x1v) {
#pragma unroll
    for (int j = H; j < H + 16; ++j) {
        const int4 pr = lds128(par_addr + 16u * j);
        uint32_t xu = static_cast<uint32_t>(static_cast<int32_t>(v[j]) >> p.acc_lg) + static_cast<uint32_t>(pr.x);
        if (ZX) {
            if (p.zx_table != nullptr) {
                const int k = min(kc + j, p.K - 1);
                const int RS1 = p.S + 1;
                const int32_t *t = p.zx_table + static_cast<int64_t>(k) * (p.R + 1) * RS1;
                const int32_t rect = __ldg(t + zr1 * RS1 + zs1) - __ldg(t + zr0 * RS1 + zs1) -
                                     __ldg(t + zr1 * RS1 + zs0) + __ldg(t + zr0 * RS1 + zs0);
                xu -= static_cast<uint32_t>(p.x_zero) * static_cast<uint32_t>(rect);
            }
            xu -= static_cast<uint32_t>(pr.w) * static_cast<uint32_t>(x1v);
        }
        const int32_t x = static_cast<int32_t>(xu);
        if (OUT == OUT_S32) {
            v[j] = xu;
        } else if (OutTraits<OUT>::kFloat) {
            float f = __fmul_rn(__int2float_rn(x), __int_as_float(pr.y));
            if (p.relu && !(f > 0.0f)) f = 0.0f;
            v[j] = __float_as_uint(f);
        } else {
            int64_t t;
            if (p.round_tfl) {
                t = requant_tflite(x, pr.y, pr.z);
            } else {
                const int64_t prod = static_cast<int64_t>(x) * pr.y + (static_cast<int64_t>(1) << (pr.z - 1));
                t = prod >> pr.z;
            }
            const int64_t lo64 = static_cast<int64_t>(p.clamp_lo) - p.y_zero;
            const int64_t hi64 = static_cast<int64_t>(p.clamp_hi) - p.y_zero;
            t = t < lo64 ? lo64 : (t > hi64 ? hi64 : t);
            v[j] = static_cast<uint32_t>(static_cast<int32_t>(t) + p.y_zero);
        }
    }
}

// Requantize the 32 accumulators of one chunk in place (mode per chunk, see EpiCol).
template <int OUT, bool ZX, int H>
__device__ __forceinline__ void epi_requant16(const ConvParams &p, uint32_t (&v)[32], uint32_t pa,
                                              int4 ci, int kc, int zr0, int zr1, int zs0, int zs1,
                                              int32_t x1v = 0) {
    if (ci.x == 0) {
        if (p.need_clamp) epi_fast16<H, true>(v, pa, p.clamp_lo, p.clamp_hi);
        else epi_fast16<H, false>(v, pa, p.clamp_lo, p.clamp_hi);
    } else if (ci.x == 1) {
        if (p.need_clamp) epi_mid16<H, true>(v, pa, p.clamp_lo, p.clamp_hi, ci.y, ci.z);
        else epi_mid16<H, false>(v, pa, p.clamp_lo, p.clamp_hi, ci.y, ci.z);
    } else {
        epi_general16<OUT, ZX, H>(p, v, pa, kc, zr0, zr1, zs0, zs1, x1v);
    }
}

// Position in an NS-stage mbarrier ring (stage, phase parity), advanced without divisions.
struct RingPos {
    int stage = 0;
    uint32_t phase = 0;
    __device__ __forceinline__ void next(int ns) {
        if (++stage == ns) { stage = 0; phase ^= 1u; }
    }
};

// Pack and store outputs v[H .. H+16) of one row = output channels [kc, kc+16) straight
// to global memory (int32 and float outputs, and packed outputs without a TMA store map).
template <int OUT, int H>
__device__ __forceinline__ void store16(const ConvParams &p, const uint32_t (&v)[32], int kc,
                                        int64_t m) {
    uint8_t *rowp = static_cast<uint8_t *>(p.y) + m * p.y_row_bytes;
    const bool in_range = kc + 16 <= p.K;
    if (OUT == OUT_S32 || OUT == OUT_F32) {
        uint32_t *dst = reinterpret_cast<uint32_t *>(rowp) + kc;
        if (in_range && (reinterpret_cast<uintptr_t>(dst) & 15u) == 0) {
#pragma unroll
            for (int j = 0; j < 16; j += 4) st_global_v4(dst + j, v[H + j], v[H + j + 1], v[H + j + 2], v[H + j + 3]);
        } else {
#pragma unroll
            for (int j = 0; j < 16; ++j)
                if (kc + j < p.K) dst[j] = v[H + j];
        }
    } else if (OUT == OUT_BF16) {
        uint32_t w[8];
#pragma unroll
        for (int j = 0; j < 8; ++j) {
            const uint32_t lo = __bfloat16_as_ushort(__float2bfloat16_rn(__uint_as_float(v[H + 2 * j])));
            const uint32_t hi = __bfloat16_as_ushort(__float2bfloat16_rn(__uint_as_float(v[H + 2 * j + 1])));
            w[j] = lo | (hi << 16);
        }
        uint16_t *dst = reinterpret_cast<uint16_t *>(rowp) + kc;
        if (in_range && (reinterpret_cast<uintptr_t>(dst) & 15u) == 0) {
            st_global_v4(dst, w[0], w[1], w[2], w[3]);
            st_global_v4(dst + 8, w[4], w[5], w[6], w[7]);
        } else {
#pragma unroll
            for (int j = 0; j < 16; ++j)
                if (kc + j < p.K) dst[j] = static_cast<uint16_t>(w[j >> 1] >> (16 * (j & 1)));
        }
    } else if (OUT == OUT_U8 || OUT == OUT_S8) {
        uint32_t w[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            const int32_t *y = reinterpret_cast<const int32_t *>(&v[H + 4 * j]);
            if (OUT == OUT_U8)
                w[j] = pack_sat_u8(y[1], y[0], pack_sat_u8(y[3], y[2], 0u));
            else
                w[j] = pack_sat_s8(y[1], y[0], pack_sat_s8(y[3], y[2], 0u));
        }
        uint8_t *dst = rowp + kc;
        if (in_range && (reinterpret_cast<uintptr_t>(dst) & 15u) == 0) {
            st_global_v4(dst, w[0], w[1], w[2], w[3]);
        } else {
#pragma unroll
            for (int j = 0; j < 16; ++j)
                if (kc + j < p.K) dst[j] = static_cast<uint8_t>(w[j >> 2] >> (8 * (j & 3)));
        }
    } else {
        uint32_t w[2];
#pragma unroll
        for (int j = 0; j < 2; ++j) {
            const int32_t *y = reinterpret_cast<const int32_t *>(&v[H + 8 * j]);
            if (OUT == OUT_U4) {
                uint32_t t = pack_sat_u4(y[7], y[6], 0u);
                t = pack_sat_u4(y[5], y[4], t);
                t = pack_sat_u4(y[3], y[2], t);
                w[j] = pack_sat_u4(y[1], y[0], t);
            } else {
                uint32_t t = pack_sat_s4(y[7], y[6], 0u);
                t = pack_sat_s4(y[5], y[4], t);
                t = pack_sat_s4(y[3], y[2], t);
                w[j] = pack_sat_s4(y[1], y[0], t);
            }
        }
        uint8_t *dst = rowp + kc / 2;
        if (in_range && (reinterpret_cast<uintptr_t>(dst) & 7u) == 0) {
            asm volatile("st.global.v2.b32 [%0], {%1, %2};" ::"l"(dst), "r"(w[0]), "r"(w[1]) : "memory");
        } else {
#pragma unroll
            for (int j = 0; j < 8; ++j)
                if (kc + 2 * j < p.K) dst[j] = static_cast<uint8_t>(w[j >> 2] >> (8 * (j & 3)));
        }
    }
}

// Pack outputs v[H .. H+16) (output channels col .. col+16 of the tile) of row `row` into the
// tile staging buffer: groups of y_gw bytes per row, each group a [128][y_gw] block with the
// TMA swizzle of that width (16-byte unit index XOR address bits 7.., as the TMA store reads it).
template <int OUT, int H>
__device__ __forceinline__ void stage16(const ConvParams &p, const uint32_t (&v)[32], uint32_t sbase,
                                        int row, int col) {
    constexpr bool kInt4 = OutTraits<OUT>::kInt4;
    const uint32_t ob = kInt4 ? static_cast<uint32_t>(col) / 2u : static_cast<uint32_t>(col);
    const uint32_t gw = static_cast<uint32_t>(p.y_gw);
    const uint32_t g = ob / gw, o = ob - g * gw;
    const uint32_t off = static_cast<uint32_t>(row) * gw + o;
    const uint32_t addr = sbase + g * 128u * gw + (off ^ (((off >> 7) & static_cast<uint32_t>(p.y_gmask)) << 4));
    if (!kInt4) {
        uint32_t w[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            const int32_t *y = reinterpret_cast<const int32_t *>(&v[H + 4 * j]);
            if (OUT == OUT_U8)
                w[j] = pack_sat_u8(y[1], y[0], pack_sat_u8(y[3], y[2], 0u));
            else
                w[j] = pack_sat_s8(y[1], y[0], pack_sat_s8(y[3], y[2], 0u));
        }
        sts128(addr, w[0], w[1], w[2], w[3]);
    } else {
        uint32_t w[2];
#pragma unroll
        for (int j = 0; j < 2; ++j) {
            const int32_t *y = reinterpret_cast<const int32_t *>(&v[H + 8 * j]);
            if (OUT == OUT_U4) {
                uint32_t t = pack_sat_u4(y[7], y[6], 0u);
                t = pack_sat_u4(y[5], y[4], t);
                t = pack_sat_u4(y[3], y[2], t);
                w[j] = pack_sat_u4(y[1], y[0], t);
            } else {
                uint32_t t = pack_sat_s4(y[7], y[6], 0u);
                t = pack_sat_s4(y[5], y[4], t);
                t = pack_sat_s4(y[3], y[2], t);
                w[j] = pack_sat_s4(y[1], y[0], t);
            }
        }
        sts64(addr, w[0], w[1]);
    }
}

template <int OUT, bool ZX, int H>
__device__ __forceinline__ void epi_half(const ConvParams &p, uint32_t (&v)[32], uint32_t pa,
                                         int4 cinfo, int kc, int64_t m, bool row_ok,
                                         int zr0, int zr1, int zs0, int zs1, int32_t x1v) {
    epi_requant16<OUT, ZX, H>(p, v, pa, cinfo, kc - H, zr0, zr1, zs0, zs1, x1v);
    if (row_ok) store16<OUT, H>(p, v, kc, m);
}

// Effective bias of column k in units of the true accumulator: the caller's bias, minus
// 8*sum_w when signed 4-bit activations were widened with the +8 offset (widen_word).
__device__ __forceinline__ int64_t eff_bias(const ConvParams &p, int k) {
    int64_t b = p.bias ? __ldg(p.bias + k) : 0;
    if (p.wsum) b -= 8 * static_cast<int64_t>(__ldg(p.wsum + k));
    return b;
}

// The re-quantization modes (fast / mid) a column can take, see EpiCol.
__device__ __forceinline__ bool mid_multiplier_ok(int32_t m) {
    return m == 0 || m >= (1 << 30) || m <= -(1 << 30);
}

// Per-column epilogue constants for the N tile at n0 (see EpiCol); called by all
// kNumEpiWarps epilogue warps together; thread (ew, lane) owns column 32*ew+lane.
// With acc_lg = L the accumulator is 2^L * (acc + offset): the fast/mid modes use the
// shift n + L and the bias 2^L * b_eff (the same rational, so the same exactness proofs),
// which needs |b_eff| < 2^26 (|2^L b_eff| < 2^30, |2^L b_eff m| < 2^61); the general mode
// shifts the accumulator back first.  Integer outputs with the TFLite rounding, int32 and
// float outputs and the zero-point kernels (ZX) always take the general mode.
template <int OUT>
__device__ __forceinline__ void fill_epilogue_params(const ConvParams &p, EpiCol *par, int4 *chunk_info,
                                                     int n0, int ew, int lane, bool force_general) {
    named_bar_sync(1, kNumEpiWarps * 32);
    force_general = force_general || !OutTraits<OUT>::kPacked || p.round_tfl;
    const int c = ew * 32 + lane;
    const int k = n0 + c;
    const bool kok = k < p.K;
    const int lg = p.acc_lg;
    const int64_t beff = kok ? eff_bias(p, k) : 0;
    EpiCol e;
    e.b = static_cast<int32_t>(beff);
    e.m = 0; e.c2 = 0; e.c3 = (p.zw != nullptr && kok) ? __ldg(p.zw + k) : 0;
    int32_t nn = 40 - lg;
    if (OutTraits<OUT>::kPacked && kok) {
        e.m = __ldg(p.mult + k);
        nn = __ldg(p.shift + k);
    } else if (OutTraits<OUT>::kFloat && kok) {
        e.m = __float_as_int(__ldg(p.dq_scale + k));
    }
    const int ne = nn + lg;
    const bool b_ok = lg == 0 ? (beff == static_cast<int64_t>(static_cast<int32_t>(beff)))
                              : (beff > -(int64_t(1) << 26) && beff < (int64_t(1) << 26));
    const bool all_fast = __ballot_sync(0xffffffffu, b_ok && ne >= 33 && ne <= 52) == 0xffffffffu;
    const bool all_mid = __ballot_sync(0xffffffffu, b_ok && ne >= 20 && ne <= 50 && mid_multiplier_ok(e.m)) ==
                         0xffffffffu;
    const int mode = force_general ? 2 : (all_fast ? 0 : (all_mid ? 1 : 2));
    const int T = max(33, __reduce_max_sync(0xffffffffu, ne));
    if (OutTraits<OUT>::kPacked && kok) {
        if (mode == 0) {
            const int64_t c64 = (beff << lg) * e.m + (static_cast<int64_t>(1) << (ne - 1)) +
                                (static_cast<int64_t>(p.y_zero) << ne);
            e.b = e.m;                                   // {m, sh, C_lo, C_hi}
            e.m = ne - 32;
            e.c2 = static_cast<int32_t>(static_cast<uint32_t>(c64));
            e.c3 = static_cast<int32_t>(c64 >> 32);
        } else if (mode == 1) {
            e.b = static_cast<int32_t>(beff << lg);
            e.c2 = T - ne;
            e.c3 = 1 << (ne - 20);
        } else {
            e.c2 = nn;
        }
    }
    if (c < p.BN) *reinterpret_cast<EpiCol *>(reinterpret_cast<uint8_t *>(par) + 16 * c) = e;
    if (lane == 0)
        chunk_info[ew] = make_int4(mode, mode == 1 ? (1 << (T - 33)) + p.y_zero * (1 << (T - 32)) : 0,
                                   T - 32, 0);
    named_bar_sync(1, kNumEpiWarps * 32);
}

// ------------------------------------------------------------------ int4 -> int8 widening
// "Nibble-plane" widening of one 32-bit word of eight packed 4-bit codes (element 2i in the
// low nibble of byte i) into two int8 words with no shifts or byte permutes:
//   lo = w' & 0x0F0F0F0F  -> bytes = the even elements        (x)
//   hi = w' & 0xF0F0F0F0  -> bytes = the odd elements times 16 (16 x)
// where w' = w for unsigned codes and w ^ 0x88888888 for signed ones (x + 8 in [0, 15], so
// the operand is always unsigned; the OOB zero fill of TMA stays x = 0 after the XOR).
// The prepared weights compensate (prep.cuh widen_w4_kernel): within every 32-channel
// group the even channels come first and carry 16 w, the odd channels follow with w, so
// the MMA sums 16 * x * w over every channel: acc = 16 (acc_true + 8 sum_w [signed]).  The
// epilogue folds the 16 into the re-quantization shift and the offset into the bias.
// Two LOP3 per word, versus shift + mask + two PRMT per word for in-order widening.
__device__ __forceinline__ void widen_word(uint32_t w, uint32_t xo, uint32_t &lo, uint32_t &hi) {
    lo = (w ^ xo) & 0x0F0F0F0Fu;
    hi = (w ^ xo) & 0xF0F0F0F0u;
}

// int4 -> int8 widening of one staged operand tile (Sec.3.2 P:L231-235 bit unpacking,
// done on chip): 16-byte packed chunk g of row g>>cshift becomes 32 widened bytes, written
// with the 128B/64B/32B swizzle the MMA descriptor expects.  A thread's chunks are kStride
// apart, i.e. (kStride >> cshift) >= 32 rows apart, so their swizzle phase is the same and
// the destination offsets are computed once.  Four chunks are loaded before any is
// converted so the shared-memory latency overlaps.
__device__ __forceinline__ void widen_stage(uint32_t stg, uint32_t adst, int ct, int nchunks,
                                            int cshift, uint32_t bkb, uint32_t sw, uint32_t xo,
                                            uint32_t ssw) {
    constexpr int kStride = kNumCvtWarps * 32;
    constexpr int U = 4;
    const uint32_t rr = static_cast<uint32_t>(ct) >> cshift;
    const uint32_t cir = static_cast<uint32_t>(ct) & ((1u << cshift) - 1u);
    const uint32_t off0 = rr * bkb + 32u * cir;
    const uint32_t off1 = off0 + 16u;
    const uint32_t d0 = adst + (off0 ^ (((off0 >> 7) & sw) << 4));
    const uint32_t d1 = adst + (off1 ^ (((off1 >> 7) & sw) << 4));
    const uint32_t dstep = (static_cast<uint32_t>(kStride) >> cshift) * bkb;
    // source chunk in the (TMA-swizzled) packed staging; the XOR term is the same for all of
    // this thread's chunks (they are >= 32 rows apart)
    const uint32_t soff = 16u * static_cast<uint32_t>(ct);
    const uint32_t s0 = stg + (soff ^ (((soff >> 7) & ssw) << 4));
    int i = 0;
    const int n_mine = ct < nchunks ? (nchunks - ct + kStride - 1) / kStride : 0;
    for (; i + U <= n_mine; i += U) {
        uint4 pk[U];
#pragma unroll
        for (int u = 0; u < U; ++u) pk[u] = lds128u(s0 + 16u * kStride * static_cast<uint32_t>(i + u));
#pragma unroll
        for (int u = 0; u < U; ++u) {
            uint32_t o[8];
            widen_word(pk[u].x, xo, o[0], o[4]);
            widen_word(pk[u].y, xo, o[1], o[5]);
            widen_word(pk[u].z, xo, o[2], o[6]);
            widen_word(pk[u].w, xo, o[3], o[7]);
            const uint32_t dd = dstep * static_cast<uint32_t>(i + u);
            sts128(d0 + dd, o[0], o[1], o[2], o[3]);
            sts128(d1 + dd, o[4], o[5], o[6], o[7]);
        }
    }
    for (; i < n_mine; ++i) {
        const uint4 pk = lds128u(s0 + 16u * kStride * static_cast<uint32_t>(i));
        uint32_t o[8];
        widen_word(pk.x, xo, o[0], o[4]);
        widen_word(pk.y, xo, o[1], o[5]);
        widen_word(pk.z, xo, o[2], o[6]);
        widen_word(pk.w, xo, o[3], o[7]);
        const uint32_t dd = dstep * static_cast<uint32_t>(i);
        sts128(d0 + dd, o[0], o[1], o[2], o[3]);
        sts128(d1 + dd, o[4], o[5], o[6], o[7]);
    }
}

}  // namespace qc
