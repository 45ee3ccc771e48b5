// conv_fwd.cuh -- implicit-GEMM 4/8-bit quantized convolution for sm_100a.
//
// Paper mapping (Han, Hu et al., ICPP'20, section 4; P:Lnnn = PAPER.md line):
//   * implicit(-precomp) GEMM conv, Alg.2: GEMM rows m = (n,p,q)
//     output pixels, columns = output channels k, reduction = (r,s,c).  The
//     paper's precomputed offset buffer is replaced by the TMA im2col
//     descriptor: the hardware generates the gather addresses and zero-fills
//     out-of-bounds taps, with no global workspace.
//   * data partition: CTA tile = 128 output pixels x BN output
//     channels (one UMMA tile, accumulator in TMEM), K-stage = one filter tap
//     x BK bytes of channels.  Warp specialisation replaces the paper's warp
//     tiling: warp 0 issues TMA, one thread of warp 1 issues tcgen05.mma,
//     warps 4-11 run the epilogue, (4-bit) warps 12-15 widen int4 to int8.
//   * register prefetch buffer -> a multi-stage shared-memory
//     ring guarded by mbarriers; the epilogue of tile i overlaps the MMAs of
//     tile i+1 through two TMEM accumulator buffers.
//   * in-register bias + re-quantization (P:L223 l.15) and ReLU by
//     truncation range: fused epilogue, TMEM -> registers -> int8 /
//     int4-packed / int32 stores straight to HBM, no int32 round trip.
//   * 4-bit (P:L92 uses Turing's native m8n8k32 s4): sm_100 has no int4
//     MMA, so packed int4 activation tiles are TMA-loaded as bytes and widened
//     to int8 in shared memory by converter warps; weights are widened once
//     by qconv_prepare_weights.
#pragma once
#include <cstdint>
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

enum OutKind { OUT_S32 = 0, OUT_U8 = 1, OUT_S8 = 2, OUT_U4 = 3, OUT_S4 = 4 };

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
    int32_t y_gw, y_gmask, n_ygroups; // staging group width (32/64/128 B), swizzle mask, count
    int32_t cvt_shift;                // log2(16-byte packed chunks per pixel) for the converter
    int32_t need_clamp;               // clamp range narrower than the output dtype range
    unsigned long long *trace;        // debug: per-event timestamps of CTA 0 (QC_TRACE), or null
    int32_t exp_flags;                // debug experiments (QC_EXPERIMENT): 1 no B reload, 2 no A reload,
                                      // 4 no MMA, 8 epilogue: TMEM loads only, 16 epilogue: nothing
    uint32_t idesc, tmem_cols;
    // halo mode (stride-1 convs; a tile = Rt whole padded output rows of width Wh)
    int32_t Wh, Rt, HR, tiles_per_img, nplanes, nk_planes, tap_pair;
    uint32_t h_plane_bytes, off_hx, off_hp, hx_stage_bytes, hp_stage_bytes, off_bres, b_res_bytes;
    uint32_t halo_tx;
    int32_t halo_flat;                // halo loaded as whole pixel rows (3-D int64 view): staged
                                      // pixel-major [HR][Wh][c_px bytes] instead of 16-byte planes
    int32_t c_px;                     // packed bytes per input pixel (halo_flat)
    int32_t w_early;                  // weights may be loaded before griddep_wait (they were not
                                      // written by a kernel of this call)
    int32_t stg_sw;                   // TMA swizzle mask of the packed 4-bit staging rows (0 none,
                                      // 1 32B, 3 64B, 7 128B): SWIZZLE_NONE loads move 16 B per
                                      // request and are several times slower than swizzled ones
    uint32_t off_mtab; int32_t n_mma;  // halo: per-MMA descriptor offsets {a>>4, b>>4}
    // shared memory carve-up (byte offsets from the 1024-aligned base)
    uint32_t off_a, off_b, off_stg, off_bar, off_par;
    uint32_t a_stage_bytes, b_stage_bytes, stg_stage_bytes;
    // epilogue
    int32_t y_zero, clamp_lo, clamp_hi, x_zero;
    const int32_t *bias, *mult, *shift;
    const int32_t *zx_table;          // [K][(R+1)*(S+1)] inclusive 2-D prefix sums of sum_c w
    // 4-bit activations (nibble-plane widening, see widen_word): the accumulator holds
    // 2^acc_lg * (acc + 8*sum_w if x_sgn4) -- acc_lg = 4 for 4-bit inputs, 0 for 8-bit
    int32_t acc_lg, x_sgn4;
    const int32_t *wsum;              // [K] sum_{r,s,c} w (true values) when x_sgn4, else null
    void *y;
    int64_t y_row_bytes;
};

// ------------------------------------------------------------------ epilogue helpers
// Per-column epilogue constants (16 B in smem).  Their meaning is chosen per
// 32-column chunk (warp-uniform branch, no per-element branches):
//   fast chunk  {m, sh, C_lo, C_hi}: 33 <= shift <= 52 for all 32 columns, x_zero == 0:
//       y = clamp(hi32(acc*m + C) >> sh),  C = b*m + 2^(n-1) + zy*2^n (int64), sh = n-32
//     exact: |(acc+b)*m| < 2^62 under the int32 contract, so the int64 sum is exact, and
//     floor(P / 2^n) = floor(hi32(P) / 2^(n-32)) for n >= 32 (one IMAD.HI + one shift)
//   mid chunk   {b, m, k, vlim}: 20 <= shift <= 50 for all 32 columns; T = max(33, max shift
//     of the chunk), k = T-n, vlim = 2^(n-20); per chunk rhiT = 2^(T-33) + zy*2^(T-32):
//       x = clamp(acc + b, -vlim, vlim) << k;  y = clamp((mulhi(x, m) + rhiT) >> (T-32))
//     exact: scaling numerator and denominator by 2^k gives the common shift T; |acc+b| >
//     2^(n-20) already saturates every 8-bit output range (|t| >= 2^10), so the pre-clamp
//     changes nothing and keeps |x << k| <= 2^30
//   general chunk {b, m, n, 0}: t = (int64(v)*m + 2^(n-1)) >> n (int64), clamp, + zy
//   S32 output   {b, 0, 0, 0}:  y = acc + b
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

template <int OUT, bool ZX, int H>
__device__ __forceinline__ void epi_general16(const ConvParams &p, uint32_t (&v)[32],
                                              uint32_t par_addr, int kc, int zr0, int zr1,
                                              int zs0, int zs1);

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

// Requantize the 32 accumulators of one chunk in place (mode per chunk, see EpiCol).
template <int OUT, bool ZX, int H>
__device__ __forceinline__ void epi_requant16(const ConvParams &p, uint32_t (&v)[32], uint32_t pa,
                                              int4 ci, int kc, int zr0, int zr1, int zs0, int zs1) {
    if (ci.x == 0) {
        if (p.need_clamp) epi_fast16<H, true>(v, pa, p.clamp_lo, p.clamp_hi);
        else epi_fast16<H, false>(v, pa, p.clamp_lo, p.clamp_hi);
    } else if (ci.x == 1) {
        if (p.need_clamp) epi_mid16<H, true>(v, pa, p.clamp_lo, p.clamp_hi, ci.y, ci.z);
        else epi_mid16<H, false>(v, pa, p.clamp_lo, p.clamp_hi, ci.y, ci.z);
    } else {
        epi_general16<OUT, ZX, H>(p, v, pa, kc, zr0, zr1, zs0, zs1);
    }
}

// General chunk (any shift, optional x_zero border correction, or int32 output).
template <int OUT, bool ZX, int H>
__device__ __forceinline__ void epi_general16(const ConvParams &p, uint32_t (&v)[32],
                                              uint32_t par_addr, int kc, int zr0, int zr1,
                                              int zs0, int zs1) {
#pragma unroll
    for (int j = H; j < H + 16; ++j) {
        const int4 pr = lds128(par_addr + 16u * j);
        int32_t x = (static_cast<int32_t>(v[j]) >> p.acc_lg) + pr.x;
        if (ZX) {
            const int k = min(kc + j, p.K - 1);
            const int RS1 = p.S + 1;
            const int32_t *t = p.zx_table + static_cast<int64_t>(k) * (p.R + 1) * RS1;
            const int32_t rect = __ldg(t + zr1 * RS1 + zs1) - __ldg(t + zr0 * RS1 + zs1) -
                                 __ldg(t + zr1 * RS1 + zs0) + __ldg(t + zr0 * RS1 + zs0);
            x -= p.x_zero * rect;
        }
        if (OUT == OUT_S32) {
            v[j] = static_cast<uint32_t>(x);
        } else {
            const int64_t prod = static_cast<int64_t>(x) * pr.y + (static_cast<int64_t>(1) << (pr.z - 1));
            int64_t t = prod >> pr.z;
            const int64_t lo64 = static_cast<int64_t>(p.clamp_lo) - p.y_zero;
            const int64_t hi64 = static_cast<int64_t>(p.clamp_hi) - p.y_zero;
            t = t < lo64 ? lo64 : (t > hi64 ? hi64 : t);
            v[j] = static_cast<uint32_t>(static_cast<int32_t>(t) + p.y_zero);
        }
    }
}

// Pack and store outputs v[H .. H+16) of one row = output channels [kc, kc+16).
template <int OUT, int H>
__device__ __forceinline__ void store16(const ConvParams &p, const uint32_t (&v)[32], int kc,
                                        int64_t m) {
    uint8_t *rowp = static_cast<uint8_t *>(p.y) + m * p.y_row_bytes;
    const bool in_range = kc + 16 <= p.K;
    if (OUT == OUT_S32) {
        uint32_t *dst = reinterpret_cast<uint32_t *>(rowp) + kc;
        if (in_range && (reinterpret_cast<uintptr_t>(dst) & 15u) == 0) {
#pragma unroll
            for (int j = 0; j < 16; j += 4) st_global_v4(dst + j, v[H + j], v[H + j + 1], v[H + j + 2], v[H + j + 3]);
        } else {
#pragma unroll
            for (int j = 0; j < 16; ++j)
                if (kc + j < p.K) dst[j] = v[H + j];
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
    constexpr bool kInt4 = (OUT == OUT_U4 || OUT == OUT_S4);
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
                                         int zr0, int zr1, int zs0, int zs1) {
    epi_requant16<OUT, ZX, H>(p, v, pa, cinfo, kc - H, zr0, zr1, zs0, zs1);
    if (row_ok) store16<OUT, H>(p, v, kc, m);
}

// Per-column epilogue constants for the N tile at n0 (see EpiCol); called by all
// kNumEpiWarps epilogue warps together; thread (ew, lane) owns column 32*ew+lane.
// Effective bias of column k in units of the true accumulator: the caller's bias, minus
// 8*sum_w when signed 4-bit activations were widened with the +8 offset (widen_word).
__device__ __forceinline__ int64_t eff_bias(const ConvParams &p, int k) {
    int64_t b = p.bias ? __ldg(p.bias + k) : 0;
    if (p.wsum) b -= 8 * static_cast<int64_t>(__ldg(p.wsum + k));
    return b;
}

// Per-column epilogue constants for the N tile at n0 (see EpiCol); called by all
// kNumEpiWarps epilogue warps together; thread (ew, lane) owns column 32*ew+lane.
// With acc_lg = L the accumulator is 2^L * (acc + offset): the fast/mid modes use the
// shift n + L and the bias 2^L * b_eff (the same rational, so the same exactness proofs),
// which needs |b_eff| < 2^26 (|2^L b_eff| < 2^30, |2^L b_eff m| < 2^61); the general mode
// shifts the accumulator back first.
template <int OUT>
__device__ __forceinline__ void fill_epilogue_params(const ConvParams &p, EpiCol *par, int4 *chunk_info,
                                                     int n0, int ew, int lane, bool force_general) {
    named_bar_sync(1, kNumEpiWarps * 32);
    const int c = ew * 32 + lane;
    const int k = n0 + c;
    const int lg = p.acc_lg;
    const int64_t beff = k < p.K ? eff_bias(p, k) : 0;
    EpiCol e;
    e.b = static_cast<int32_t>(beff);
    e.m = 0; e.c2 = 0; e.c3 = 0;
    int32_t nn = 40 - lg;
    if (OUT != OUT_S32 && k < p.K) {
        e.m = __ldg(p.mult + k);
        nn = __ldg(p.shift + k);
    }
    const int ne = nn + lg;
    const bool b_ok = lg == 0 ? (beff == static_cast<int64_t>(static_cast<int32_t>(beff)))
                              : (beff > -(int64_t(1) << 26) && beff < (int64_t(1) << 26));
    const bool all_fast = __ballot_sync(0xffffffffu, b_ok && ne >= 33 && ne <= 52) == 0xffffffffu;
    const bool all_mid = __ballot_sync(0xffffffffu, b_ok && ne >= 20 && ne <= 50) == 0xffffffffu;
    const int mode = force_general ? 2 : (all_fast ? 0 : (all_mid ? 1 : 2));
    const int T = max(33, __reduce_max_sync(0xffffffffu, ne));
    if (OUT != OUT_S32 && k < p.K) {
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

__device__ __forceinline__ void trace_ev(const ConvParams &p, int ev, int seq) {
    if (p.trace != nullptr && blockIdx.x == 0 && seq < 1024) p.trace[ev * 1024 + seq] = globaltimer_ns();
}

// ------------------------------------------------------------------ the kernel
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

template <bool IS4, int OUT, bool ZX>
__global__ void __launch_bounds__(IS4 ? 512 : 384, 1)
qconv_fwd_kernel(const __grid_constant__ CUtensorMap xmap, const __grid_constant__ CUtensorMap wmap,
                 const __grid_constant__ CUtensorMap ymap, const __grid_constant__ ConvParams p) {
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                                ~uintptr_t(1023));
    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;
    const int NS = p.stages;

    uint64_t *bars = reinterpret_cast<uint64_t *>(smem + p.off_bar);
    uint64_t *full = bars;                  // [NS] TMA -> (converter | MMA)
    uint64_t *empty = bars + NS;            // [NS] MMA -> TMA
    uint64_t *aready = bars + 2 * NS;       // [NS] converter -> MMA (4-bit)
    uint64_t *tfull = bars + 3 * NS;        // [2]  MMA -> epilogue
    uint64_t *tempty = bars + 3 * NS + 2;   // [2]  epilogue -> MMA
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(bars + 3 * NS + 4);
    EpiCol *par = reinterpret_cast<EpiCol *>(smem + p.off_par);
    int4 *chunk_info = reinterpret_cast<int4 *>(smem + p.off_par + 16 * kMaxBN);  // [8] {mode, rhiT, shT, 0}

    griddep_launch_dependents();
    if (warp == kWarpTMA && lane == 0) {
        tma_prefetch_desc(&xmap);
        tma_prefetch_desc(&wmap);
        if (p.y_tma) tma_prefetch_desc(&ymap);
        for (int i = 0; i < NS; ++i) {
            mbar_init(&full[i], 1);
            mbar_init(&empty[i], 1);
            mbar_init(&aready[i], kNumCvtWarps);
        }
        for (int i = 0; i < 2; ++i) {
            mbar_init(&tfull[i], 1);
            mbar_init(&tempty[i], kNumEpiWarps);
        }
        fence_mbar_init();
    }
    if (warp == kWarpMMA) tmem_alloc(tmem_slot, p.tmem_cols);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;
    const int taps_per_r = p.S * p.chunks;

    if (warp == kWarpTMA || warp == 2 || warp == 3) {
        // ===================== TMA producers (lane 0 of warps 0, 2, 3) =====================
        // Each TMA issue costs the issuing thread a few hundred cycles (measured on B200:
        // ~300-420 cycles per wait+expect_tx+load sequence, independent of box size up to
        // 16 KB), so K-stages are dealt round-robin to kNumProducers threads.
        if (lane == 0) {   // one thread issues (measured faster than an elected warp-wide loop)
            constexpr bool leader = true;
            griddep_wait();                                         // activations of the previous layer
            const int pi = warp == kWarpTMA ? 0 : warp - 1;       // 0, 1, 2
            const uint32_t tx = static_cast<uint32_t>(kBM * (p.pair ? 32 : p.bkp) + p.BN * p.BK);
            int g = 0;                                              // CTA-local K-stage counter
            for (int tile = blockIdx.x; tile < p.num_tiles; tile += gridDim.x) {
                const int m0 = (tile / p.n_tiles_n) * kBM;
                const int n0 = (tile % p.n_tiles_n) * p.BN;
                const int img = m0 / p.PQ;
                const int rem = m0 - img * p.PQ;
                const int p0 = rem / p.Q;
                const int q0 = rem - p0 * p.Q;
                const int wb = q0 * p.stride_w - p.pad_w;
                const int hb = p0 * p.stride_h - p.pad_h;
                for (int kb = 0; kb < p.num_kb; ++kb, ++g) {
                    if (g % kNumProducers != pi) continue;
                    const int stage = g % NS;
                    const uint32_t phase = static_cast<uint32_t>(g / NS) & 1u;
                    mbar_wait(&empty[stage], phase ^ 1u);
                    if (leader) trace_ev(p, 0, g);
                    const bool skip_b = (p.exp_flags & 1) && tile != static_cast<int>(blockIdx.x) && g >= NS;
                    const bool skip_a = (p.exp_flags & 2) && tile != static_cast<int>(blockIdx.x) && g >= NS;
                    if (leader) mbar_arrive_expect_tx(&full[stage], (skip_b ? tx - static_cast<uint32_t>(p.BN * p.BK) : tx) -
                                                            (skip_a ? static_cast<uint32_t>(kBM * p.bkp) : 0u));
                    if (p.pair) {
                        const int RS = p.R * p.S;
                        const int t0 = 2 * kb, t1 = t0 + 1;
                        const int r0 = t0 / p.S, s0 = t0 - r0 * p.S;
                        int r1 = r0, s1 = s0, kg1 = RS * 16;        // odd tail: B slot OOB -> 0
                        if (t1 < RS) { r1 = t1 / p.S; s1 = t1 - r1 * p.S; kg1 = t1 * 16; }
                        uint8_t *adst = smem + p.off_a + stage * p.a_stage_bytes;
                        uint8_t *bdst = smem + p.off_b + stage * p.b_stage_bytes;
                        if (leader) tma_load_im2col_4d(adst, &xmap, &full[stage], 0, wb, hb, img,
                                           static_cast<uint16_t>(s0 * p.dil_w), static_cast<uint16_t>(r0 * p.dil_h));
                        if (leader) tma_load_im2col_4d(adst + kBM * 16, &xmap, &full[stage], 0, wb, hb, img,
                                           static_cast<uint16_t>(s1 * p.dil_w), static_cast<uint16_t>(r1 * p.dil_h));
                        if (leader) tma_load_2d(bdst, &wmap, &full[stage], t0 * 16, n0);
                        if (leader) tma_load_2d(bdst + p.BN * 16, &wmap, &full[stage], kg1, n0);
                    } else {
                        const int r = kb / taps_per_r;
                        const int rem2 = kb - r * taps_per_r;
                        const int s = rem2 / p.chunks;
                        const int ch = rem2 - s * p.chunks;
                        uint8_t *adst = IS4 ? smem + p.off_stg + stage * p.stg_stage_bytes
                                            : smem + p.off_a + stage * p.a_stage_bytes;
                        if (!skip_a)
                            if (leader) tma_load_im2col_4d(adst, &xmap, &full[stage], ch * p.bkp, wb, hb, img,
                                               static_cast<uint16_t>(s * p.dil_w),
                                               static_cast<uint16_t>(r * p.dil_h));
                        if (!skip_b)
                            if (leader) tma_load_2d(smem + p.off_b + stage * p.b_stage_bytes, &wmap, &full[stage],
                                        (r * p.S + s) * p.C8 + ch * p.BK, n0);
                    }
                }
            }
        }
    } else if (warp == kWarpMMA) {
        // ===================== MMA issuer (whole warp, one elected lane issues) =============
        // Warp-uniform issue (measured, scripts/micro/commit_bench.cu): ~72 cycles per
        // 128xNx32 MMA and a free per-stage commit at N=256, versus ~150 cycles per MMA for a
        // lane-0-only loop.
        {
            const bool leader = lane == 0;
            int stage = 0;
            uint32_t phase = 0;
            int it = 0;
            int gstage = 0;
            const uint32_t sbo = 8u * static_cast<uint32_t>(p.BK);
            const int ksteps = p.BK / 32;
            for (int tile = blockIdx.x; tile < p.num_tiles; tile += gridDim.x, ++it) {
                const int buf = it & 1;
                const uint32_t acc_phase = static_cast<uint32_t>(it >> 1) & 1u;
                mbar_wait(&tempty[buf], acc_phase ^ 1u);
                if (leader) trace_ev(p, 2, it);
                __syncwarp();
                tc_fence_after();
                const uint32_t d_tmem = tmem_base + static_cast<uint32_t>(buf * p.BN);
                for (int kb = 0; kb < p.num_kb; ++kb) {
                    mbar_wait(IS4 ? &aready[stage] : &full[stage], phase);
                    if (leader) trace_ev(p, 3, gstage);
                    ++gstage;
                    __syncwarp();
                    tc_fence_after();
                    const uint32_t a_addr = smem_u32(smem + p.off_a + stage * p.a_stage_bytes);
                    const uint32_t b_addr = smem_u32(smem + p.off_b + stage * p.b_stage_bytes);
                    if (p.pair) {
                        // canonical no-swizzle K-major: core matrices 8 rows x 16 B; the two
                        // 16-byte K halves (filter taps) are LBO apart, 8-row groups SBO = 128 B
                        const uint64_t ad = make_smem_desc(a_addr, kBM * 16u, 128u, 0u);
                        const uint64_t bd = make_smem_desc(b_addr, static_cast<uint32_t>(p.BN) * 16u, 128u, 0u);
                        mma_i8_warp(d_tmem, ad, bd, p.idesc, kb != 0 ? 1u : 0u);
                    } else {
                        const uint64_t ad0 = make_smem_desc(a_addr, 16u, sbo, p.sw_layout);
                        const uint64_t bd0 = make_smem_desc(b_addr, 16u, sbo, p.sw_layout);
                        const uint32_t alo = static_cast<uint32_t>(ad0), ahi = static_cast<uint32_t>(ad0 >> 32);
                        const uint32_t blo = static_cast<uint32_t>(bd0), bhi = static_cast<uint32_t>(bd0 >> 32);
                        if (ksteps == 4) {
#pragma unroll
                            for (int k = 0; k < 4; ++k)
                                if (!(p.exp_flags & 4) || (kb | k) == 0)
                                    mma_i8_warp_lo(d_tmem, alo + 2u * k, ahi, blo + 2u * k, bhi, p.idesc,
                                                   (kb | k) != 0 ? 1u : 0u);
                        } else {
                            for (int k = 0; k < ksteps; ++k)
                                if (!(p.exp_flags & 4) || (kb | k) == 0)
                                    mma_i8_warp_lo(d_tmem, alo + 2u * k, ahi, blo + 2u * k, bhi, p.idesc,
                                                   (kb | k) != 0 ? 1u : 0u);
                        }
                    }
                    mma_commit_warp(&empty[stage]);
                    if (++stage == NS) { stage = 0; phase ^= 1u; }
                }
                mma_commit_warp(&tfull[buf]);
                if (leader) trace_ev(p, 4, it);
            }
        }
    } else if (warp >= kWarpEpi0 && warp < kWarpEpi0 + kNumEpiWarps) {
        // ===================== epilogue (8 warps: lane quarter = warp%4, column half) ============
        griddep_wait();                                   // params / tables written in-stream
        const int ew = warp - kWarpEpi0;                 // 0..7
        const int quarter = warp & 3;                    // TMEM lanes 32*quarter .. +31
        const int half = ew >> 2;                        // which 32-column chunks
        const int row = quarter * 32 + lane;
        const uint32_t par_base = smem_u32(par);
        const int nchunks = (p.BN + 31) / 32;
        const bool force_general = (OUT == OUT_S32) || ZX;
        int cached_n0 = -1;
        int it = 0;
        const uint32_t ystg_base = smem_u32(smem + p.off_ystg);
        for (int tile = blockIdx.x; tile < p.num_tiles; tile += gridDim.x, ++it) {
            const int buf = it & 1;
            const uint32_t acc_phase = static_cast<uint32_t>(it >> 1) & 1u;
            const int m0 = (tile / p.n_tiles_n) * kBM;
            const int n0 = (tile % p.n_tiles_n) * p.BN;
            if (n0 != cached_n0) {
                fill_epilogue_params<OUT>(p, par, chunk_info, n0, ew, lane, force_general);
                cached_n0 = n0;
            }
            const int64_t m = static_cast<int64_t>(m0) + row;
            const bool row_ok = m < p.M;
            int zr0 = 0, zr1 = 0, zs0 = 0, zs1 = 0;
            if (ZX) {
                const int mm = row_ok ? static_cast<int>(m) : 0;
                const int rem = mm % p.PQ;
                const int pp = rem / p.Q;
                const int qq = rem - pp * p.Q;
                valid_tap_range(pp, p.stride_h, p.pad_h, p.dil_h, p.H, p.R, zr0, zr1);
                valid_tap_range(qq, p.stride_w, p.pad_w, p.dil_w, p.W, p.S, zs0, zs1);
            }
            mbar_wait(&tfull[buf], acc_phase);
            if (ew == 0 && lane == 0) trace_ev(p, 5, it);
            tc_fence_after();
            const uint32_t taddr = tmem_base + (static_cast<uint32_t>(quarter * 32) << 16) +
                                   static_cast<uint32_t>(buf * p.BN);
            uint32_t v[32];
            if (OUT != OUT_S32 && p.y_tma) {
                // whole-tile staging in smem, written back by TMA stores of [128 rows x y_gw]
                // groups (full 32..128-byte rows; rows >= M and columns >= K clipped by the map)
                const bool storer = ew == 0 && lane == 0;
                if (storer) bulk_wait_read<1>();          // the store that used this buffer is done
                named_bar_sync(1, kNumEpiWarps * 32);
                const uint32_t ystg_it = ystg_base + static_cast<uint32_t>(it & 1) * p.ystg_bytes;
                // TMEM loads double-buffered: chunk ci+2 is in flight while chunk ci is requantized
                uint32_t (&va)[32] = v;
                uint32_t vb[32];
                auto process = [&](uint32_t (&vv)[32], int ci) {
                    const int col0 = ci * 32;
                    const uint32_t pa = par_base + 16u * col0;
                    const int4 cinfo = chunk_info[ci];
                    if (p.exp_flags & 48) {            // experiment: TMEM loads only
                        uint32_t x = 0;
                        for (int j = 0; j < 32; ++j) x ^= vv[j];
                        if (x == 0x9e3779b9u && col0 == 12345) asm volatile("trap;");
                        return;
                    }
                    epi_requant16<OUT, ZX, 0>(p, vv, pa, cinfo, n0 + col0, zr0, zr1, zs0, zs1);
                    epi_requant16<OUT, ZX, 16>(p, vv, pa, cinfo, n0 + col0, zr0, zr1, zs0, zs1);
                    if (p.exp_flags & 64) {            // experiment: no staging stores
                        if (vv[0] == 0x9e3779b9u && col0 == 12345) asm volatile("trap;");
                        return;
                    }
                    stage16<OUT, 0>(p, vv, ystg_it, row, col0);
                    stage16<OUT, 16>(p, vv, ystg_it, row, col0 + 16);
                };
                if (!IS4) {   // 8-bit kernels (384 threads) have the registers to double-buffer
                    __syncwarp();
                    if (half < nchunks) tmem_ld_32x32b_x32(taddr + half * 32, va);
                    for (int ci = half; ci < nchunks; ci += 4) {
                        tmem_wait_ld();
                        __syncwarp();
                        if (ci + 2 < nchunks) tmem_ld_32x32b_x32(taddr + (ci + 2) * 32, vb);
                        process(va, ci);
                        if (ci + 2 >= nchunks) break;
                        tmem_wait_ld();
                        __syncwarp();
                        if (ci + 4 < nchunks) tmem_ld_32x32b_x32(taddr + (ci + 4) * 32, va);
                        process(vb, ci + 2);
                    }
                } else {
                    for (int ci = half; ci < nchunks; ci += 2) {
                        __syncwarp();
                        tmem_ld_32x32b_x32(taddr + ci * 32, va);
                        tmem_wait_ld();
                        process(va, ci);
                    }
                }
                tc_fence_before();
                __syncwarp();
                if (lane == 0) mbar_arrive(&tempty[buf]);    // accumulator drained: MMA may reuse it
                if (ew == 0 && lane == 0) trace_ev(p, 6, it);
                fence_proxy_async_smem();
                named_bar_sync(1, kNumEpiWarps * 32);
                if (storer && !(p.exp_flags & 128)) {
                    constexpr int kBits = (OUT == OUT_U4 || OUT == OUT_S4) ? 4 : 8;
                    for (int g = 0; g < p.n_ygroups; ++g)
                        tma_store_2d(&ymap, smem + p.off_ystg + (it & 1) * p.ystg_bytes + g * 128 * p.y_gw,
                                     n0 * kBits / 8 + g * p.y_gw, m0);
                    bulk_commit();
                    trace_ev(p, 7, it);
                }
                continue;
            } else {
                for (int ci = half; ci < nchunks; ci += 2) {
                    const int col0 = ci * 32;
                    const int nc = min(32, p.BN - col0);
                    __syncwarp();
                    if (nc == 32) tmem_ld_32x32b_x32(taddr + col0, v);
                    else tmem_ld_32x32b_x16(taddr + col0, v);
                    tmem_wait_ld();
                    const uint32_t pa = par_base + 16u * col0;
                    const int4 cinfo = chunk_info[ci];
                    epi_half<OUT, ZX, 0>(p, v, pa, cinfo, n0 + col0, m, row_ok, zr0, zr1, zs0, zs1);
                    if (nc == 32)
                        epi_half<OUT, ZX, 16>(p, v, pa, cinfo, n0 + col0 + 16, m, row_ok, zr0, zr1, zs0, zs1);
                }
            }
            tc_fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive(&tempty[buf]);
        }
        if (OUT != OUT_S32 && p.y_tma && ew == 0 && lane == 0) bulk_wait<0>();
    } else if (IS4 && warp >= kWarpCvt0 && warp < kWarpCvt0 + kNumCvtWarps) {
        // ===================== int4 -> int8 widening (4 warps) =====================
        const int ct = (warp - kWarpCvt0) * 32 + lane;      // 0..127
        int cstage = 0;
        const int cshift = p.cvt_shift;                      // log2(16-byte packed chunks/pixel)
        const int nchunks = kBM << cshift;
        const uint32_t xo = p.x_sgn4 ? 0x88888888u : 0u;
        const uint32_t sw = static_cast<uint32_t>(p.sw_mask);
        const uint32_t bkb = static_cast<uint32_t>(p.BK);
        int stage = 0;
        uint32_t phase = 0;
        for (int tile = blockIdx.x; tile < p.num_tiles; tile += gridDim.x) {
            for (int kb = 0; kb < p.num_kb; ++kb) {
                mbar_wait(&full[stage], phase);
                if (ct == 0) trace_ev(p, 8, cstage++);
                const uint32_t stg = smem_u32(smem + p.off_stg + stage * p.stg_stage_bytes);
                const uint32_t adst = smem_u32(smem + p.off_a + stage * p.a_stage_bytes);
                widen_stage(stg, adst, ct, nchunks, cshift, bkb, sw, xo, static_cast<uint32_t>(p.stg_sw));
                fence_proxy_async_smem();
                __syncwarp();
                if (lane == 0) mbar_arrive(&aready[stage]);
                if (ct == 0) trace_ev(p, 9, cstage - 1);
                if (++stage == NS) { stage = 0; phase ^= 1u; }
            }
        }
    }

    tc_fence_before();
    __syncthreads();
    if (warp == kWarpMMA) {
        __syncwarp();
        tc_fence_after();
        tmem_dealloc(tmem_base, p.tmem_cols);
    }
}

// Debug: one im2col TMA tile straight to global memory (no swizzle).
__global__ void qconv_debug_im2col_kernel(const __grid_constant__ CUtensorMap xmap, int32_t c,
                                          int32_t w, int32_t h, int32_t n, uint16_t ow,
                                          uint16_t oh, uint32_t bytes, uint8_t *out) {
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                                ~uintptr_t(1023));
    __shared__ __align__(8) uint64_t bar;
    if (threadIdx.x == 0) {
        mbar_init(&bar, 1);
        fence_mbar_init();
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        mbar_arrive_expect_tx(&bar, bytes);
        tma_load_im2col_4d(smem, &xmap, &bar, c, w, h, n, ow, oh);
    }
    mbar_wait(&bar, 0);
    for (uint32_t i = threadIdx.x; i < bytes; i += blockDim.x) out[i] = smem[i];
}

}  // namespace qc
