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
//     warps 4-7 run the epilogue, (4-bit) warps 8-11 widen int4 to int8.
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
constexpr int kWarpEpi0 = 4;         // warps 4..7: epilogue (TMEM lane quarters 0..3)
constexpr int kNumEpiWarps = 4;
constexpr int kWarpCvt0 = 8;         // warps 8..11: int4 -> int8 converters (4-bit only)
constexpr int kNumCvtWarps = 4;

enum OutKind { OUT_S32 = 0, OUT_U8 = 1, OUT_S8 = 2, OUT_U4 = 3, OUT_S4 = 4 };

struct ConvParams {
    // GEMM geometry
    int32_t M, P, Q, PQ, K;
    int32_t BN, n_tiles_n, num_tiles, num_kb, chunks, S;
    int32_t stride_h, stride_w, pad_h, pad_w, dil_h, dil_w;
    int32_t H, W, R, C8;              // C8 = channels (int8 bytes per pixel after widening)
    int32_t BK, bkp, stages, sw_layout, sw_mask;
    uint32_t idesc, tmem_cols;
    // shared memory carve-up (byte offsets from the 1024-aligned base)
    uint32_t off_a, off_b, off_stg, off_bar, off_par;
    uint32_t a_stage_bytes, b_stage_bytes, stg_stage_bytes;
    // epilogue
    int32_t y_zero, clamp_lo, clamp_hi, x_zero;
    const int32_t *bias, *mult, *shift;
    const int32_t *zx_table;          // [K][(R+1)*(S+1)] inclusive 2-D prefix sums of sum_c w
    void *y;
    int64_t y_row_bytes;
};

// ------------------------------------------------------------------ epilogue helpers
// Per-column re-quantization constants (built once per N tile into smem):
//   mode 0 (shift in [32,52]): t+zy = hi32(acc*m + C) >> (shift-32),
//          C = bias*m + 2^(shift-1) + zy*2^shift   (exact)
//   mode 1 (other shifts):     t = (acc*m + C) >> shift (int64), C = bias*m + 2^(shift-1)
//   S32:                       y = acc + bias
struct __align__(16) ColParam {
    int32_t m;
    int32_t shm;     // shift amount | mode << 8
    int64_t c;
};

__device__ __forceinline__ ColParam make_col_param(const ConvParams &p, int k, bool s32) {
    ColParam cp;
    const int32_t b = (p.bias && k < p.K) ? __ldg(p.bias + k) : 0;
    if (s32 || k >= p.K) {
        cp.m = 0; cp.shm = 0; cp.c = b;
        return cp;
    }
    const int32_t m = __ldg(p.mult + k);
    const int32_t n = __ldg(p.shift + k);
    const int64_t prod = static_cast<int64_t>(b) * m + (static_cast<int64_t>(1) << (n - 1));
    cp.m = m;
    if (n >= 32 && n <= 52) {
        cp.c = prod + (static_cast<int64_t>(p.y_zero) << n);
        cp.shm = n - 32;
    } else {
        cp.c = prod;
        cp.shm = n | (1 << 8);
    }
    return cp;
}

template <int OUT>
__device__ __forceinline__ int32_t requant_one(int32_t acc, const ColParam &cp, int32_t lo,
                                               int32_t hi, int32_t zy) {
    if (OUT == OUT_S32) return acc + static_cast<int32_t>(cp.c);
    int32_t y;
    if ((cp.shm >> 8) == 0) {
        const int64_t prod = static_cast<int64_t>(acc) * cp.m + cp.c;   // mad.wide.s32
        y = static_cast<int32_t>(prod >> 32) >> (cp.shm & 63);
    } else {
        const int64_t prod = static_cast<int64_t>(acc) * cp.m + cp.c;
        int64_t t = prod >> (cp.shm & 63);
        const int64_t lo64 = static_cast<int64_t>(lo) - zy, hi64 = static_cast<int64_t>(hi) - zy;
        t = t < lo64 ? lo64 : (t > hi64 ? hi64 : t);
        y = static_cast<int32_t>(t) + zy;
    }
    return min(hi, max(lo, y));
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

// Process NC (16 or 32) accumulator columns of one output row and store them.
template <int OUT, int NC>
__device__ __forceinline__ void epilogue_chunk(const ConvParams &p, const uint32_t (&v)[32],
                                               const ColParam *par, int col0, int n0, int64_t m,
                                               bool row_ok, int zx_r0, int zx_r1, int zx_s0,
                                               int zx_s1) {
    int32_t yv[NC];
#pragma unroll
    for (int j = 0; j < NC; ++j) {
        int32_t acc = static_cast<int32_t>(v[j]);
        if (p.x_zero != 0) {
            const int k = n0 + col0 + j;
            if (k < p.K) {
                const int RS1 = p.S + 1;
                const int32_t *t = p.zx_table + static_cast<int64_t>(k) * (p.R + 1) * RS1;
                const int32_t rect = __ldg(t + zx_r1 * RS1 + zx_s1) - __ldg(t + zx_r0 * RS1 + zx_s1) -
                                     __ldg(t + zx_r1 * RS1 + zx_s0) + __ldg(t + zx_r0 * RS1 + zx_s0);
                acc -= p.x_zero * rect;
            }
        }
        const ColParam cp = par[col0 + j];
        yv[j] = requant_one<OUT>(acc, cp, p.clamp_lo, p.clamp_hi, p.y_zero);
    }
    if (!row_ok) return;
    const int kc = n0 + col0;                    // first output channel of the chunk
    const bool in_range = kc + NC <= p.K;
    if (OUT == OUT_S32) {
        int32_t *dst = reinterpret_cast<int32_t *>(static_cast<uint8_t *>(p.y) + m * p.y_row_bytes) + kc;
        if (in_range && (reinterpret_cast<uintptr_t>(dst) & 15u) == 0) {
#pragma unroll
            for (int j = 0; j < NC; j += 4) st_global_v4(dst + j, yv[j], yv[j + 1], yv[j + 2], yv[j + 3]);
        } else {
            for (int j = 0; j < NC && kc + j < p.K; ++j) dst[j] = yv[j];
        }
    } else if (OUT == OUT_U8 || OUT == OUT_S8) {
        uint32_t w[NC / 4];
#pragma unroll
        for (int j = 0; j < NC / 4; ++j) {
            if (OUT == OUT_U8)
                w[j] = pack_sat_u8(yv[4 * j + 1], yv[4 * j], pack_sat_u8(yv[4 * j + 3], yv[4 * j + 2], 0u));
            else
                w[j] = pack_sat_s8(yv[4 * j + 1], yv[4 * j], pack_sat_s8(yv[4 * j + 3], yv[4 * j + 2], 0u));
        }
        uint8_t *dst = static_cast<uint8_t *>(p.y) + m * p.y_row_bytes + kc;
        if (in_range && (reinterpret_cast<uintptr_t>(dst) & 15u) == 0) {
#pragma unroll
            for (int j = 0; j < NC / 4; j += 4) st_global_v4(dst + 4 * j, w[j], w[j + 1], w[j + 2], w[j + 3]);
        } else {
            for (int j = 0; j < NC && kc + j < p.K; ++j) dst[j] = static_cast<uint8_t>(w[j >> 2] >> (8 * (j & 3)));
        }
    } else {
        uint32_t w[NC / 8];
#pragma unroll
        for (int j = 0; j < NC / 8; ++j) {
            const int b = 8 * j;
            if (OUT == OUT_U4) {
                uint32_t t = pack_sat_u4(yv[b + 7], yv[b + 6], 0u);
                t = pack_sat_u4(yv[b + 5], yv[b + 4], t);
                t = pack_sat_u4(yv[b + 3], yv[b + 2], t);
                w[j] = pack_sat_u4(yv[b + 1], yv[b], t);
            } else {
                uint32_t t = pack_sat_s4(yv[b + 7], yv[b + 6], 0u);
                t = pack_sat_s4(yv[b + 5], yv[b + 4], t);
                t = pack_sat_s4(yv[b + 3], yv[b + 2], t);
                w[j] = pack_sat_s4(yv[b + 1], yv[b], t);
            }
        }
        uint8_t *dst = static_cast<uint8_t *>(p.y) + m * p.y_row_bytes + kc / 2;
        if (in_range && (reinterpret_cast<uintptr_t>(dst) & (NC == 32 ? 15u : 7u)) == 0) {
            if (NC == 32) st_global_v4(dst, w[0], w[1], w[2], w[3]);
            else *reinterpret_cast<uint2 *>(dst) = make_uint2(w[0], w[1]);
        } else {
            for (int j = 0; 2 * j < NC && kc + 2 * j < p.K; ++j)
                dst[j] = static_cast<uint8_t>(w[j >> 2] >> (8 * (j & 3)));
        }
    }
}

// ------------------------------------------------------------------ the kernel
template <bool IS4, int OUT>
__global__ void __launch_bounds__(IS4 ? 384 : 256, 1)
qconv_fwd_kernel(const __grid_constant__ CUtensorMap xmap, const __grid_constant__ CUtensorMap wmap,
                 const __grid_constant__ ConvParams p) {
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
    ColParam *par = reinterpret_cast<ColParam *>(smem + p.off_par);

    if (warp == kWarpTMA && lane == 0) {
        tma_prefetch_desc(&xmap);
        tma_prefetch_desc(&wmap);
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

    if (warp == kWarpTMA) {
        // ===================== TMA producer (one thread) =====================
        if (lane == 0) {
            int stage = 0;
            uint32_t phase = 0;
            const uint32_t tx = static_cast<uint32_t>(kBM * p.bkp + p.BN * p.BK);
            for (int tile = blockIdx.x; tile < p.num_tiles; tile += gridDim.x) {
                const int m0 = (tile / p.n_tiles_n) * kBM;
                const int n0 = (tile % p.n_tiles_n) * p.BN;
                const int img = m0 / p.PQ;
                const int rem = m0 - img * p.PQ;
                const int p0 = rem / p.Q;
                const int q0 = rem - p0 * p.Q;
                const int wb = q0 * p.stride_w - p.pad_w;
                const int hb = p0 * p.stride_h - p.pad_h;
                for (int kb = 0; kb < p.num_kb; ++kb) {
                    const int r = kb / taps_per_r;
                    const int rem2 = kb - r * taps_per_r;
                    const int s = rem2 / p.chunks;
                    const int ch = rem2 - s * p.chunks;
                    mbar_wait(&empty[stage], phase ^ 1u);
                    mbar_arrive_expect_tx(&full[stage], tx);
                    uint8_t *adst = IS4 ? smem + p.off_stg + stage * p.stg_stage_bytes
                                        : smem + p.off_a + stage * p.a_stage_bytes;
                    tma_load_im2col_4d(adst, &xmap, &full[stage], ch * p.bkp, wb, hb, img,
                                       static_cast<uint16_t>(s * p.dil_w),
                                       static_cast<uint16_t>(r * p.dil_h));
                    tma_load_2d(smem + p.off_b + stage * p.b_stage_bytes, &wmap, &full[stage],
                                (r * p.S + s) * p.C8 + ch * p.BK, n0);
                    if (++stage == NS) { stage = 0; phase ^= 1u; }
                }
            }
        }
    } else if (warp == kWarpMMA) {
        // ===================== MMA issuer (one thread) =====================
        if (lane == 0) {
            int stage = 0;
            uint32_t phase = 0;
            int it = 0;
            const uint32_t sbo = 8u * static_cast<uint32_t>(p.BK);
            const int ksteps = p.BK / 32;
            for (int tile = blockIdx.x; tile < p.num_tiles; tile += gridDim.x, ++it) {
                const int buf = it & 1;
                const uint32_t acc_phase = static_cast<uint32_t>(it >> 1) & 1u;
                mbar_wait(&tempty[buf], acc_phase ^ 1u);
                tc_fence_after();
                const uint32_t d_tmem = tmem_base + static_cast<uint32_t>(buf * p.BN);
                for (int kb = 0; kb < p.num_kb; ++kb) {
                    mbar_wait(IS4 ? &aready[stage] : &full[stage], phase);
                    tc_fence_after();
                    const uint32_t a_addr = smem_u32(smem + p.off_a + stage * p.a_stage_bytes);
                    const uint32_t b_addr = smem_u32(smem + p.off_b + stage * p.b_stage_bytes);
                    for (int k = 0; k < ksteps; ++k) {
                        const uint64_t ad = make_smem_desc(a_addr + 32u * k, 16u, sbo, p.sw_layout);
                        const uint64_t bd = make_smem_desc(b_addr + 32u * k, 16u, sbo, p.sw_layout);
                        mma_i8(d_tmem, ad, bd, p.idesc, (kb | k) != 0 ? 1u : 0u);
                    }
                    mma_commit(&empty[stage]);
                    if (++stage == NS) { stage = 0; phase ^= 1u; }
                }
                mma_commit(&tfull[buf]);
            }
        }
    } else if (warp >= kWarpEpi0 && warp < kWarpEpi0 + kNumEpiWarps) {
        // ===================== epilogue (4 warps, one TMEM lane quarter each) =====================
        const int quarter = warp & 3;
        const int row = quarter * 32 + lane;
        const int et = (warp - kWarpEpi0) * 32 + lane;     // 0..127
        int cached_n0 = -1;
        int it = 0;
        for (int tile = blockIdx.x; tile < p.num_tiles; tile += gridDim.x, ++it) {
            const int buf = it & 1;
            const uint32_t acc_phase = static_cast<uint32_t>(it >> 1) & 1u;
            const int m0 = (tile / p.n_tiles_n) * kBM;
            const int n0 = (tile % p.n_tiles_n) * p.BN;
            if (n0 != cached_n0) {
                named_bar_sync(1, kNumEpiWarps * 32);
                for (int c = et; c < p.BN; c += kNumEpiWarps * 32)
                    par[c] = make_col_param(p, n0 + c, OUT == OUT_S32);
                named_bar_sync(1, kNumEpiWarps * 32);
                cached_n0 = n0;
            }
            const int64_t m = static_cast<int64_t>(m0) + row;
            const bool row_ok = m < p.M;
            int zr0 = 0, zr1 = 0, zs0 = 0, zs1 = 0;
            if (p.x_zero != 0) {
                const int mm = row_ok ? static_cast<int>(m) : 0;
                const int rem = mm % p.PQ;
                const int pp = rem / p.Q;
                const int qq = rem - pp * p.Q;
                valid_tap_range(pp, p.stride_h, p.pad_h, p.dil_h, p.H, p.R, zr0, zr1);
                valid_tap_range(qq, p.stride_w, p.pad_w, p.dil_w, p.W, p.S, zs0, zs1);
            }
            mbar_wait(&tfull[buf], acc_phase);
            tc_fence_after();
            const uint32_t taddr = tmem_base + (static_cast<uint32_t>(quarter * 32) << 16) +
                                   static_cast<uint32_t>(buf * p.BN);
            uint32_t v[32];
            int col0 = 0;
            for (; col0 + 32 <= p.BN; col0 += 32) {
                __syncwarp();
                tmem_ld_32x32b_x32(taddr + col0, v);
                tmem_wait_ld();
                epilogue_chunk<OUT, 32>(p, v, par, col0, n0, m, row_ok, zr0, zr1, zs0, zs1);
            }
            if (col0 < p.BN) {
                __syncwarp();
                tmem_ld_32x32b_x16(taddr + col0, v);
                tmem_wait_ld();
                epilogue_chunk<OUT, 16>(p, v, par, col0, n0, m, row_ok, zr0, zr1, zs0, zs1);
            }
            tc_fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive(&tempty[buf]);
        }
    } else if (IS4 && warp >= kWarpCvt0 && warp < kWarpCvt0 + kNumCvtWarps) {
        // ===================== int4 -> int8 widening (4 warps) =====================
        const int ct = (warp - kWarpCvt0) * 32 + lane;      // 0..127
        const int chunks_per_row = p.bkp / 16;               // 16-byte packed chunks per pixel
        const int nchunks = kBM * chunks_per_row;
        const bool sgn = ((p.idesc >> 7) & 1u) != 0;
        int stage = 0;
        uint32_t phase = 0;
        for (int tile = blockIdx.x; tile < p.num_tiles; tile += gridDim.x) {
            for (int kb = 0; kb < p.num_kb; ++kb) {
                mbar_wait(&full[stage], phase);
                const uint8_t *stg = smem + p.off_stg + stage * p.stg_stage_bytes;
                uint8_t *adst = smem + p.off_a + stage * p.a_stage_bytes;
                for (int g = ct; g < nchunks; g += kNumCvtWarps * 32) {
                    const int rr = g / chunks_per_row;
                    const int cir = g - rr * chunks_per_row;
                    const uint4 pk = *reinterpret_cast<const uint4 *>(stg + 16 * g);
                    const uint32_t src[4] = {pk.x, pk.y, pk.z, pk.w};
                    uint32_t o[8];
#pragma unroll
                    for (int j = 0; j < 4; ++j) {
                        uint32_t lo = src[j] & 0x0F0F0F0Fu;
                        uint32_t hi = (src[j] >> 4) & 0x0F0F0F0Fu;
                        if (sgn) {
                            lo = ((lo ^ 0x08080808u) + 0x78787878u) ^ 0x80808080u;
                            hi = ((hi ^ 0x08080808u) + 0x78787878u) ^ 0x80808080u;
                        }
                        o[2 * j] = __byte_perm(lo, hi, 0x5140);
                        o[2 * j + 1] = __byte_perm(lo, hi, 0x7362);
                    }
                    // widened bytes [32*cir, 32*cir+32) of row rr, swizzled like the TMA would
                    const uint32_t off0 = static_cast<uint32_t>(rr * p.BK + 32 * cir);
                    const uint32_t off1 = off0 + 16u;
                    const uint32_t sw = static_cast<uint32_t>(p.sw_mask);
                    const uint32_t ph0 = off0 ^ (((off0 >> 7) & sw) << 4);
                    const uint32_t ph1 = off1 ^ (((off1 >> 7) & sw) << 4);
                    *reinterpret_cast<uint4 *>(adst + ph0) = make_uint4(o[0], o[1], o[2], o[3]);
                    *reinterpret_cast<uint4 *>(adst + ph1) = make_uint4(o[4], o[5], o[6], o[7]);
                }
                fence_proxy_async_smem();
                __syncwarp();
                if (lane == 0) mbar_arrive(&aready[stage]);
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
