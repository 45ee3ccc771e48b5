// trans.cuh -- channel-major ("transposed") variant of the implicit-GEMM conv for
// 1x1 convolutions, whose cost is dominated by the fused epilogue.
//
// Same method (Alg.2, epilogue P:L223/P:L253/P:L265), operands swapped:
// the UMMA computes D^T = W * X^T with M = BMc output channels (weights as the A
// operand) and N = BNp output pixels (im2col activations as the B operand).  A TMEM
// lane is then one output channel, so each epilogue thread keeps its channel's
// re-quantization constants in registers (no per-element shared-memory loads): per
// output one IMAD.HI (with the 64-bit bias/rounding addend), one shift and one
// saturating pack.  The byte-per-channel results of 32 lanes form 32 contiguous
// bytes of an NHWC row, staged in shared memory and written by TMA stores.
#pragma once
#include "conv_fwd.cuh"

namespace qc {

struct TChan {          // per-channel constants held in registers by the epilogue thread
    int64_t c64;        // fast/mid: 64-bit addend of the IMAD.HI (bias*m, rounding, zero point)
    int32_t m, sh, b, k, vlim, n, mode;
};

// Re-quantize one 32-pixel chunk of this thread's channel (Eq.(3)-(4)) and
// store its bytes into the staging rows (row = pixel, stride ROWB bytes).  `mode` is warp
// uniform: 0 fast (shift 33..52), 1 mid (shift 20..50), 2 general.
template <int OUT, int ROWB>
__device__ __forceinline__ void t_chunk(const ConvParams &p, const TChan &cp, uint32_t (&v)[32],
                                        uint32_t ystg, int lane, bool lane_ok) {
    constexpr bool kInt4 = (OUT == OUT_U4 || OUT == OUT_S4);
    int32_t *y = reinterpret_cast<int32_t *>(v);
    if (cp.mode == 0) {
#pragma unroll
        for (int j = 0; j < 32; ++j) {
            const int64_t prod = static_cast<int64_t>(static_cast<int32_t>(v[j])) * cp.m + cp.c64;
            y[j] = static_cast<int32_t>(prod >> 32) >> cp.sh;
        }
    } else if (cp.mode == 1) {
#pragma unroll
        for (int j = 0; j < 32; ++j) {
            int32_t x = static_cast<int32_t>(v[j]) + cp.b;
            x = min(cp.vlim, max(-cp.vlim, x)) << cp.k;
            const int64_t prod = static_cast<int64_t>(x) * cp.m + cp.c64;
            y[j] = static_cast<int32_t>(prod >> 32) >> cp.sh;
        }
    } else {
        const int64_t lo64 = static_cast<int64_t>(p.clamp_lo) - p.y_zero;
        const int64_t hi64 = static_cast<int64_t>(p.clamp_hi) - p.y_zero;
#pragma unroll
        for (int j = 0; j < 32; ++j) {
            const int64_t prod = static_cast<int64_t>((static_cast<int32_t>(v[j]) >> p.acc_lg) + cp.b) * cp.m +
                                 (static_cast<int64_t>(1) << (cp.n - 1));
            int64_t t = prod >> cp.n;
            t = t < lo64 ? lo64 : (t > hi64 ? hi64 : t);
            y[j] = static_cast<int32_t>(t) + p.y_zero;
        }
    }
    if (p.need_clamp) {
#pragma unroll
        for (int j = 0; j < 32; ++j) y[j] = min(p.clamp_hi, max(p.clamp_lo, y[j]));
    }
    if (kInt4) {
        // channel pair (2i, 2i+1) shares a byte: the even lane writes pixels 0..15 of the
        // chunk, the odd lane pixels 16..31, each fetching its partner's half
        const bool odd = lane & 1;
        const uint32_t base = ystg + (odd ? 16u * ROWB : 0u);
#pragma unroll
        for (int j = 0; j < 16; ++j) {
            const int32_t mine = odd ? y[j + 16] : y[j];
            const int32_t give = odd ? y[j] : y[j + 16];
            const int32_t other = __shfl_xor_sync(0xffffffffu, give, 1);
            const int32_t lo = odd ? other : mine;
            const int32_t hi = odd ? mine : other;
            const uint32_t byte = OUT == OUT_U4 ? pack_sat_u4(hi, lo, 0u) : pack_sat_s4(hi, lo, 0u);
            if (lane_ok) asm volatile("st.shared.u8 [%0], %1;" ::"r"(base + j * ROWB), "r"(byte));
        }
    } else {
#pragma unroll
        for (int j = 0; j < 32; ++j) {
            const uint32_t byte = OUT == OUT_U8 ? pack_sat_u8(0, y[j], 0u) : pack_sat_s8(0, y[j], 0u);
            if (lane_ok) asm volatile("st.shared.u8 [%0], %1;" ::"r"(ystg + j * ROWB), "r"(byte));
        }
    }
}

template <bool IS4, int OUT, bool M64>
__global__ void __launch_bounds__(IS4 ? 512 : 384, 1)
qconv_t_kernel(const __grid_constant__ CUtensorMap xmap, const __grid_constant__ CUtensorMap wmap,
               const __grid_constant__ CUtensorMap ymap, const __grid_constant__ ConvParams p) {
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                                ~uintptr_t(1023));
    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;
    const int NS = p.stages;
    constexpr int BMc = M64 ? 64 : 128;   // output channels per tile (UMMA M)
    constexpr int kBNp = 256;             // output pixels per tile (UMMA N)
    constexpr int BNp = kBNp;
    constexpr bool kInt4 = (OUT == OUT_U4 || OUT == OUT_S4);
    constexpr int kRowBytes = BMc * (kInt4 ? 4 : 8) / 8;      // staging row = one pixel
    constexpr int kChunksPerWarp = kBNp / 32 / 2;             // two warps per lane quarter

    uint64_t *bars = reinterpret_cast<uint64_t *>(smem + p.off_bar);
    uint64_t *full = bars;
    uint64_t *empty = bars + NS;
    uint64_t *aready = bars + 2 * NS;
    uint64_t *tfull = bars + 3 * NS;
    uint64_t *tempty = bars + 3 * NS + 2;
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(bars + 3 * NS + 4);

    if (warp == kWarpTMA && lane == 0) {
        tma_prefetch_desc(&xmap);
        tma_prefetch_desc(&wmap);
        tma_prefetch_desc(&ymap);
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

    if (warp == kWarpTMA || warp == 2 || warp == 3) {
        // ===================== TMA producers =====================
        if (lane == 0) {
            const int pi = warp == kWarpTMA ? 0 : warp - 1;
            const uint32_t tx = static_cast<uint32_t>(BNp * p.bkp + BMc * p.BK);
            int g = 0;
            for (int tile = blockIdx.x; tile < p.num_tiles; tile += gridDim.x) {
                const int m0 = (tile / p.n_tiles_n) * BNp;          // first output pixel
                const int c0 = (tile % p.n_tiles_n) * BMc;          // first output channel
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
                    trace_ev(p, 0, g);
                    mbar_arrive_expect_tx(&full[stage], tx);
                    // 1x1: K-stage kb = channel chunk kb
                    uint8_t *xdst = IS4 ? smem + p.off_stg + stage * p.stg_stage_bytes
                                        : smem + p.off_a + stage * p.a_stage_bytes;
                    tma_load_im2col_4d(xdst, &xmap, &full[stage], kb * p.bkp, wb, hb, img, 0, 0);
                    tma_load_2d(smem + p.off_b + stage * p.b_stage_bytes, &wmap, &full[stage], kb * p.BK, c0);
                }
            }
        }
    } else if (warp == kWarpMMA) {
        // ===================== MMA issuer: D[c, px] += W[c, :] . X[px, :] =====================
        if (lane == 0) {
            int it = 0, g = 0;
            const uint32_t sbo = 8u * static_cast<uint32_t>(p.BK);
            const int ksteps = p.BK / 32;
            for (int tile = blockIdx.x; tile < p.num_tiles; tile += gridDim.x, ++it) {
                const int buf = it & 1;
                const uint32_t acc_phase = static_cast<uint32_t>(it >> 1) & 1u;
                mbar_wait(&tempty[buf], acc_phase ^ 1u);
                tc_fence_after();
                trace_ev(p, 2, it);
                const uint32_t d_tmem = tmem_base + static_cast<uint32_t>(buf * BNp);
                for (int kb = 0; kb < p.num_kb; ++kb, ++g) {
                    const int stage = g % NS;
                    const uint32_t phase = static_cast<uint32_t>(g / NS) & 1u;
                    mbar_wait(IS4 ? &aready[stage] : &full[stage], phase);
                    tc_fence_after();
                    trace_ev(p, 3, g);
                    const uint32_t w_addr = smem_u32(smem + p.off_b + stage * p.b_stage_bytes);
                    const uint32_t x_addr = smem_u32(smem + p.off_a + stage * p.a_stage_bytes);
                    for (int k = 0; k < ksteps; ++k) {
                        const uint64_t ad = make_smem_desc(w_addr + 32u * k, 16u, sbo, p.sw_layout);
                        const uint64_t bd = make_smem_desc(x_addr + 32u * k, 16u, sbo, p.sw_layout);
                        if (!(p.exp_flags & 4) || (kb | k) == 0)
                            mma_i8(d_tmem, ad, bd, p.idesc, (kb | k) != 0 ? 1u : 0u);
                    }
                    mma_commit(&empty[stage]);
                }
                mma_commit(&tfull[buf]);
                trace_ev(p, 4, it);
            }
        }
    } else if (warp >= kWarpEpi0 && warp < kWarpEpi0 + kNumEpiWarps) {
        // ===================== epilogue: lane = output channel =====================
        const int ew = warp - kWarpEpi0;
        const int quarter = warp & 3;
        const int half = ew >> 2;
        // M=128: channel = 32*quarter + lane.  M=64 (1-CTA): rows live in lanes 0..15 of
        // each 32-lane quarter, channel = 16*quarter + lane.
        const int ch_local = M64 ? 16 * quarter + lane : 32 * quarter + lane;
        const bool lane_ok = !M64 || lane < 16;
        const uint32_t ystg_base = smem_u32(smem + p.off_ystg);
        int cached_c0 = -1;
        TChan cp{};
        int it = 0;
        for (int tile = blockIdx.x; tile < p.num_tiles; tile += gridDim.x, ++it) {
            const int buf = it & 1;
            const uint32_t acc_phase = static_cast<uint32_t>(it >> 1) & 1u;
            const int m0 = (tile / p.n_tiles_n) * kBNp;
            const int c0 = (tile % p.n_tiles_n) * BMc;
            if (c0 != cached_c0) {
                const int k = c0 + ch_local;
                const bool kok = lane_ok && k < p.K;
                const int lg = p.acc_lg;                      // see fill_epilogue_params
                const int64_t beff = kok ? eff_bias(p, k) : 0;
                const int32_t m = kok ? __ldg(p.mult + k) : 0;
                const int32_t n = kok ? __ldg(p.shift + k) : 40 - lg;
                const int ne = n + lg;
                const bool b_ok = lg == 0 ? (beff == static_cast<int64_t>(static_cast<int32_t>(beff)))
                                          : (beff > -(int64_t(1) << 26) && beff < (int64_t(1) << 26));
                const unsigned act = 0xffffffffu;
                const bool all_fast = __ballot_sync(act, b_ok && ne >= 33 && ne <= 52) == act;
                const bool all_mid = __ballot_sync(act, b_ok && ne >= 20 && ne <= 50) == act;
                cp.mode = all_fast ? 0 : (all_mid ? 1 : 2);
                const int T = max(33, __reduce_max_sync(act, ne));
                cp.m = m; cp.b = static_cast<int32_t>(beff); cp.n = n;
                if (cp.mode == 0) {
                    cp.c64 = (beff << lg) * m + (static_cast<int64_t>(1) << (ne - 1)) +
                             (static_cast<int64_t>(p.y_zero) << ne);
                    cp.sh = ne - 32;
                } else if (cp.mode == 1) {
                    cp.b = static_cast<int32_t>(beff << lg);
                    cp.k = T - ne;
                    cp.vlim = 1 << (ne - 20);
                    cp.sh = T - 32;
                    cp.c64 = static_cast<int64_t>((1 << (T - 33)) + p.y_zero * (1 << (T - 32))) << 32;
                }
                cached_c0 = c0;
            }
            mbar_wait(&tfull[buf], acc_phase);
            tc_fence_after();
            if (ew == 0 && lane == 0) trace_ev(p, 5, it);
            const uint32_t taddr = tmem_base + (static_cast<uint32_t>(quarter * 32) << 16) +
                                   static_cast<uint32_t>(buf * kBNp);
            const bool storer = ew == 0 && lane == 0;
            if (storer) bulk_wait_read<1>();
            named_bar_sync(1, kNumEpiWarps * 32);
            // byte of this channel inside a staging row (row = pixel, unswizzled)
            const uint32_t ystg = ystg_base + static_cast<uint32_t>(it & 1) * p.ystg_bytes +
                                  static_cast<uint32_t>(kInt4 ? ch_local >> 1 : ch_local);
            // chunks half, half+2, ...: TMEM loads double-buffered against the requantization
            uint32_t va[32], vb[32];
            tmem_ld_32x32b_x32(taddr + half * 32, va);
#pragma unroll
            for (int t = 0; t < kChunksPerWarp; t += 2) {
                const int ci = half + 2 * t;
                tmem_wait_ld_regs(va);
                if (t + 1 < kChunksPerWarp) tmem_ld_32x32b_x32(taddr + (ci + 2) * 32, vb);
                t_chunk<OUT, kRowBytes>(p, cp, va, ystg + static_cast<uint32_t>(ci * 32 * kRowBytes), lane, lane_ok);
                if (t + 1 < kChunksPerWarp) {
                    tmem_wait_ld_regs(vb);
                    if (t + 2 < kChunksPerWarp) tmem_ld_32x32b_x32(taddr + (ci + 4) * 32, va);
                    t_chunk<OUT, kRowBytes>(p, cp, vb, ystg + static_cast<uint32_t>((ci + 2) * 32 * kRowBytes), lane,
                                            lane_ok);
                }
            }
            tc_fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive(&tempty[buf]);
            if (ew == 0 && lane == 0) trace_ev(p, 6, it);
            fence_proxy_async_smem();
            named_bar_sync(1, kNumEpiWarps * 32);
            if (storer && !(p.exp_flags & 128)) {
                tma_store_2d(&ymap, smem + p.off_ystg + (it & 1) * p.ystg_bytes, c0 * (kInt4 ? 4 : 8) / 8, m0);
                bulk_commit();
            }
        }
        if (ew == 0 && lane == 0) bulk_wait<0>();
    } else if (IS4 && warp >= kWarpCvt0 && warp < kWarpCvt0 + kNumCvtWarps) {
        // ===================== int4 -> int8 widening of the activation tile =====================
        const int ct = (warp - kWarpCvt0) * 32 + lane;
        const int cshift = p.cvt_shift;
        const int nchunks = BNp << cshift;
        const uint32_t xo = p.x_sgn4 ? 0x88888888u : 0u;
        const uint32_t sw = static_cast<uint32_t>(p.sw_mask);
        const uint32_t bkb = static_cast<uint32_t>(p.BK);
        int g = 0;
        for (int tile = blockIdx.x; tile < p.num_tiles; tile += gridDim.x) {
            for (int kb = 0; kb < p.num_kb; ++kb, ++g) {
                const int stage = g % NS;
                const uint32_t phase = static_cast<uint32_t>(g / NS) & 1u;
                mbar_wait(&full[stage], phase);
                if (ct == 0) trace_ev(p, 8, g);
                const uint32_t stg = smem_u32(smem + p.off_stg + stage * p.stg_stage_bytes);
                const uint32_t adst = smem_u32(smem + p.off_a + stage * p.a_stage_bytes);
                if (!(p.exp_flags & 8)) widen_stage(stg, adst, ct, nchunks, cshift, bkb, sw, xo);
                if (ct == 0) trace_ev(p, 10, g);
                fence_proxy_async_smem();
                __syncwarp();
                if (lane == 0) mbar_arrive(&aready[stage]);
                if (ct == 0) trace_ev(p, 9, g);
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

}  // namespace qc
