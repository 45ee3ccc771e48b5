// trans.cuh -- channel-major ("transposed") variant of the implicit-GEMM conv for
// 1x1 convolutions, whose cost is dominated by the fused epilogue.
//
// Same method (Alg.2, epilogue P:L223/P:L253/P:L265), operands swapped:
// the UMMA computes D^T = W * X^T with M = BMc output channels (weights as the A
// operand) and N = BNp output pixels (im2col activations as the B operand).  A TMEM
// lane is then one output channel.  The weight rows are loaded permuted (a 4-D TMA view,
// qconv.cu encode_w_map_pairs) so that TMEM lanes l and l+8 of every 16-lane group hold
// the channel pair (2i, 2i+1); a 16x256b TMEM load then gives each epilogue thread both
// channels of a pair for two adjacent pixels.  The thread keeps the pair's
// re-quantization constants in registers (no per-element shared-memory loads) and per
// output pair does two IMAD.HI (with the 64-bit bias/rounding addend), two shifts and one
// saturating pack into the pair's byte (4-bit) or 16-bit word (8-bit) of an NHWC row,
// staged (swizzled) in shared memory and written by TMA stores.
#pragma once
#include "epilogue.cuh"

namespace qc {

struct TChan {          // per-channel constants held in registers by the epilogue thread
    int64_t c64;        // fast/mid: 64-bit addend of the IMAD.HI (bias*m, rounding, zero point)
    int32_t m, sh, b, k, vlim, n;
};

// Re-quantize one accumulator of one channel; `mode` is warp uniform:
// 0 fast (shift 33..52), 1 mid (shift 20..50, |m| >= 2^30 or m == 0), 2 general (see
// epilogue.cuh EpiCol).  The TFLite rounding is not taken here (qconv.cu plans it elsewhere).
template <int MODE>
__device__ __forceinline__ int32_t t_requant(const ConvParams &p, const TChan &c, uint32_t acc) {
    int32_t y;
    if (MODE == 0) {
        y = static_cast<int32_t>((static_cast<int64_t>(static_cast<int32_t>(acc)) * c.m + c.c64) >> 32) >> c.sh;
    } else if (MODE == 1) {
        int32_t x = static_cast<int32_t>(acc) + c.b;
        x = min(c.vlim, max(-c.vlim, x)) << c.k;
        y = static_cast<int32_t>((static_cast<int64_t>(x) * c.m + c.c64) >> 32) >> c.sh;
    } else {
        const int64_t lo64 = static_cast<int64_t>(p.clamp_lo) - p.y_zero;
        const int64_t hi64 = static_cast<int64_t>(p.clamp_hi) - p.y_zero;
        const int32_t x = static_cast<int32_t>(static_cast<uint32_t>(static_cast<int32_t>(acc) >> p.acc_lg) +
                                               static_cast<uint32_t>(c.b));
        const int64_t prod = static_cast<int64_t>(x) * c.m + (static_cast<int64_t>(1) << (c.n - 1));
        int64_t t = prod >> c.n;
        t = t < lo64 ? lo64 : (t > hi64 ? hi64 : t);
        y = static_cast<int32_t>(t) + p.y_zero;
    }
    return y;
}

// 64 pixels (columns) of one channel pair: v from tmem_ld_16x256b_x8, repetition k holds
// pixels px0 = 8k + 2(lane%4) and px0 + 1 for the even (v[4k], v[4k+1]) and odd
// (v[4k+2], v[4k+3]) channel.  Stores the pair's byte (4-bit) / 16-bit word (8-bit) of each
// pixel into the swizzled staging rows.  The swizzle term of row px0 + 8k does not depend on
// k (rows step by 8, the XOR uses row bits below 8 rows), so the two store addresses are
// computed once and the repetitions use immediate offsets.
template <int OUT, int MODE, bool CLAMP, int RB, int GMASK, bool ALU_PACK = false>
__device__ __forceinline__ void t_pairs(const ConvParams &p, const TChan &ce, const TChan &co,
                                        const uint32_t (&v)[32], uint32_t ystg, int row0, uint32_t boff) {
    constexpr bool kInt4 = (OUT == OUT_U4 || OUT == OUT_S4);
    const uint32_t off0 = static_cast<uint32_t>(row0) * RB + boff, off1 = off0 + RB;
    const uint32_t a0 = ystg + (off0 ^ (((off0 >> 7) & GMASK) << 4));
    const uint32_t a1 = ystg + (off1 ^ (((off1 >> 7) & GMASK) << 4));
    const int32_t lo = p.clamp_lo, hi = p.clamp_hi;
#pragma unroll
    for (int k = 0; k < 8; ++k) {
        int32_t ye0 = t_requant<MODE>(p, ce, v[4 * k]), ye1 = t_requant<MODE>(p, ce, v[4 * k + 1]);
        int32_t yo0 = t_requant<MODE>(p, co, v[4 * k + 2]), yo1 = t_requant<MODE>(p, co, v[4 * k + 3]);
        if (CLAMP) {
            ye0 = min(hi, max(lo, ye0)); ye1 = min(hi, max(lo, ye1));
            yo0 = min(hi, max(lo, yo0)); yo1 = min(hi, max(lo, yo1));
        }
        const uint32_t d = static_cast<uint32_t>(8 * k * RB);
        if (ALU_PACK) {
            // saturate with min/max and pack with one LEA (ALU pipe) instead of I2IP
            constexpr int32_t qlo = OUT == OUT_U4 ? 0 : (OUT == OUT_S4 ? -8 : (OUT == OUT_U8 ? 0 : -128));
            constexpr int32_t qhi = OUT == OUT_U4 ? 15 : (OUT == OUT_S4 ? 7 : (OUT == OUT_U8 ? 255 : 127));
            constexpr uint32_t msk = kInt4 ? 0xFu : 0xFFu;
            constexpr int sh = kInt4 ? 4 : 8;
            if (!CLAMP) {
                ye0 = min(qhi, max(qlo, ye0)); ye1 = min(qhi, max(qlo, ye1));
                yo0 = min(qhi, max(qlo, yo0)); yo1 = min(qhi, max(qlo, yo1));
            }
            const uint32_t w0 = (static_cast<uint32_t>(yo0) << sh) | (static_cast<uint32_t>(ye0) & msk);
            const uint32_t w1 = (static_cast<uint32_t>(yo1) << sh) | (static_cast<uint32_t>(ye1) & msk);
            if (kInt4) { sts8(a0 + d, w0); sts8(a1 + d, w1); }
            else { sts16(a0 + d, w0); sts16(a1 + d, w1); }
        } else if (kInt4) {
            sts8(a0 + d, OUT == OUT_U4 ? pack_sat_u4(yo0, ye0, 0u) : pack_sat_s4(yo0, ye0, 0u));
            sts8(a1 + d, OUT == OUT_U4 ? pack_sat_u4(yo1, ye1, 0u) : pack_sat_s4(yo1, ye1, 0u));
        } else {
            sts16(a0 + d, OUT == OUT_U8 ? pack_sat_u8(yo0, ye0, 0u) : pack_sat_s8(yo0, ye0, 0u));
            sts16(a1 + d, OUT == OUT_U8 ? pack_sat_u8(yo1, ye1, 0u) : pack_sat_s8(yo1, ye1, 0u));
        }
    }
}

template <int OUT, int RB, int GMASK>
__device__ __forceinline__ void t_pairs_mode(const ConvParams &p, int mode, const TChan &ce, const TChan &co,
                                             const uint32_t (&v)[32], uint32_t ystg, int row0, uint32_t boff) {
    if (p.need_clamp) {
        if (mode == 0) t_pairs<OUT, 0, true, RB, GMASK>(p, ce, co, v, ystg, row0, boff);
        else if (mode == 1) t_pairs<OUT, 1, true, RB, GMASK>(p, ce, co, v, ystg, row0, boff);
        else t_pairs<OUT, 2, true, RB, GMASK>(p, ce, co, v, ystg, row0, boff);
    } else {
        if (mode == 0) t_pairs<OUT, 0, false, RB, GMASK>(p, ce, co, v, ystg, row0, boff);
        else if (mode == 1) t_pairs<OUT, 1, false, RB, GMASK>(p, ce, co, v, ystg, row0, boff);
        else t_pairs<OUT, 2, false, RB, GMASK>(p, ce, co, v, ystg, row0, boff);
    }
}

// Per-channel constants of tile-relative channel k (fill_epilogue_params' rules).
__device__ __forceinline__ void t_chan_params(const ConvParams &p, int k, bool kok, TChan &c, int &ne, bool &b_ok) {
    const int lg = p.acc_lg;
    const int64_t beff = kok ? eff_bias(p, k) : 0;
    c.m = kok ? __ldg(p.mult + k) : 0;
    c.n = kok ? __ldg(p.shift + k) : 40 - lg;
    ne = c.n + lg;
    b_ok = lg == 0 ? (beff == static_cast<int64_t>(static_cast<int32_t>(beff)))
                   : (beff > -(int64_t(1) << 26) && beff < (int64_t(1) << 26));
    c.b = static_cast<int32_t>(beff);
    c.c64 = (beff << lg) * c.m + (static_cast<int64_t>(1) << (ne - 1)) + (static_cast<int64_t>(p.y_zero) << ne);
    c.sh = ne - 32;
}
__device__ __forceinline__ void t_chan_mid(const ConvParams &p, TChan &c, int ne, int T) {
    c.b = static_cast<int32_t>(static_cast<int64_t>(c.b) << p.acc_lg);
    c.k = T - ne;
    c.vlim = 1 << (ne - 20);
    c.sh = T - 32;
    c.c64 = static_cast<int64_t>((1 << (T - 33)) + p.y_zero * (1 << (T - 32))) << 32;
}


template <bool IS4, int OUT, bool M64>
__global__ void __launch_bounds__(IS4 ? kTThreads4 : kTThreads8, 1)
qconv_t_kernel(const __grid_constant__ CUtensorMap xmap, const __grid_constant__ CUtensorMap wmap,
               const __grid_constant__ CUtensorMap ymap, const __grid_constant__ ConvParams p) {
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    // 1024-byte aligned base by pointer arithmetic on the shared array itself (no integer round
    // trip): the compiler keeps it in the shared window, so every smem_u32() below is one add
    uint8_t *smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;
    const int NS = p.stages;
    constexpr int BMc = M64 ? 64 : 128;   // output channels per tile (UMMA M)
    constexpr int kBNp = kTBNp;           // output pixels per tile (UMMA N)
    constexpr int BNp = kBNp;
    constexpr int kNB = kTGroups;         // accumulator buffers = staging buffers = epilogue groups
    constexpr int kLgNB = kNB == 4 ? 2 : 1;
    constexpr bool kInt4 = (OUT == OUT_U4 || OUT == OUT_S4);
    constexpr int kRowBytes = BMc * (kInt4 ? 4 : 8) / 8;      // staging row = one pixel

    uint64_t *bars = reinterpret_cast<uint64_t *>(smem + p.off_bar);
    uint64_t *full = bars;
    uint64_t *empty = bars + NS;
    uint64_t *aready = bars + 2 * NS;
    uint64_t *tfull = bars + 3 * NS;        // [kNB] MMA -> epilogue group: accumulator written
    uint64_t *tempty = bars + 3 * NS + 4;   // [kNB] epilogue group -> MMA: accumulator read
    uint64_t *sfull = bars + 3 * NS + 8;    // [kNB] epilogue group -> storer: staging buffer written
    uint64_t *sfree = bars + 3 * NS + 12;   // [kNB] storer -> epilogue group: its TMA store has read it
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(bars + 3 * NS + 16);

    griddep_launch_dependents();
    if (warp == kWarpTMA && lane == 0) {
        tma_prefetch_desc(&xmap);
        tma_prefetch_desc(&wmap);
        tma_prefetch_desc(&ymap);
        for (int i = 0; i < NS; ++i) {
            mbar_init(&full[i], 1);
            mbar_init(&empty[i], 1);
            mbar_init(&aready[i], kNumCvtWarps);
        }
        for (int i = 0; i < kNB; ++i) {
            mbar_init(&tfull[i], 1);
            mbar_init(&tempty[i], kTEpiWarps / kTGroups);
            mbar_init(&sfull[i], kTEpiWarps / kTGroups);
            mbar_init(&sfree[i], 1);
        }
        fence_mbar_init();
    }
    if (warp == kWarpMMA) tmem_alloc(tmem_slot, p.tmem_cols);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;

    if (warp == kWarpTMA || warp == 2 || warp == 3) {
        // ===================== output storer (warp 2, lane 0) =====================
        // The epilogue warps never wait for each other: each arrives on sfull[b] once its part
        // of staging buffer b is written; this thread waits for all 16, issues the TMA store, and
        // releases the other buffer (sfree) once the store issued before has read it.
        if (warp == 2 && lane == 0) {
            int it = 0;
            for (int tile = blockIdx.x; tile < p.num_tiles; tile += gridDim.x, ++it) {
                const int b = it & (kNB - 1);
                const int m0 = (tile / p.n_tiles_n) * BNp;
                const int c0 = (tile % p.n_tiles_n) * BMc;
                mbar_wait(&sfull[b], static_cast<uint32_t>(it >> kLgNB) & 1u);
                tma_store_2d(&ymap, smem + p.off_ystg + b * p.ystg_bytes, c0 * (kInt4 ? 4 : 8) / 8, m0);
                bulk_commit();
                // buffer b belongs to one epilogue group: release it as soon as its own store
                // has read it (the other groups keep working meanwhile)
                bulk_wait_read<0>();
                mbar_arrive(&sfree[b]);
                trace_ev(p, 7, it);
            }
            bulk_wait<0>();
        }
        // ===================== TMA producers =====================
        if (lane == 0 && warp != 2) {   // lane 0 of warps 0 and 3 issue (warp 2 stores)
            griddep_wait();                                         // activations of the previous layer
            const int pi = warp == kWarpTMA ? 0 : 1;
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
                    if (g % kTProducers != pi) continue;
                    const int stage = g % NS;
                    const uint32_t phase = static_cast<uint32_t>(g / NS) & 1u;
                    mbar_wait(&empty[stage], phase ^ 1u);
                    trace_ev(p, 0, g);
                    mbar_arrive_expect_tx(&full[stage], tx);
                    // 1x1: K-stage kb = channel chunk kb
                    uint8_t *xdst = IS4 ? smem + p.off_stg + stage * p.stg_stage_bytes
                                        : smem + p.off_a + stage * p.a_stage_bytes;
                    tma_load_im2col_4d(xdst, &xmap, &full[stage], kb * p.bkp, wb, hb, img, 0, 0);
                    tma_load_4d(smem + p.off_b + stage * p.b_stage_bytes, &wmap, &full[stage], kb * p.BK, 0, 0,
                                c0 / 16);
                }
            }
        }
    } else if (warp == kWarpMMA) {
        // ===================== MMA issuer: D[c, px] += W[c, :] . X[px, :] =====================
        // whole warp runs the loop, one elected lane issues (see conv_fwd.cuh)
        {
            int it = 0, g = 0;
            RingPos rp;
            const uint32_t sbo = 8u * static_cast<uint32_t>(p.BK);
            const int ksteps = p.BK / 32;
            // Per tile the accumulator hand-back (tempty) is the critical path: the first K-stage's
            // operands are waited for and its descriptors formed BEFORE waiting on tempty, so only
            // the fence and the branch-free issue (ksteps <= 4, predicated) follow it.
            for (int tile = blockIdx.x; tile < p.num_tiles; tile += gridDim.x, ++it) {
                const int buf = it & (kNB - 1);
                const uint32_t acc_phase = static_cast<uint32_t>(it >> kLgNB) & 1u;
                const uint32_t d_tmem = tmem_base + static_cast<uint32_t>(buf * BNp);
                for (int kb = 0; kb < p.num_kb; ++kb, ++g, rp.next(NS)) {
                    const int stage = rp.stage;
                    mbar_wait(IS4 ? &aready[stage] : &full[stage], rp.phase);
                    const uint32_t w_addr = smem_u32(smem + p.off_b + stage * p.b_stage_bytes);
                    const uint32_t x_addr = smem_u32(smem + p.off_a + stage * p.a_stage_bytes);
                    const uint64_t ad0 = make_smem_desc(w_addr, 16u, sbo, p.sw_layout);
                    const uint64_t bd0 = make_smem_desc(x_addr, 16u, sbo, p.sw_layout);
                    const uint32_t alo = static_cast<uint32_t>(ad0), ahi = static_cast<uint32_t>(ad0 >> 32);
                    const uint32_t blo = static_cast<uint32_t>(bd0), bhi = static_cast<uint32_t>(bd0 >> 32);
                    if (kb == 0) {
                        mbar_wait(&tempty[buf], acc_phase ^ 1u);
                        if (lane == 0) trace_ev(p, 2, it);
                    }
                    __syncwarp();
                    tc_fence_after();
                    if (lane == 0) trace_ev(p, 3, g);
#pragma unroll
                    for (int k = 0; k < 4; ++k)
                        mma_i8_warp_lo_if(d_tmem, alo + 2u * k, ahi, blo + 2u * k, bhi, p.idesc,
                                          (kb | k) != 0 ? 1u : 0u, k < ksteps ? 1u : 0u);
                    mma_commit_warp(&empty[stage]);
                }
                mma_commit_warp(&tfull[buf]);
                if (lane == 0) trace_ev(p, 4, it);
            }
        }
    } else if (warp >= kWarpEpi0 && warp < kWarpEpi0 + kTEpiWarps) {
        // ===================== epilogue: lane = output channel, thread = channel pair ===========
        griddep_wait();                                   // params written in-stream
        const int ew = warp - kWarpEpi0;
        const int quarter = warp & 3;
        const int sub = ew >> 2;                           // 0..3: the 4 warps of a lane quarter
        // kTGroups epilogue groups take the tiles round robin (group g: tiles it = g mod kTGroups,
        // accumulator and staging buffer g), so one group's waits overlap the other groups'
        // arithmetic instead of all 16 warps stopping together between tiles.  M=128: quarter q
        // holds 16-lane groups 2q, 2q+1; M=64: rows live in lanes 0..15 of each quarter.
        //  2 groups: a warp covers one 16-lane group, 256 pixels (M=64: 128 pixels)
        //  4 groups: a warp covers its whole quarter (both 16-lane groups at M=128), 128 pixels
        const int gsel = kTGroups == 4 ? sub : (sub >> 1);
        const int wq = kTGroups == 4 ? 0 : (sub & 1);
        constexpr int kNH = (!M64 && kTGroups == 4) ? 2 : 1;     // 16-lane groups per warp
        constexpr int kCols = (M64 && kTGroups == 2) ? kBNp / 2 : kBNp;
        const int col_begin = (M64 && kTGroups == 2) ? wq * kCols : 0;
        constexpr int kGMask = kRowBytes >= 128 ? 7 : (kRowBytes == 64 ? 3 : 1);
        int pair[kNH];
        uint32_t lane_base[kNH];
#pragma unroll
        for (int hh = 0; hh < kNH; ++hh) {
            const int grp = M64 ? quarter : 2 * quarter + (kTGroups == 4 ? hh : (wq & 1));
            pair[hh] = 8 * grp + (lane >> 2);               // channel pair of the tile
            lane_base[hh] = M64 ? 32u * static_cast<uint32_t>(quarter) : 16u * static_cast<uint32_t>(grp);
        }
        const uint32_t ystg_base = smem_u32(smem + p.off_ystg);
        int cached_c0 = -1;
        TChan ce[kNH], co[kNH];
        int mode[kNH];
#pragma unroll
        for (int hh = 0; hh < kNH; ++hh) { ce[hh] = TChan{}; co[hh] = TChan{}; mode[hh] = 2; }
        int it = gsel;
        // channel tile of the CTA's current tile, advanced without divisions
        const int ntn = p.n_tiles_n;
        const int cstep = static_cast<int>((static_cast<int64_t>(gridDim.x) * kTGroups) % ntn);
        int cm = static_cast<int>((blockIdx.x + static_cast<int64_t>(gsel) * gridDim.x) % ntn);
        for (int tile = blockIdx.x + gsel * gridDim.x; tile < p.num_tiles; tile += kTGroups * gridDim.x, it += kTGroups) {
            const int buf = it & (kNB - 1);
            const uint32_t acc_phase = static_cast<uint32_t>(it >> kLgNB) & 1u;
            const int c0 = cm * BMc;
            cm += cstep;
            if (cm >= ntn) cm -= ntn;
            if (c0 != cached_c0) {
#pragma unroll
                for (int hh = 0; hh < kNH; ++hh) {
                    const int ke = c0 + 2 * pair[hh], ko = ke + 1;
                    int nee, neo;
                    bool be, bo;
                    t_chan_params(p, ke, ke < p.K, ce[hh], nee, be);
                    t_chan_params(p, ko, ko < p.K, co[hh], neo, bo);
                    const unsigned act = 0xffffffffu;
                    const bool all_fast = __ballot_sync(act, be && bo && nee >= 33 && nee <= 52 && neo >= 33 && neo <= 52) == act;
                    const bool all_mid = __ballot_sync(act, be && bo && nee >= 20 && nee <= 50 && neo >= 20 && neo <= 50 &&
                                                                mid_multiplier_ok(ce[hh].m) && mid_multiplier_ok(co[hh].m)) == act;
                    mode[hh] = all_fast ? 0 : (all_mid ? 1 : 2);
                    if (mode[hh] == 1) {
                        const int T = max(33, __reduce_max_sync(act, max(nee, neo)));
                        t_chan_mid(p, ce[hh], nee, T);
                        t_chan_mid(p, co[hh], neo, T);
                    }
                }
                cached_c0 = c0;
            }
            mbar_wait(&tfull[buf], acc_phase);
            tc_fence_after();
            if (ew == 0 && lane == 0) trace_ev(p, 5, it);
            // staging buffer `buf` is free once the store of tile it - kNB has read it
            mbar_wait(&sfree[buf], acc_phase ^ 1u);
            const uint32_t ystg = ystg_base + static_cast<uint32_t>(buf) * p.ystg_bytes;
            const int row0 = col_begin + 2 * (lane & 3);
#pragma unroll
            for (int hh = 0; hh < kNH; ++hh) {
                const uint32_t taddr = tmem_base + (lane_base[hh] << 16) + static_cast<uint32_t>(buf * kBNp + col_begin);
                const uint32_t boff = static_cast<uint32_t>(kInt4 ? pair[hh] : 2 * pair[hh]);
                // 64-pixel chunks
#pragma unroll 1
                for (int t = 0; t < kCols / 64; ++t) {
                    uint32_t va[32];
                    tmem_ld_16x256b_x8(taddr + static_cast<uint32_t>(t * 64), va);
                    tmem_wait_ld_regs(va);
                    t_pairs_mode<OUT, kRowBytes, kGMask>(p, mode[hh], ce[hh], co[hh], va, ystg, row0 + 64 * t, boff);
                }
            }
            tc_fence_before();
            fence_proxy_async_smem();                 // staging writes -> visible to the TMA store
            __syncwarp();
            if (lane == 0) {
                mbar_arrive(&tempty[buf]);
                mbar_arrive(&sfull[buf]);
            }
            if (ew == 0 && lane == 0) trace_ev(p, 6, it);
        }
    } else if (IS4 && warp >= kTWarpCvt0 && warp < kTWarpCvt0 + kNumCvtWarps) {
        // ===================== int4 -> int8 widening of the activation tile =====================
        const int ct = (warp - kTWarpCvt0) * 32 + lane;
        const int cshift = p.cvt_shift;
        const int nchunks = BNp << cshift;
        const uint32_t xo = p.x_sgn4 ? 0x88888888u : 0u;
        const uint32_t sw = static_cast<uint32_t>(p.sw_mask);
        const uint32_t bkb = static_cast<uint32_t>(p.BK);
        int g = 0;
        RingPos rp;
        for (int tile = blockIdx.x; tile < p.num_tiles; tile += gridDim.x) {
            for (int kb = 0; kb < p.num_kb; ++kb, ++g, rp.next(NS)) {
                const int stage = rp.stage;
                mbar_wait(&full[stage], rp.phase);
                if (ct == 0) trace_ev(p, 8, g);
                const uint32_t stg = smem_u32(smem + p.off_stg + stage * p.stg_stage_bytes);
                const uint32_t adst = smem_u32(smem + p.off_a + stage * p.a_stage_bytes);
                widen_stage(stg, adst, ct, nchunks, cshift, bkb, sw, xo, static_cast<uint32_t>(p.stg_sw));
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
