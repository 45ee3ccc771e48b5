// halo.cuh -- "halo" variant of the implicit-GEMM conv for stride-1 convolutions.
//
// Same method as conv_fwd.cuh (Alg.2 P:L216-223 with the fused epilogue of
// P:L223/P:L253/P:L265), different data movement, chosen for B200's TMA:
//  * A tile = Rt whole output rows, each padded to Wh = W + 2*pad_w columns
//    (columns >= Q are computed and discarded).  Instead of one im2col TMA per
//    filter tap (R*S loads of 128 pixels, every input pixel fetched R*S times),
//    ONE tiled TMA brings the (Rt+R-1) x Wh input halo of the tile, all channels,
//    as 16-byte channel planes [plane][row][col][16 B] (zero-filled outside the
//    image = the padding).  Every tap (r, s) is then the same buffer read at a
//    pixel offset r*Wh + s: the UMMA no-swizzle K-major descriptor takes
//    start = plane + (r*Wh+s)*16, SBO = 128 (8 pixels), LBO = plane stride.
//  * B (weights of the CTA's N tile) is resident in shared memory for the whole
//    kernel, loaded by one TMA as [K-chunk plane][BN rows][16 B].
//  * The C=16 space-to-depth stem pairs taps (r,s),(r,s+1) in one K=32 MMA
//    (LBO = 16: the next tap is the next pixel).
// The paper's precomputed-offset gather and register prefetch
// have no counterpart: the hardware gathers, shared memory reuses.
#pragma once
#include "epilogue.cuh"
#include "quant.cuh"
#include "trans.cuh"

namespace qc {


// Fused fp32 quantization of the space-to-depth stem (F32): the producer TMA-loads the tile's
// 2*HR fp32 input rows (a 4-D [n][h][w*c/4][4] view: rows outside the image are zero-filled, and
// quantize to the zero point, the space-to-depth padding code), and the converter warps quantize
// them (reading Z4: one fp32 multiply by fl32(1/scale), round to nearest even, + z, clamp; NaN ->
// z) straight into the byte-coded halo X2[i][j][(2b+b')*c + cc] = q(x[2i+b-pad_h, 2j+b'-pad_w, cc])
// -- no X2 tensor in global memory and no separate quantize launch.
// NaN-propagating float min / max (fminf / fmaxf return the other operand for a NaN).
__device__ __forceinline__ float fmax_nan(float a, float b) {
    float r;
    asm("max.NaN.f32 %0, %1, %2;" : "=f"(r) : "f"(a), "f"(b));
    return r;
}
__device__ __forceinline__ float fmin_nan(float a, float b) {
    float r;
    asm("min.NaN.f32 %0, %1, %2;" : "=f"(r) : "f"(a), "f"(b));
    return r;
}

// quantize_one (quant.cuh, reading Z4) without branches: the clamp to the integer bounds
// [qmin - z, qmax - z] in the float domain commutes with round-to-nearest-even, so no integer
// clamp follows, and a NaN passes the NaN-propagating clamp and converts to 0, i.e. code z.
__device__ __forceinline__ int32_t f32_q(const ConvParams &p, float x) {
    const float t = fmin_nan(fmax_nan(__fmul_rn(x, p.q_inv_s), p.q_flo), p.q_fhi);
    return __float2int_rn(t) + p.q_z;
}

// One space-to-depth pixel X2[i][j] (16 code bytes, channel (2b+b')*C + cc; the 4C..15 tail
// holds the zero point) from the two staged fp32 input rows 2i - pad_h, +1.  addr[blk] is the
// address of input pixel (2i + (blk >> 1) - pad_h, 2j + (blk & 1) - pad_w), or of a zeroed
// 16-byte area when that pixel is outside the image (+0.0 quantizes to the zero point).
template <int C>
__device__ __forceinline__ void f32_s2d_pixel(const ConvParams &p, const uint32_t (&addr)[4], uint32_t (&w)[4]) {
    int32_t code[16];
#pragma unroll
    for (int blk = 0; blk < 4; ++blk) {
#pragma unroll
        for (int cc = 0; cc < C; ++cc) {
            float v;
            if (p.bf16) {     // bf16 input: the exact fp32 value is the bf16 bits << 16
                uint32_t u;
                asm volatile("ld.shared.u16 %0, [%1];" : "=r"(u) : "r"(addr[blk] + 2u * cc));
                v = __uint_as_float(u << 16);
            } else {
                asm volatile("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"(addr[blk] + 4u * cc));
            }
            code[blk * C + cc] = f32_q(p, v);
        }
    }
#pragma unroll
    for (int k = 4 * C; k < 16; ++k) code[k] = p.q_z;
    // codes are in [qmin, qmax] already: the saturating packs only place the bytes
    if (p.q_qmin < 0) {
#pragma unroll
        for (int k = 0; k < 4; ++k)
            w[k] = pack_sat_s8(code[4 * k + 1], code[4 * k], pack_sat_s8(code[4 * k + 3], code[4 * k + 2], 0u));
    } else {
#pragma unroll
        for (int k = 0; k < 4; ++k)
            w[k] = pack_sat_u8(code[4 * k + 1], code[4 * k], pack_sat_u8(code[4 * k + 3], code[4 * k + 2], 0u));
    }
}

// Per-thread source layout of X2 column j: byte offsets within a staged row pair of its four
// input pixels and a mask of those inside the image.
__device__ __forceinline__ uint32_t f32_s2d_offsets(const ConvParams &p, int j, uint32_t (&off)[4]) {
    uint32_t ok = 0;
#pragma unroll
    for (int blk = 0; blk < 4; ++blk) {
        const int ww = 2 * j + (blk & 1) - p.f_pad_w;
        const bool in = ww >= 0 && ww < p.f_w;
        off[blk] = (blk >> 1) * static_cast<uint32_t>(p.f_rowbytes) +
                   (p.bf16 ? 2u : 4u) * static_cast<uint32_t>((in ? ww : 0) * p.f_c);
        ok |= in ? (1u << blk) : 0u;
    }
    return ok;
}
__device__ __forceinline__ void f32_s2d_addr(uint32_t rows, const uint32_t (&off)[4], uint32_t ok, uint32_t zero,
                                             uint32_t (&addr)[4]) {
#pragma unroll
    for (int blk = 0; blk < 4; ++blk) addr[blk] = (ok >> blk) & 1u ? rows + off[blk] : zero;
}

// CM = channel-major variant (K = 64): the UMMA computes D^T = W * X^T with M = 64 output
// channels (the resident weights, rows permuted so TMEM lanes l and l+8 hold a channel pair)
// and N = Rt * Wh pixels (the halo, rows padded to Wh = a multiple of 8, N <= 256); the
// epilogue is the channel-pair epilogue of trans.cuh (constants in registers, ~3 instructions
// per output) with 16 warps, and the storer writes one output row per TMA store.
template <bool IS4, int OUT, bool F32 = false, bool CM = false>
__global__ void __launch_bounds__(CM ? ((IS4 || F32) ? kTThreads4 : kTThreads8)
                                     : ((IS4 || F32) ? 512 : 384), 1)
qconv_halo_kernel(const __grid_constant__ CUtensorMap hmap, const __grid_constant__ CUtensorMap bmap,
                  const __grid_constant__ CUtensorMap ymap, const __grid_constant__ ConvParams p) {
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    // 1024-byte aligned base by pointer arithmetic on the shared array itself (no integer round
    // trip): the compiler keeps it in the shared window, so every smem_u32() below is one add
    uint8_t *smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;
    const int NS = p.stages;

    uint64_t *bars = reinterpret_cast<uint64_t *>(smem + p.off_bar);
    uint64_t *hfull = bars;                 // [NS] halo TMA -> (converter | MMA)
    uint64_t *hempty = bars + NS;           // [NS] MMA -> producer
    uint64_t *hready = bars + 2 * NS;       // [NS] converter -> MMA (4-bit)
    uint64_t *tfull = bars + 3 * NS;        // [2]
    uint64_t *tempty = bars + 3 * NS + 2;   // [2]
    uint64_t *bfull = bars + 3 * NS + 4;    // [1] resident weights landed
    uint64_t *sfull = bars + 3 * NS + 5;    // [kMaxYstg] epilogue warps -> storer: staging buffer written
    uint64_t *sfree = bars + 3 * NS + 5 + kMaxYstg;   // [kMaxYstg] storer -> epilogue warps: store read it
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(bars + 3 * NS + 5 + 2 * kMaxYstg);
    const int NB = p.n_ystg;                 // staging buffers
    EpiCol *par = reinterpret_cast<EpiCol *>(smem + p.off_par);
    int4 *chunk_info = reinterpret_cast<int4 *>(smem + p.off_par + 16 * kMaxBN);

    // Warp roles: epilogue 0-7 (TMEM lane quarter = warp % 4), converters 8-11 (4-bit), then
    // the single-thread roles with the highest ids -- the SM's warp arbiter favours higher warp
    // ids (B300_MICROARCH "hi-wid-first"), and the MMA warp's issue loop (8-18 MMAs per tile)
    // is on the kernel's critical path, so it must not wait behind epilogue instructions.
    constexpr int kEpi0 = 0;
    constexpr int kNEpi = CM ? kTEpiWarps : kNumEpiWarps;
    constexpr int kCvt0 = kNEpi;
    constexpr bool kCvt = IS4 || F32;                // converter warps present
    constexpr int kCtl0 = kNEpi + (kCvt ? kNumCvtWarps : 0);
    constexpr int kProd = kCtl0, kStorer = kCtl0 + 1, kMma = kCtl0 + 3;
    griddep_launch_dependents();
    if (warp == kProd && lane == 0) {
        tma_prefetch_desc(&hmap);
        tma_prefetch_desc(&bmap);
        tma_prefetch_desc(&ymap);
        for (int i = 0; i < NS; ++i) {
            mbar_init(&hfull[i], 1);
            mbar_init(&hempty[i], 1);
            mbar_init(&hready[i], kNumCvtWarps);
        }
        for (int i = 0; i < 2; ++i) {
            mbar_init(&tfull[i], 1);
            mbar_init(&tempty[i], CM ? kNEpi / 2 : kNEpi);
        }
        for (int i = 0; i < kMaxYstg; ++i) {
            mbar_init(&sfull[i], CM ? kNEpi / 2 : kNEpi);
            mbar_init(&sfree[i], 1);
        }
        mbar_init(bfull, 1);
        fence_mbar_init();
    }
    if (warp == kMma) tmem_alloc(tmem_slot, p.tmem_cols);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;
    // Tiles of this CTA: round robin over the grid, or -- for the fused fp32 stem -- one
    // contiguous run of output rows, so a tile's space-to-depth halo shares HR-1 of its HR rows
    // with the previous tile's (converted once, copied forward) and only two new fp32 rows are
    // loaded per tile.  (F32 always has one N tile: K <= 256.)
    int t_first = static_cast<int>(blockIdx.x), t_step = static_cast<int>(gridDim.x), t_end = p.num_tiles;
    if (F32) {
        t_first = static_cast<int>(static_cast<int64_t>(blockIdx.x) * p.num_tiles / gridDim.x);
        t_end = static_cast<int>(static_cast<int64_t>(blockIdx.x + 1) * p.num_tiles / gridDim.x);
        t_step = 1;
    }
    // all tiles of this CTA share one N tile (grid is a multiple of n_tiles_n)
    const int n0 = (static_cast<int>(blockIdx.x) % p.n_tiles_n) * p.BN;

    if (warp == kStorer) {
        // ===================== output storer (see trans.cuh) =====================
        if (lane == 0) {
            int it = 0;
            int b = 0, bprev = 0;                   // staging buffer of this / the previous tile
            uint32_t bphase = 0;
            for (int tile = t_first; tile < t_end; tile += t_step, ++it) {
                const int mt = p.fd_ntn.div(tile);
                const int img = p.fd_tpi.div(mt);
                const int p0 = (mt - img * p.tiles_per_img) * p.Rt;
                mbar_wait(&sfull[b], bphase);
                if (CM) {   // one store per output row: staging row = accumulator column
                    for (int rr = 0; rr < p.Rt; ++rr)
                        tma_store_4d(&ymap, smem + p.off_ystg + b * p.ystg_bytes + rr * p.Wh * p.y_gw, 0, 0,
                                     p0 + rr, img);
                } else {
                    constexpr int kBits = (OUT == OUT_U4 || OUT == OUT_S4) ? 4 : 8;
                    for (int gi = 0; gi < p.n_ygroups; ++gi)
                        tma_store_4d(&ymap, smem + p.off_ystg + b * p.ystg_bytes + gi * 128 * p.y_gw,
                                     n0 * kBits / 8 + gi * p.y_gw, 0, p0, img);
                }
                bulk_commit();
                if (CM && NB == 2) {
                    // staging buffer b belongs to one epilogue group: release it once its own
                    // store has read it (the other group keeps working meanwhile)
                    bulk_wait_read<0>();
                    mbar_arrive(&sfree[b]);
                } else {
                    // keep two stores in flight: the previous one has read its buffer -> release it
                    bulk_wait_read<1>();
                    if (it > 0) mbar_arrive(&sfree[bprev]);
                }
                bprev = b;
                if (++b == NB) { b = 0; bphase ^= 1u; }
                trace_ev(p, 7, it);
            }
            bulk_wait<0>();
        }
    } else if (warp == kProd) {
        // ===================== TMA producer =====================
        if (lane == 0) {   // one thread issues (measured faster than an elected warp-wide loop)
            constexpr bool leader = true;
            // the weights may have been written by the kernel just before this one in the
            // stream (weight preparation, or the caller's own kernels): wait for it first
            griddep_wait();
            if (leader) mbar_arrive_expect_tx(bfull, p.b_res_bytes);
            if (CM) {   // permuted 5-D view (channel pairs on TMEM lanes l, l+8); K = 64: n0 = 0
                if (leader) tma_load_5d(smem + p.off_bres, &bmap, bfull, 0, 0, 0, 0, 0);
            } else {
                if (leader) tma_load_3d(smem + p.off_bres, &bmap, bfull, 0, n0, 0);
            }
            int g = 0;
            RingPos rp;
            for (int tile = t_first; tile < t_end; tile += t_step, ++g, rp.next(NS)) {
                const int mt = p.fd_ntn.div(tile);
                const int img = p.fd_tpi.div(mt);
                const int p0 = (mt - img * p.tiles_per_img) * p.Rt;
                const int stage = rp.stage;
                mbar_wait(&hempty[stage], rp.phase ^ 1u);
                if (leader) trace_ev(p, 0, g);
                uint8_t *dst = kCvt ? smem + p.off_hp + stage * p.hp_stage_bytes
                                    : smem + p.off_hx + stage * p.hx_stage_bytes;
                if (F32) {
                    // fp32 input row pairs (2*(p0+hr) - pad_h, +1) of the original image; a
                    // continuation tile only needs the pair of its last halo row
                    const bool cont = tile != t_first && p0 != 0 && p.Rt < p.HR;
                    const int hr0 = cont ? p.HR - p.Rt : 0;
                    if (leader) mbar_arrive_expect_tx(&hfull[stage], static_cast<uint32_t>(2 * (p.HR - hr0) * p.f_rowbytes));
                    for (int hr = hr0; hr < p.HR; ++hr)
                        tma_load_4d(dst + 2 * (hr - hr0) * p.f_rowbytes, &hmap, &hfull[stage], 0, 0,
                                    2 * (p0 + hr) - p.f_pad_h, img);
                } else if (p.halo_flat) {
                    if (leader) mbar_arrive_expect_tx(&hfull[stage], p.halo_tx);     // rows of Wh pixels as int64 elements: few long TMA rows
                    if (leader) tma_load_3d(dst, &hmap, &hfull[stage], -p.pad_w * (p.c_px / 8), p0 - p.pad_h, img);
                } else {
                    if (leader) mbar_arrive_expect_tx(&hfull[stage], p.halo_tx);
                    if (leader) tma_load_5d(dst, &hmap, &hfull[stage], 0, -p.pad_w, p0 - p.pad_h, img, 0);
                }
            }
        }
    } else if (warp == kMma) {
        // ===================== MMA issuer =====================
        {   // the whole warp runs the (uniform) loop, one elected lane issues
            const bool leader = lane == 0;
            // per-MMA descriptor offsets (16-byte units) are computed in registers: a table in
            // shared memory puts a generic load + its latency in front of every MMA issue
            const uint32_t bplane = static_cast<uint32_t>(p.BN) * 16u;
            const uint32_t a_pl16 = p.h_plane_bytes >> 4, b_pl16 = bplane >> 4;
            const int sstep = p.tap_pair ? 2 : 1;
            const int npl = p.tap_pair ? 1 : p.nplanes;
            const uint64_t bdesc0 = make_smem_desc(smem_u32(smem + p.off_bres), bplane, 128u, 0u);
            const uint32_t a_lbo = p.tap_pair ? 16u : p.h_plane_bytes;
            // per-MMA descriptor offsets (16-byte units), K order = (r, s, plane pair)
            uint32_t aoff[kHaloMaxMMA], boff[kHaloMaxMMA];
            const int nmma = p.n_mma;
            {
                int r = 0, sx = 0, j = 0;
#pragma unroll
                for (int i = 0; i < kHaloMaxMMA; ++i) {
                    const uint32_t tap = static_cast<uint32_t>(r * p.S + sx);
                    aoff[i] = static_cast<uint32_t>(r * p.Wh + sx) + static_cast<uint32_t>(j) * a_pl16;
                    boff[i] = (p.tap_pair ? tap : tap * static_cast<uint32_t>(p.nplanes) + static_cast<uint32_t>(j)) * b_pl16;
                    j += 2;
                    if (j >= npl) { j = 0; sx += sstep; if (sx >= p.S) { sx = 0; ++r; } }
                }
            }
            const uint64_t adesc_st = make_smem_desc(smem_u32(smem + p.off_hx), a_lbo, 128u, 0u);
            const uint32_t ahi = static_cast<uint32_t>(adesc_st >> 32);
            const uint32_t blo0 = static_cast<uint32_t>(bdesc0), bhi = static_cast<uint32_t>(bdesc0 >> 32);
            mbar_wait(bfull, 0);
            __syncwarp();
            tc_fence_after();
            int it = 0;
            int stage = 0;                           // ring position, advanced incrementally
            uint32_t phase = 0;
            int f_base = 0;                          // F32: ring row of the tile's halo row 0
            for (int tile = t_first; tile < t_end; tile += t_step, ++it) {
                const int buf = it & 1;
                const uint32_t acc_phase = static_cast<uint32_t>(it >> 1) & 1u;
                // operands first: after the accumulator hand-back only the fence and the issue remain
                mbar_wait(kCvt ? &hready[stage] : &hfull[stage], phase);
                if (leader) trace_ev(p, 3, it);
                mbar_wait(&tempty[buf], acc_phase ^ 1u);
                if (leader) trace_ev(p, 2, it);
                __syncwarp();
                tc_fence_after();
                if (leader) trace_ev(p, 1, it);
                const uint32_t d_tmem = tmem_base + static_cast<uint32_t>(buf * (CM ? 256 : p.BN));
                uint32_t alo0 = static_cast<uint32_t>(adesc_st) +
                                ((static_cast<uint32_t>(stage) * p.hx_stage_bytes) >> 4);
                if (F32) {   // the tile's window of the converter's code-row ring (same sequence)
                    const int mt = p.fd_ntn.div(tile);
                    const int p0 = (mt - p.fd_tpi.div(mt) * p.tiles_per_img) * p.Rt;
                    if (tile != t_first && p0 != 0 && p.Rt < p.HR) {
                        f_base += p.Rt;
                        if (f_base >= p.HR + p.Rt) f_base -= p.HR + p.Rt;
                    } else {
                        f_base = 0;
                    }
                    alo0 = static_cast<uint32_t>(adesc_st) + ((static_cast<uint32_t>(f_base) * static_cast<uint32_t>(p.Wh)));
                }
                // fully unrolled and branch-free over the precomputed per-MMA offsets (MMAs past
                // n_mma are predicated off).  The tensor pipe takes an M128 x N64 x K32 MMA from
                // shared memory per 52 cycles (scripts/micro/mma_bench3.cu); guarded by a branch
                // each, the issue chain paced them at ~150-270.
#pragma unroll
                for (int i = 0; i < kHaloMaxMMA; ++i) {
                    if (CM)      // A = the weights (M = 64 channels), B = the halo (N pixels)
                        mma_i8_warp_lo_if(d_tmem, blo0 + boff[i], bhi, alo0 + aoff[i], ahi, p.idesc,
                                          i > 0 ? 1u : 0u, i < nmma ? 1u : 0u);
                    else
                        mma_i8_warp_lo_if(d_tmem, alo0 + aoff[i], ahi, blo0 + boff[i], bhi, p.idesc,
                                          i > 0 ? 1u : 0u, i < nmma ? 1u : 0u);
                }
                if (leader) trace_ev(p, 11, it);
                mma_commit_warp(&hempty[stage]);
                if (leader) trace_ev(p, 12, it);
                mma_commit_warp(&tfull[buf]);
                if (leader) trace_ev(p, 4, it);
                if (++stage == NS) { stage = 0; phase ^= 1u; }
            }
        }
    } else if (CM && warp >= kEpi0 && warp < kEpi0 + kNEpi) {
        // ===================== channel-major epilogue (trans.cuh, M = 64) =====================
        // warp w: TMEM lanes 32 (w % 4) .. +15 (output channels 16 (w % 4) .. +15 as 8 pairs,
        // lanes l and l+8 = channels 2i, 2i+1 of the permuted weight rows), accumulator columns
        // 64 (w / 4) .. +63 (tile pixels; staging row = column, 8-row-aligned output rows)
        griddep_wait();                                   // params written in-stream
        const int ew = warp - kEpi0;
        const int quarter = warp & 3;
        const int sub = ew >> 2;
        constexpr bool kInt4 = (OUT == OUT_U4 || OUT == OUT_S4);
        constexpr int kRowBytes = 64 * (kInt4 ? 4 : 8) / 8;
        constexpr int kGMask = kRowBytes >= 128 ? 7 : (kRowBytes == 64 ? 3 : 1);
        const uint32_t lane_base = 32u * static_cast<uint32_t>(quarter);
        // two warp groups (sub >> 1) take alternating tiles; a warp covers 128 pixel columns
        const int gsel = sub >> 1;
        const int col_begin = (sub & 1) * 128;
        const int pair = 8 * quarter + (lane >> 2);
        const uint32_t boff = static_cast<uint32_t>(kInt4 ? pair : 2 * pair);
        const uint32_t ystg_base = smem_u32(smem + p.off_ystg);
        TChan ce{}, co{};
        int mode;
        {
            const int ke = 2 * pair, ko = ke + 1;
            int nee, neo;
            bool be, bo;
            t_chan_params(p, ke, ke < p.K, ce, nee, be);
            t_chan_params(p, ko, ko < p.K, co, neo, bo);
            const unsigned act = 0xffffffffu;
            const bool all_fast = __ballot_sync(act, be && bo && nee >= 33 && nee <= 52 && neo >= 33 && neo <= 52) == act;
            const bool all_mid = __ballot_sync(act, be && bo && nee >= 20 && nee <= 50 && neo >= 20 && neo <= 50 &&
                                                        mid_multiplier_ok(ce.m) && mid_multiplier_ok(co.m)) == act;
            mode = all_fast ? 0 : (all_mid ? 1 : 2);
            if (mode == 1) {
                const int T = max(33, __reduce_max_sync(act, max(nee, neo)));
                t_chan_mid(p, ce, nee, T);
                t_chan_mid(p, co, neo, T);
            }
        }
        const uint32_t taddr0 = tmem_base + (lane_base << 16) + static_cast<uint32_t>(col_begin);
        const int row0 = col_begin + 2 * (lane & 3);
        int it = gsel;
        for (int tile = t_first + gsel * t_step; tile < t_end; tile += 2 * t_step, it += 2) {
            const int buf = it & 1;
            const uint32_t acc_phase = static_cast<uint32_t>(it >> 1) & 1u;
            const int sb = it % NB;
            const uint32_t sphase = static_cast<uint32_t>(it / NB) & 1u;
            mbar_wait(&tfull[buf], acc_phase);
            tc_fence_after();
            if (ew == 0 && lane == 0) trace_ev(p, 5, it);
            mbar_wait(&sfree[sb], sphase ^ 1u);
            if (ew == 0 && lane == 0) trace_ev(p, 10, it);
            const uint32_t ystg = ystg_base + static_cast<uint32_t>(sb) * p.ystg_bytes;
#pragma unroll 1
            for (int t = 0; t < 2; ++t) {
                uint32_t va[32];
                tmem_ld_16x256b_x8(taddr0 + static_cast<uint32_t>(buf * 256 + 64 * t), va);
                // the multipliers re-enter the loop as plain 32-bit registers: hoisted out of it as
                // sign-extended 64-bit values they turned every product into a 64x64 multiply
                asm volatile("" : "+r"(ce.m), "+r"(co.m));
                tmem_wait_ld_regs(va);
                t_pairs_mode<OUT, kRowBytes, kGMask>(p, mode, ce, co, va, ystg, row0 + 64 * t, boff);
            }
            if (ew == 0 && lane == 0) trace_ev(p, 14, it);
            tc_fence_before();
            fence_proxy_async_smem();                 // staging writes -> visible to the TMA store
            __syncwarp();
            if (lane == 0) {
                mbar_arrive(&tempty[buf]);
                mbar_arrive(&sfull[sb]);
            }
            if (ew == 0 && lane == 0) trace_ev(p, 6, it);
        }
    } else if (!CM && warp >= kEpi0 && warp < kEpi0 + kNumEpiWarps) {
        // ===================== epilogue =====================
        griddep_wait();                                   // params written in-stream
        const int ew = warp - kEpi0;
        const int quarter = warp & 3;
        const int half = ew >> 2;
        const int row = quarter * 32 + lane;           // accumulator row = padded output index
        const int rr = row / p.Wh;
        const int qq = row - rr * p.Wh;
        const bool row_ok = rr < p.Rt && qq < p.Q;      // rows beyond P are clipped by the Y map
        const int srow = rr * p.Q + qq;                 // row inside the [Rt][Q] staging box
        const uint32_t par_base = smem_u32(par);
        const int nchunks = p.BN / 32;
        const uint32_t ystg_base = smem_u32(smem + p.off_ystg);
        fill_epilogue_params<OUT>(p, par, chunk_info, n0, ew, lane, false);
        const uint32_t cinfo_base = smem_u32(chunk_info);
        const uint32_t taddr0 = tmem_base + (static_cast<uint32_t>(quarter * 32) << 16);
        int it = 0;
        int sb = 0;                                      // staging buffer, advanced incrementally
        uint32_t sphase = 0;
        for (int tile = t_first; tile < t_end; tile += t_step, ++it) {
            const int buf = it & 1;
            const uint32_t acc_phase = static_cast<uint32_t>(it >> 1) & 1u;
            mbar_wait(&tfull[buf], acc_phase);
            if (ew == 0 && lane == 0) trace_ev(p, 5, it);
            tc_fence_after();
            const uint32_t taddr = taddr0 + static_cast<uint32_t>(buf * p.BN);
            mbar_wait(&sfree[sb], sphase ^ 1u);
            const uint32_t ystg_it = ystg_base + static_cast<uint32_t>(sb) * p.ystg_bytes;
            // TMEM loads double-buffered: chunk ci+2 is in flight while chunk ci is requantized
            uint32_t va[32], vb[32];
            auto process = [&](uint32_t (&v)[32], int ci) {
                const int col0 = ci * 32;
                const uint32_t pa = par_base + 16u * col0;
                const int4 cinfo = lds128(cinfo_base + 16u * static_cast<uint32_t>(ci));
                epi_requant16<OUT, false, 0>(p, v, pa, cinfo, n0 + col0, 0, 0, 0, 0);
                epi_requant16<OUT, false, 16>(p, v, pa, cinfo, n0 + col0, 0, 0, 0, 0);
                if (row_ok) {
                    stage16<OUT, 0>(p, v, ystg_it, srow, col0);
                    stage16<OUT, 16>(p, v, ystg_it, srow, col0 + 16);
                }
            };
            if (!kCvt) {  // 384-thread kernels have the registers to double-buffer
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
                if (ew == 0 && lane == 0) trace_ev(p, 10, it);
                for (int ci = half; ci < nchunks; ci += 2) {
                    __syncwarp();
                    tmem_ld_32x32b_x32(taddr + ci * 32, va);
                    tmem_wait_ld();
                    if (ew == 0 && lane == 0) trace_ev(p, 13, it);
                    process(va, ci);
                }
                if (ew == 0 && lane == 0) trace_ev(p, 14, it);
            }
            tc_fence_before();
            fence_proxy_async_smem();                 // staging writes -> visible to the TMA store
            __syncwarp();
            if (lane == 0) {
                mbar_arrive(&tempty[buf]);
                mbar_arrive(&sfull[sb]);
            }
            if (++sb == NB) { sb = 0; sphase ^= 1u; }
            if (ew == 0 && lane == 0) trace_ev(p, 6, it);
        }
    } else if (F32 && warp >= kCvt0 && warp < kCvt0 + kNumCvtWarps) {
        // ===================== fp32 -> space-to-depth codes (fused quantization) ===========
        // The byte-coded halo X2 lives in a ring of NR = HR + Rt rows, every row stored twice
        // (ring rows s and s + NR), so the HR rows of any tile are one contiguous window for
        // the MMA descriptors.  A fresh tile (first of the CTA's run or of an image) quantizes
        // its HR rows into ring rows 0..HR-1; a continuation tile only its Rt new rows (the run
        // is contiguous: the others are the previous tile's), Rt ring rows further on.  Those
        // rows last held rows of the tile two back (one back for a fresh tile), whose MMAs are
        // waited for first.  Per tile: shifts, adds, selects -- no divisions.
        const int ct = (warp - kCvt0) * 32 + lane;
        const int NR = p.HR + p.Rt;
        const uint32_t ring = smem_u32(smem + p.off_hx);
        const uint32_t rowpx = static_cast<uint32_t>(p.Wh) * 16u;
        const uint32_t mirror = static_cast<uint32_t>(NR) * rowpx;
        const uint32_t zero = ring + 2u * mirror;        // 64 zero bytes after the ring
        if (ct < 16) sts32(zero + 4u * ct, 0u);
        const int tile_px = p.Rt * p.Wh;
        // this thread's pixels of a continuation tile (Rt new rows: tile_px <= 256, so at most
        // two per thread): new row nr, column jc, source offsets
        constexpr int kMaxNew = 2;
        int nr[kMaxNew], jc[kMaxNew];
        uint32_t src_nr[kMaxNew], coff[kMaxNew][4], cok[kMaxNew];
#pragma unroll
        for (int u = 0; u < kMaxNew; ++u) {
            const int px = ct + u * kNumCvtWarps * 32;
            const int pq = px < tile_px ? px : 0;
            nr[u] = pq / p.Wh;
            jc[u] = pq - nr[u] * p.Wh;
            src_nr[u] = 2u * static_cast<uint32_t>(nr[u]) * static_cast<uint32_t>(p.f_rowbytes);
            cok[u] = f32_s2d_offsets(p, jc[u], coff[u]);
        }
        named_bar_sync(2, kNumCvtWarps * 32);           // the zero area is written
        int base = 0;                                    // ring row of the tile's halo row 0
        int g = 0;
        RingPos rp, rp1, rp2;                            // tiles g, g-1, g-2
        for (int tile = t_first; tile < t_end; tile += t_step, ++g, rp2 = rp1, rp1 = rp, rp.next(NS)) {
            const int stage = rp.stage;
            const int mt = p.fd_ntn.div(tile);
            const int p0 = (mt - p.fd_tpi.div(mt) * p.tiles_per_img) * p.Rt;
            const bool cont = tile != t_first && p0 != 0 && p.Rt < p.HR;
            // MMAs still reading the ring rows rewritten here: tile g-2 (g-1 for a fresh tile)
            if (cont ? g >= 2 : g >= 1) {
                const RingPos &rb = cont ? rp2 : rp1;
                mbar_wait(&hempty[rb.stage], rb.phase);
            }
            mbar_wait(&hfull[stage], rp.phase);
            if (ct == 0) trace_ev(p, 8, g);
            const uint32_t src = smem_u32(smem + p.off_hp + stage * p.hp_stage_bytes);
            if (cont) {
                base += p.Rt;
                if (base >= NR) base -= NR;
                // both pixels computed unconditionally (a thread without a second pixel redoes
                // its first), so the 2 x 12 load -> quantize chains interleave; stores predicated
                uint32_t w[kMaxNew][4];
#pragma unroll
                for (int u = 0; u < kMaxNew; ++u) {
                    uint32_t addr[4];
                    f32_s2d_addr(src + src_nr[u], coff[u], cok[u], zero, addr);
                    if (p.f_c == 3) f32_s2d_pixel<3>(p, addr, w[u]);
                    else f32_s2d_pixel<4>(p, addr, w[u]);
                }
#pragma unroll
                for (int u = 0; u < kMaxNew; ++u) {
                    if (ct + u * kNumCvtWarps * 32 < tile_px) {
                        // halo row HR - Rt + nr from staged rows 2 nr, 2 nr + 1
                        int slot = base + p.HR - p.Rt + nr[u];
                        if (slot >= NR) slot -= NR;
                        const uint32_t dst = ring + static_cast<uint32_t>(slot) * rowpx + 16u * static_cast<uint32_t>(jc[u]);
                        sts128(dst, w[u][0], w[u][1], w[u][2], w[u][3]);
                        sts128(dst + mirror, w[u][0], w[u][1], w[u][2], w[u][3]);
                    }
                }
            } else {
                base = 0;
                for (int px = ct; px < p.HR * p.Wh; px += kNumCvtWarps * 32) {
                    const int hr = px / p.Wh, j = px - (px / p.Wh) * p.Wh;
                    uint32_t off[4], addr[4], w[4];
                    const uint32_t ok = f32_s2d_offsets(p, j, off);
                    f32_s2d_addr(src + 2u * static_cast<uint32_t>(hr) * static_cast<uint32_t>(p.f_rowbytes), off, ok,
                                 zero, addr);
                    if (p.f_c == 3) f32_s2d_pixel<3>(p, addr, w);
                    else f32_s2d_pixel<4>(p, addr, w);
                    const uint32_t dst = ring + static_cast<uint32_t>(hr) * rowpx + 16u * static_cast<uint32_t>(j);
                    sts128(dst, w[0], w[1], w[2], w[3]);
                    sts128(dst + mirror, w[0], w[1], w[2], w[3]);
                }
            }
            fence_proxy_async_smem();                   // code rows -> visible to the MMA
            __syncwarp();
            if (lane == 0) mbar_arrive(&hready[stage]);
            if (ct == 0) trace_ev(p, 9, g);
        }
    } else if (IS4 && warp >= kCvt0 && warp < kCvt0 + kNumCvtWarps) {
        // ===================== int4 -> int8 plane widening =====================
        // packed plane j (16 B = 32 channels per pixel) -> int8 planes 2j (channels 0..15)
        // and 2j+1 (16..31) at the same pixel offset
        const int ct = (warp - kCvt0) * 32 + lane;
        const uint32_t xo = p.x_sgn4 ? 0x88888888u : 0u;
        const int npix = p.HR * p.Wh;
        int g = 0;
        RingPos rp;
        for (int tile = t_first; tile < t_end; tile += t_step, ++g, rp.next(NS)) {
            const int stage = rp.stage;
            mbar_wait(&hfull[stage], rp.phase);
            if (ct == 0) trace_ev(p, 8, g);
            const uint32_t src = smem_u32(smem + p.off_hp + stage * p.hp_stage_bytes);
            const uint32_t dst = smem_u32(smem + p.off_hx + stage * p.hx_stage_bytes);
            constexpr int kStride = kNumCvtWarps * 32;
            constexpr int U = 4;            // loads batched ahead of the conversion
            // packed 16-byte chunk j of pixel px: plane-major staging (5-D load) or pixel-major
            // staging (flat load)
            const uint32_t sstr = p.halo_flat ? static_cast<uint32_t>(p.c_px) : 16u;
            for (int j = 0; j < p.nplanes / 2; ++j) {
                const uint32_t sj = src + (p.halo_flat ? 16u * static_cast<uint32_t>(j)
                                                       : static_cast<uint32_t>(j * npix) * 16u);
                const uint32_t dj = dst + static_cast<uint32_t>(2 * j) * p.h_plane_bytes;
                int px = ct;
                for (; px + (U - 1) * kStride < npix; px += U * kStride) {
                    uint4 pk[U];
#pragma unroll
                    for (int u = 0; u < U; ++u) pk[u] = lds128u(sj + static_cast<uint32_t>(px + u * kStride) * sstr);
#pragma unroll
                    for (int u = 0; u < U; ++u) {
                        uint32_t o[8];
                        widen_word(pk[u].x, xo, o[0], o[4]);
                        widen_word(pk[u].y, xo, o[1], o[5]);
                        widen_word(pk[u].z, xo, o[2], o[6]);
                        widen_word(pk[u].w, xo, o[3], o[7]);
                        const uint32_t d0 = dj + static_cast<uint32_t>(px + u * kStride) * 16u;
                        sts128(d0, o[0], o[1], o[2], o[3]);
                        sts128(d0 + p.h_plane_bytes, o[4], o[5], o[6], o[7]);
                    }
                }
                for (; px < npix; px += kStride) {
                    const uint4 pk = lds128u(sj + static_cast<uint32_t>(px) * sstr);
                    uint32_t o[8];
                    widen_word(pk.x, xo, o[0], o[4]);
                    widen_word(pk.y, xo, o[1], o[5]);
                    widen_word(pk.z, xo, o[2], o[6]);
                    widen_word(pk.w, xo, o[3], o[7]);
                    const uint32_t d0 = dj + static_cast<uint32_t>(px) * 16u;
                    sts128(d0, o[0], o[1], o[2], o[3]);
                    sts128(d0 + p.h_plane_bytes, o[4], o[5], o[6], o[7]);
                }
            }
            fence_proxy_async_smem();
            __syncwarp();
            if (lane == 0) mbar_arrive(&hready[stage]);
            if (ct == 0) trace_ev(p, 9, g);
        }
    }

    tc_fence_before();
    __syncthreads();
    if (warp == kMma) {
        __syncwarp();
        tc_fence_after();
        tmem_dealloc(tmem_base, p.tmem_cols);
    }
}

}  // namespace qc
