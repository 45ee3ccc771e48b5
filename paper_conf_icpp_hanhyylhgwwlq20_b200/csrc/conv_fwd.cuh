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
#include "epilogue.cuh"

namespace qc {

template <bool IS4, int OUT, bool ZX>
__global__ void __launch_bounds__(IS4 ? 512 : 384, 1)
qconv_fwd_kernel(const __grid_constant__ CUtensorMap xmap, const __grid_constant__ CUtensorMap wmap,
                 const __grid_constant__ CUtensorMap ymap, const __grid_constant__ ConvParams p) {
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    // 1024-byte aligned base by pointer arithmetic on the shared array itself (no integer round
    // trip): the compiler keeps it in the shared window, so every smem_u32() below is one add
    uint8_t *smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
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
                const int mt = p.fd_ntn.div(tile);
                const int m0 = mt * kBM;
                const int n0 = (tile - mt * p.n_tiles_n) * p.BN;
                const int img = p.fd_pq.div(m0);
                const int rem = m0 - img * p.PQ;
                const int p0 = p.fd_q.div(rem);
                const int q0 = rem - p0 * p.Q;
                const int wb = q0 * p.stride_w - p.pad_w;
                const int hb = p0 * p.stride_h - p.pad_h;
                for (int kb = 0; kb < p.num_kb; ++kb, ++g) {
                    if (g % kNumProducers != pi) continue;
                    const int stage = g % NS;
                    const uint32_t phase = static_cast<uint32_t>(g / NS) & 1u;
                    mbar_wait(&empty[stage], phase ^ 1u);
                    if (leader) trace_ev(p, 0, g);
                    if (leader) mbar_arrive_expect_tx(&full[stage], tx);
                    if (p.pair) {
                        const int RS = p.R * p.S;
                        const int t0 = 2 * kb, t1 = t0 + 1;
                        const int r0 = p.fd_s.div(t0), s0 = t0 - r0 * p.S;
                        int r1 = r0, s1 = s0, kg1 = RS * 16;        // odd tail: B slot OOB -> 0
                        if (t1 < RS) { r1 = p.fd_s.div(t1); s1 = t1 - r1 * p.S; kg1 = t1 * 16; }
                        uint8_t *adst = smem + p.off_a + stage * p.a_stage_bytes;
                        uint8_t *bdst = smem + p.off_b + stage * p.b_stage_bytes;
                        if (leader) tma_load_im2col_4d(adst, &xmap, &full[stage], 0, wb, hb, img,
                                           static_cast<uint16_t>(s0 * p.dil_w), static_cast<uint16_t>(r0 * p.dil_h));
                        if (leader) tma_load_im2col_4d(adst + kBM * 16, &xmap, &full[stage], 0, wb, hb, img,
                                           static_cast<uint16_t>(s1 * p.dil_w), static_cast<uint16_t>(r1 * p.dil_h));
                        if (leader) tma_load_2d(bdst, &wmap, &full[stage], t0 * 16, n0);
                        if (leader) tma_load_2d(bdst + p.BN * 16, &wmap, &full[stage], kg1, n0);
                    } else {
                        const int r = p.fd_tpr.div(kb);
                        const int rem2 = kb - r * taps_per_r;
                        const int s = p.fd_chunks.div(rem2);
                        const int ch = rem2 - s * p.chunks;
                        uint8_t *adst = IS4 ? smem + p.off_stg + stage * p.stg_stage_bytes
                                            : smem + p.off_a + stage * p.a_stage_bytes;
                        if (leader) tma_load_im2col_4d(adst, &xmap, &full[stage], ch * p.bkp, wb, hb, img,
                                               static_cast<uint16_t>(s * p.dil_w),
                                               static_cast<uint16_t>(r * p.dil_h));
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
                    if (IS4 && p.a_tmem_col > 0) {
                        // widened A rows in TMEM (converter warps), B from shared memory
                        const uint64_t bd0 = make_smem_desc(b_addr, 16u, sbo, p.sw_layout);
                        const uint32_t blo = static_cast<uint32_t>(bd0), bhi = static_cast<uint32_t>(bd0 >> 32);
                        const uint32_t a_t = tmem_base + static_cast<uint32_t>(p.a_tmem_col + stage * (p.BK / 4));
                        if (ksteps == 4) {
#pragma unroll
                            for (int k = 0; k < 4; ++k)
                                mma_i8_ts_warp(d_tmem, a_t + 8u * k, blo + 2u * k, bhi, p.idesc, (kb | k) != 0 ? 1u : 0u);
                        } else {
                            for (int k = 0; k < ksteps; ++k)
                                mma_i8_ts_warp(d_tmem, a_t + 8u * k, blo + 2u * k, bhi, p.idesc, (kb | k) != 0 ? 1u : 0u);
                        }
                    } else if (p.pair) {
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
                                mma_i8_warp_lo(d_tmem, alo + 2u * k, ahi, blo + 2u * k, bhi, p.idesc,
                                                   (kb | k) != 0 ? 1u : 0u);
                        } else {
                            for (int k = 0; k < ksteps; ++k)
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
        const bool force_general = ZX;
        int cached_n0 = -1;
        int it = 0;
        const uint32_t ystg_base = smem_u32(smem + p.off_ystg);
        for (int tile = blockIdx.x; tile < p.num_tiles; tile += gridDim.x, ++it) {
            const int buf = it & 1;
            const uint32_t acc_phase = static_cast<uint32_t>(it >> 1) & 1u;
            const int mt = p.fd_ntn.div(tile);
            const int m0 = mt * kBM;
            const int n0 = (tile - mt * p.n_tiles_n) * p.BN;
            if (n0 != cached_n0) {
                fill_epilogue_params<OUT>(p, par, chunk_info, n0, ew, lane, force_general);
                cached_n0 = n0;
            }
            const int64_t m = static_cast<int64_t>(m0) + row;
            const bool row_ok = m < p.M;
            int zr0 = 0, zr1 = 0, zs0 = 0, zs1 = 0;
            int32_t x1v = 0;
            if (ZX) {
                if (p.x1 != nullptr && row_ok) x1v = __ldg(p.x1 + m);
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
            if (OutTraits<OUT>::kPacked && p.y_tma) {
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
                    epi_requant16<OUT, ZX, 0>(p, vv, pa, cinfo, n0 + col0, zr0, zr1, zs0, zs1, x1v);
                    epi_requant16<OUT, ZX, 16>(p, vv, pa, cinfo, n0 + col0, zr0, zr1, zs0, zs1, x1v);
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
                if (storer) {
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
                    epi_half<OUT, ZX, 0>(p, v, pa, cinfo, n0 + col0, m, row_ok, zr0, zr1, zs0, zs1, x1v);
                    if (nc == 32)
                        epi_half<OUT, ZX, 16>(p, v, pa, cinfo, n0 + col0 + 16, m, row_ok, zr0, zr1, zs0, zs1, x1v);
                }
            }
            tc_fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive(&tempty[buf]);
        }
        if (OutTraits<OUT>::kPacked && p.y_tma && ew == 0 && lane == 0) bulk_wait<0>();
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
                if (p.a_tmem_col > 0) {
                    // thread = accumulator row m = ct: its pixel's bkp packed bytes -> 2 bkp widened
                    // bytes (chunk q: lo words then hi words, the order widen_stage writes) ->
                    // TMEM lane m, columns a_tmem_col + stage BK/4 ..  The packed staging is
                    // TMA-swizzled (16-byte chunk index ^= address bits 7+): conflict-free rows.
                    uint32_t o[32];
                    const uint32_t ssw = static_cast<uint32_t>(p.stg_sw);
                    const uint32_t rowoff = static_cast<uint32_t>(ct) * static_cast<uint32_t>(p.bkp);
                    // all four loads first (a short row reads past its end into the next row /
                    // stage, unused), then the widening: one latency, not four
                    uint4 v[4];
#pragma unroll
                    for (int q = 0; q < 4; ++q) {
                        const uint32_t so = rowoff + 16u * q;
                        v[q] = lds128u(stg + (so ^ (((so >> 7) & ssw) << 4)));
                    }
#pragma unroll
                    for (int q = 0; q < 4; ++q) {
                        widen_word(v[q].x, xo, o[8 * q + 0], o[8 * q + 4]);
                        widen_word(v[q].y, xo, o[8 * q + 1], o[8 * q + 5]);
                        widen_word(v[q].z, xo, o[8 * q + 2], o[8 * q + 6]);
                        widen_word(v[q].w, xo, o[8 * q + 3], o[8 * q + 7]);
                    }
                    const uint32_t ta = tmem_base + (static_cast<uint32_t>((warp & 3) * 32) << 16) +
                                        static_cast<uint32_t>(p.a_tmem_col + stage * (p.BK / 4));
                    if (p.bkp == 64) tmem_st_32x32b_x32(ta, o);
                    else if (p.bkp == 32) tmem_st_32x32b_x16(ta, o);
                    else tmem_st_32x32b_x8(ta, o);
                    tmem_wait_st();
                    tc_fence_before();
                } else {
                    const uint32_t adst = smem_u32(smem + p.off_a + stage * p.a_stage_bytes);
                    widen_stage(stg, adst, ct, nchunks, cshift, bkb, sw, xo, static_cast<uint32_t>(p.stg_sw));
                }
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

}  // namespace qc
