// fwd2.cuh -- CTA-pair (cta_group::2) variant of the im2col implicit-GEMM conv.
//
// Same method as conv_fwd.cuh (Alg.2, fused epilogue P:L223/P:L253/P:L265); the
// two CTAs of a cluster share one UMMA of M = 256 output pixels x N = BN output channels:
// CTA r loads its 128 pixels of A and BN/2 rows of B per K-stage, the leader (rank 0) issues
// `tcgen05.mma.cta_group::2`, and each CTA's TMEM receives its 128 rows of the accumulator.
// Per CTA the shared-memory traffic per MAC drops by a third (B is split, not replicated),
// which is what bounds the single-CTA kernel at N = 256.
//
// Cross-CTA protocol (all mbarriers live in each CTA at the same offsets):
//   full[s]  (local)  : TMA landed (8-bit) / aready[s] (local): converter done (4-bit)
//   8-bit: rank 1's TMA loads complete_tx on the LEADER's full[s] (.cta_group::2)
//   4-bit: aready[s] (leader) counts both CTAs' converter warps (remote arrives from rank 1)
//   empty[s] (both)   : the pair's MMAs of stage s completed -- multicast commit
//   tfull[b] (both)   : accumulator b complete -- multicast commit
//   tempty[b](leader) : both CTAs' epilogue warps drained accumulator b -- local + remote arrives
#pragma once
#ifndef QC_REMOTE_RELEASE_CLUSTER
#define QC_REMOTE_RELEASE_CLUSTER 0
#endif
#include "epilogue.cuh"

namespace qc {

__device__ __forceinline__ uint32_t cluster_ctarank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ void cluster_sync_all() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ uint32_t mapa_shared(uint32_t addr, uint32_t rank) {
    uint32_t r;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(addr), "r"(rank));
    return r;
}
__device__ __forceinline__ void mbar_wait_cluster(uint64_t *bar, uint32_t parity) {
    const uint32_t a = smem_u32(bar);
    uint32_t ok = 0;
    uint64_t t0 = 0;
    uint32_t n = 0;
    while (true) {
        asm volatile(
            "{\n\t.reg .pred p;\n\t"
            "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 p, [%1], %2;\n\t"
            "selp.u32 %0, 1, 0, p;\n\t}"
            : "=r"(ok)
            : "r"(a), "r"(parity)
            : "memory");
        if (ok) return;
        if ((++n & 63u) == 0) {
            const uint64_t t = globaltimer_ns();
            if (t0 == 0) t0 = t;
            else if (t - t0 > 4000000000ull) __trap();
        }
    }
}
// Remote arrive with the default (.release.cta) semantics, as CUTLASS's ClusterBarrier does: a
// .release.cluster arrive costs the converter warps ~0.5 us per stage (measured, trace_fwd2.py;
// re-measured late in round 2 with -DQC_REMOTE_RELEASE_CLUSTER=1: 4-bit pair family 537 -> 913 us
// per A4W4 step, 8-bit 433 -> 455).
// The data the leader's MMA then reads stays in this CTA's shared memory, made visible to the
// async proxy by the preceding fence.proxy.async.
__device__ __forceinline__ void mbar_arrive_remote(uint32_t cluster_addr) {
#if QC_REMOTE_RELEASE_CLUSTER
    // release at cluster scope: the peer's shared-memory / TMEM work before the arrive is
    // ordered before the leader's acquire.cluster wait (PTX memory model, cross-CTA)
    asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(cluster_addr) : "memory");
#else
    asm volatile("mbarrier.arrive.shared::cluster.b64 _, [%0];" ::"r"(cluster_addr) : "memory");
#endif
}
__device__ __forceinline__ void tmem_alloc2(uint32_t *dst_smem, uint32_t ncols) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(dst_smem)),
                 "r"(ncols)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
}
__device__ __forceinline__ void tmem_dealloc2(uint32_t taddr, uint32_t ncols) {
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(taddr), "r"(ncols) : "memory");
}
__device__ __forceinline__ void mma2_i8_warp_lo(uint32_t d_tmem, uint32_t alo, uint32_t ahi, uint32_t blo,
                                                uint32_t bhi, uint32_t idesc, uint32_t accumulate) {
    asm volatile(
        "{\n\t.reg .pred p, e;\n\t.reg .b64 da, db;\n\t"
        "setp.ne.b32 p, %6, 0;\n\t"
        "mov.b64 da, {%1, %2};\n\t"
        "mov.b64 db, {%3, %4};\n\t"
        "elect.sync _|e, 0xffffffff;\n\t"
        "@e tcgen05.mma.cta_group::2.kind::i8 [%0], da, db, %5, p;\n\t}" ::"r"(d_tmem),
        "r"(alo), "r"(ahi), "r"(blo), "r"(bhi), "r"(idesc), "r"(accumulate)
        : "memory");
}
// Same, issued only when `active` is non-zero: a fully unrolled, branch-free run (see
// ptx.cuh mma_i8_warp_lo_if: branch-guarded MMAs each wait for their own operand moves).
__device__ __forceinline__ void mma2_i8_warp_lo_if(uint32_t d_tmem, uint32_t alo, uint32_t ahi, uint32_t blo,
                                                   uint32_t bhi, uint32_t idesc, uint32_t accumulate,
                                                   uint32_t active) {
    asm volatile(
        "{\n\t.reg .pred p, e, q;\n\t.reg .b64 da, db;\n\t"
        "setp.ne.b32 p, %6, 0;\n\t"
        "setp.ne.b32 q, %7, 0;\n\t"
        "mov.b64 da, {%1, %2};\n\t"
        "mov.b64 db, {%3, %4};\n\t"
        "elect.sync _|e, 0xffffffff;\n\t"
        "and.pred e, e, q;\n\t"
        "@e tcgen05.mma.cta_group::2.kind::i8 [%0], da, db, %5, p;\n\t}" ::"r"(d_tmem),
        "r"(alo), "r"(ahi), "r"(blo), "r"(bhi), "r"(idesc), "r"(accumulate), "r"(active)
        : "memory");
}
// commit to the barrier at the same offset in both CTAs of the pair
__device__ __forceinline__ void mma2_commit_mc_warp(uint64_t *bar) {
    asm volatile(
        "{\n\t.reg .pred e;\n\t"
        "elect.sync _|e, 0xffffffff;\n\t"
        "@e tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;\n\t}" ::"r"(
            smem_u32(bar)),
        "h"(static_cast<uint16_t>(3))
        : "memory");
}

// TMA loads into this CTA's shared memory that complete_tx on the LEADER's mbarrier
// (`bar_cluster` = its shared::cluster address): .cta_group::2 lets the barrier be the peer's.
__device__ __forceinline__ void tma2_load_2d(void *dst, const void *map, uint32_t bar_cluster, int32_t x, int32_t y) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes.cta_group::2"
        " [%0], [%1, {%3, %4}], [%2];" ::"r"(smem_u32(dst)),
        "l"(map), "r"(bar_cluster), "r"(x), "r"(y)
        : "memory");
}
__device__ __forceinline__ void tma2_load_im2col_4d(void *dst, const void *map, uint32_t bar_cluster, int32_t c,
                                                    int32_t w, int32_t h, int32_t n, uint16_t off_w, uint16_t off_h) {
    asm volatile(
        "cp.async.bulk.tensor.4d.shared::cluster.global.im2col.mbarrier::complete_tx::bytes.cta_group::2"
        " [%0], [%1, {%3, %4, %5, %6}], [%2], {%7, %8};" ::"r"(smem_u32(dst)),
        "l"(map), "r"(bar_cluster), "r"(c), "r"(w), "r"(h), "r"(n), "h"(off_w), "h"(off_h)
        : "memory");
}

// debug (QC_TRACE): events of CTA `cta` of the first pair
#ifdef QC_DEBUG
__device__ __forceinline__ void trace_ev2(const ConvParams &p, int ev, int seq, uint32_t cta) {
    if (p.trace != nullptr && blockIdx.x == cta && seq < 1024) p.trace[ev * 1024 + seq] = globaltimer_ns();
}
#else
__device__ __forceinline__ void trace_ev2(const ConvParams &, int, int, uint32_t) {}
#endif

template <bool IS4, int OUT>
__global__ void __launch_bounds__(IS4 ? 512 : 384, 1)
qconv_fwd2_kernel(const __grid_constant__ CUtensorMap xmap, const __grid_constant__ CUtensorMap wmap,
                  const __grid_constant__ CUtensorMap ymap, const __grid_constant__ ConvParams p) {
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    // 1024-byte aligned base by pointer arithmetic on the shared array itself (no integer round
    // trip): the compiler keeps it in the shared window, so every smem_u32() below is one add
    uint8_t *smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;
    const int NS = p.stages;
    const uint32_t rank = cluster_ctarank();
    const int pair = static_cast<int>(blockIdx.x >> 1), npairs = static_cast<int>(gridDim.x >> 1);
    const int half_bn = p.BN / 2;

    uint64_t *bars = reinterpret_cast<uint64_t *>(smem + p.off_bar);
    uint64_t *full = bars;                  // [NS]
    uint64_t *empty = bars + NS;            // [NS]
    uint64_t *aready = bars + 2 * NS;       // [NS]
    uint64_t *peer = bars + 3 * NS;         // [NS] (leader)
    uint64_t *tfull = bars + 4 * NS;        // [2]
    uint64_t *tempty = bars + 4 * NS + 2;   // [2] (leader)
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(bars + 4 * NS + 4);
    EpiCol *par = reinterpret_cast<EpiCol *>(smem + p.off_par);
    int4 *chunk_info = reinterpret_cast<int4 *>(smem + p.off_par + 16 * kMaxBN);

    griddep_launch_dependents();
    if (warp == kWarpTMA && lane == 0) {
        tma_prefetch_desc(&xmap);
        tma_prefetch_desc(&wmap);
        tma_prefetch_desc(&ymap);
        for (int i = 0; i < NS; ++i) {
            mbar_init(&full[i], 1);
            mbar_init(&empty[i], 1);
            mbar_init(&aready[i], 2 * kNumCvtWarps);   // leader: both CTAs' converter warps
            mbar_init(&peer[i], 1);
        }
        for (int i = 0; i < 2; ++i) {
            mbar_init(&tfull[i], 1);
            mbar_init(&tempty[i], 2 * kNumEpiWarps);
        }
        fence_mbar_init();
    }
    if (warp == kWarpMMA) tmem_alloc2(tmem_slot, p.tmem_cols);
    tc_fence_before();
    cluster_sync_all();                     // both CTAs' barriers initialised, TMEM allocated
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;
    const int taps_per_r = p.S * p.chunks;

    if (warp == kWarpTMA || warp == 2 || warp == 3) {
        // ===================== TMA producers: this CTA's A rows and B half =====================
        if (lane == 0) {
            griddep_wait();
            const int pi = warp == kWarpTMA ? 0 : warp - 1;
            const uint32_t tx = static_cast<uint32_t>(kBM * p.bkp + half_bn * p.BK);
            int g = 0;
            for (int tile = pair; tile < p.num_tiles; tile += npairs) {
                const int mt = p.fd_ntn.div(tile);
                const int m0 = mt * (2 * kBM) + static_cast<int>(rank) * kBM;
                const int n0 = (tile - mt * p.n_tiles_n) * p.BN + static_cast<int>(rank) * half_bn;
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
                    trace_ev2(p, rank ? 7 : 0, g, rank);
                    const int r = p.fd_tpr.div(kb);
                    const int rem2 = kb - r * taps_per_r;
                    const int s = p.fd_chunks.div(rem2);
                    const int ch = rem2 - s * p.chunks;
                    uint8_t *adst = IS4 ? smem + p.off_stg + stage * p.stg_stage_bytes
                                        : smem + p.off_a + stage * p.a_stage_bytes;
                    if (IS4 || rank == 0) {
                        // 4-bit: local barrier (the converter widens, the relay tells the leader);
                        // 8-bit leader: the barrier also receives the peer's bytes
                        mbar_arrive_expect_tx(&full[stage], (!IS4 ? 2u : 1u) * tx);
                        tma_load_im2col_4d(adst, &xmap, &full[stage], ch * p.bkp, wb, hb, img,
                                           static_cast<uint16_t>(s * p.dil_w), static_cast<uint16_t>(r * p.dil_h));
                        tma_load_2d(smem + p.off_b + stage * p.b_stage_bytes, &wmap, &full[stage],
                                    (r * p.S + s) * p.C8 + ch * p.BK, n0);
                    } else {
                        // 8-bit peer: its loads complete on the leader's barrier directly
                        const uint32_t lb = mapa_shared(smem_u32(&full[stage]), 0);
                        tma2_load_im2col_4d(adst, &xmap, lb, ch * p.bkp, wb, hb, img,
                                            static_cast<uint16_t>(s * p.dil_w), static_cast<uint16_t>(r * p.dil_h));
                        tma2_load_2d(smem + p.off_b + stage * p.b_stage_bytes, &wmap, lb,
                                     (r * p.S + s) * p.C8 + ch * p.BK, n0);
                    }
                }
            }
        }
    } else if (warp == kWarpMMA) {
        if (rank != 0) {
            // the peer's stage readiness reaches the leader directly: its 8-bit TMA loads
            // complete on the leader's `full`, its 4-bit converter warps arrive on the leader's
            // `aready` -- the peer's MMA warp has nothing to do
        } else {
            // ===================== MMA issuer (leader, whole warp, one elected lane) =============
            int stage = 0;
            uint32_t phase = 0;
            int it = 0, gs = 0;
            const uint32_t sbo = 8u * static_cast<uint32_t>(p.BK);
            const int ksteps = p.BK / 32;
            for (int tile = pair; tile < p.num_tiles; tile += npairs, ++it) {
                const int buf = it & 1;
                const uint32_t acc_phase = static_cast<uint32_t>(it >> 1) & 1u;
                mbar_wait_cluster(&tempty[buf], acc_phase ^ 1u);
                __syncwarp();
                tc_fence_after();
                const uint32_t d_tmem = tmem_base + static_cast<uint32_t>(buf * p.BN);
                for (int kb = 0; kb < p.num_kb; ++kb) {
                    trace_ev2(p, 2, gs, 0);
                    if (IS4) {
                        mbar_wait_cluster(&aready[stage], phase);   // both CTAs' A widened
                    } else {
                        mbar_wait_cluster(&full[stage], phase);   // both CTAs' bytes landed
                    }
                    __syncwarp();
                    tc_fence_after();
                    const uint64_t ad0 = make_smem_desc(smem_u32(smem + p.off_a + stage * p.a_stage_bytes), 16u, sbo,
                                                        p.sw_layout);
                    const uint64_t bd0 = make_smem_desc(smem_u32(smem + p.off_b + stage * p.b_stage_bytes), 16u, sbo,
                                                        p.sw_layout);
                    const uint32_t alo = static_cast<uint32_t>(ad0), ahi = static_cast<uint32_t>(ad0 >> 32);
                    const uint32_t blo = static_cast<uint32_t>(bd0), bhi = static_cast<uint32_t>(bd0 >> 32);
#pragma unroll
                    for (int k = 0; k < 4; ++k)
                        mma2_i8_warp_lo_if(d_tmem, alo + 2u * k, ahi, blo + 2u * k, bhi, p.idesc,
                                           (kb | k) != 0 ? 1u : 0u, k < ksteps ? 1u : 0u);
                    mma2_commit_mc_warp(&empty[stage]);
                    if (lane == 0) trace_ev2(p, 3, gs, 0);
                    ++gs;
                    if (++stage == NS) { stage = 0; phase ^= 1u; }
                }
                mma2_commit_mc_warp(&tfull[buf]);
            }
        }
    } else if (warp >= kWarpEpi0 && warp < kWarpEpi0 + kNumEpiWarps) {
        // ===================== epilogue: this CTA's 128 rows =====================
        griddep_wait();
        const int ew = warp - kWarpEpi0;
        const int quarter = warp & 3;
        const int half = ew >> 2;
        const int row = quarter * 32 + lane;
        const uint32_t par_base = smem_u32(par);
        const int nchunks = (p.BN + 31) / 32;
        const uint32_t tempty0 = mapa_shared(smem_u32(tempty), 0);
        int cached_n0 = -1;
        int it = 0;
        const uint32_t ystg_base = smem_u32(smem + p.off_ystg);
        for (int tile = pair; tile < p.num_tiles; tile += npairs, ++it) {
            const int buf = it & 1;
            const uint32_t acc_phase = static_cast<uint32_t>(it >> 1) & 1u;
            const int mt = p.fd_ntn.div(tile);
            const int m0 = mt * (2 * kBM) + static_cast<int>(rank) * kBM;
            const int n0 = (tile - mt * p.n_tiles_n) * p.BN;
            if (n0 != cached_n0) {
                fill_epilogue_params<OUT>(p, par, chunk_info, n0, ew, lane, false);
                cached_n0 = n0;
            }
            mbar_wait(&tfull[buf], acc_phase);
            tc_fence_after();
            const uint32_t taddr = tmem_base + (static_cast<uint32_t>(quarter * 32) << 16) +
                                   static_cast<uint32_t>(buf * p.BN);
            // one staging buffer (more room for the ring): the previous store must have read it
            const bool storer = ew == 0 && lane == 0;
            if (storer) bulk_wait_read<0>();
            named_bar_sync(1, kNumEpiWarps * 32);
            const uint32_t ystg_it = ystg_base;
            for (int ci = half; ci < nchunks; ci += 2) {
                uint32_t v[32];
                __syncwarp();
                tmem_ld_32x32b_x32(taddr + ci * 32, v);
                tmem_wait_ld();
                const int col0 = ci * 32;
                const uint32_t pa = par_base + 16u * col0;
                const int4 cinfo = chunk_info[ci];
                epi_requant16<OUT, false, 0>(p, v, pa, cinfo, n0 + col0, 0, 0, 0, 0);
                epi_requant16<OUT, false, 16>(p, v, pa, cinfo, n0 + col0, 0, 0, 0, 0);
                stage16<OUT, 0>(p, v, ystg_it, row, col0);
                stage16<OUT, 16>(p, v, ystg_it, row, col0 + 16);
            }
            tc_fence_before();
            __syncwarp();
            if (lane == 0) {
                if (rank == 0) mbar_arrive(&tempty[buf]);
                else mbar_arrive_remote(tempty0 + 8u * static_cast<uint32_t>(buf));
            }
            fence_proxy_async_smem();
            named_bar_sync(1, kNumEpiWarps * 32);
            if (storer) {
                constexpr int kBits = (OUT == OUT_U4 || OUT == OUT_S4) ? 4 : 8;
                for (int g = 0; g < p.n_ygroups; ++g)
                    tma_store_2d(&ymap, smem + p.off_ystg + g * 128 * p.y_gw,
                                 n0 * kBits / 8 + g * p.y_gw, m0);
                bulk_commit();
            }
        }
        if (ew == 0 && lane == 0) bulk_wait<0>();
    } else if (IS4 && warp >= kWarpCvt0 && warp < kWarpCvt0 + kNumCvtWarps) {
        // ===================== int4 -> int8 widening of this CTA's A rows =====================
        const int ct = (warp - kWarpCvt0) * 32 + lane;
        const int cshift = p.cvt_shift;
        const int nchunks = kBM << cshift;
        const uint32_t xo = p.x_sgn4 ? 0x88888888u : 0u;
        const uint32_t sw = static_cast<uint32_t>(p.sw_mask);
        const uint32_t bkb = static_cast<uint32_t>(p.BK);
        const uint32_t aready0 = mapa_shared(smem_u32(aready), 0);
        int cg = 0;
        int stage = 0;
        uint32_t phase = 0;
        for (int tile = pair; tile < p.num_tiles; tile += npairs) {
            for (int kb = 0; kb < p.num_kb; ++kb) {
                mbar_wait(&full[stage], phase);
                if (ct == 0) trace_ev2(p, rank ? 8 : 5, cg, rank);
                const uint32_t stg = smem_u32(smem + p.off_stg + stage * p.stg_stage_bytes);
                const uint32_t adst = smem_u32(smem + p.off_a + stage * p.a_stage_bytes);
                widen_stage(stg, adst, ct, nchunks, cshift, bkb, sw, xo, static_cast<uint32_t>(p.stg_sw));
                fence_proxy_async_smem();
                __syncwarp();
                if (lane == 0) {
                    if (rank == 0) mbar_arrive(&aready[stage]);
                    else mbar_arrive_remote(aready0 + 8u * static_cast<uint32_t>(stage));
                }
                if (ct == 0) trace_ev2(p, rank ? 9 : 6, cg, rank);
                ++cg;
                if (++stage == NS) { stage = 0; phase ^= 1u; }
            }
        }
    }

    tc_fence_before();
    cluster_sync_all();                     // nobody frees TMEM / exits while the pair is working
    if (warp == kWarpMMA) {
        __syncwarp();
        tc_fence_after();
        tmem_dealloc2(tmem_base, p.tmem_cols);
    }
}

}  // namespace qc
