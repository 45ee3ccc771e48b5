// Microbenchmark: TMA load throughput per SM for im2col vs tiled boxes of various widths.
// Each CTA (one per SM) streams NLOADS loads through an NS-deep mbarrier ring; reports
// cycles per load and bytes/cycle/SM.  Build: nvcc -arch=sm_100a -O2 tma_bench.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <vector>

__device__ __forceinline__ uint32_t s32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int MODE>  // 0 = tiled 2D, 1 = im2col 4D, 2 = tiled 4D {c,w,h,n}
__global__ void bench(const __grid_constant__ CUtensorMap map, int nloads, int bytes, int ns,
                      int wmax, int hmax, long long *out) {
    extern __shared__ __align__(1024) uint8_t smem_all[];
    __shared__ __align__(8) uint64_t bars_all[4][32];
    const int wid = threadIdx.x / 32;
    uint64_t *bars = bars_all[wid];
    uint8_t *smem = smem_all + wid * ns * ((bytes + 1023) / 1024 * 1024);
    if ((threadIdx.x & 31) == 0) {
        for (int i = 0; i < ns; ++i) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(s32(&bars[i])));
        asm volatile("fence.mbarrier_init.release.cluster;");
        asm volatile("prefetch.tensormap [%0];" ::"l"(&map) : "memory");
    }
    __syncthreads();
    if ((threadIdx.x & 31) != 0) return;
    long long t0 = clock64();
    auto wait = [&](int s, uint32_t par) {
        uint32_t ok = 0;
        while (!ok) {
            asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p;}"
                         : "=r"(ok) : "r"(s32(&bars[s])), "r"(par));
        }
    };
    for (int i = 0; i < nloads; ++i) {
        const int stage = i % ns;
        if (i >= ns) wait(stage, ((i - ns) / ns) & 1);
        uint8_t *dst = smem + stage * ((bytes + 1023) / 1024 * 1024);
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(s32(&bars[stage])), "r"(bytes));
        int blk = (blockIdx.x * 131 + i * 7);
        if (MODE == 0) {
            int y = (blk % 64) * 128;
            asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];"
                         ::"r"(s32(dst)), "l"(&map), "r"(s32(&bars[stage])), "r"(0), "r"(y) : "memory");
        } else if (MODE == 1) {
            int n = blk % 8, h = (blk / 8) % (hmax - 4), w = 0;
            asm volatile("cp.async.bulk.tensor.4d.shared::cluster.global.im2col.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5, %6}], [%2], {%7, %8};"
                         ::"r"(s32(dst)), "l"(&map), "r"(s32(&bars[stage])), "r"(0), "r"(w), "r"(h), "r"(n), "h"((uint16_t)1), "h"((uint16_t)1) : "memory");
        } else {
            int n = blk % 8, h = (blk / 8) % (hmax - 8);
            asm volatile("cp.async.bulk.tensor.4d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5, %6}], [%2];"
                         ::"r"(s32(dst)), "l"(&map), "r"(s32(&bars[stage])), "r"(0), "r"(0), "r"(h), "r"(n) : "memory");
        }
    }
    for (int i = nloads - ns; i < nloads; ++i) wait(i % ns, (i / ns) & 1);
    if (wid == 0) out[blockIdx.x] = clock64() - t0;
}

typedef CUresult (*PFN_im2col)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *, const cuuint64_t *, const int *, const int *, cuuint32_t, cuuint32_t, const cuuint32_t *, CUtensorMapInterleave, CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
typedef CUresult (*PFN_tiled)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *, const cuuint64_t *, const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave, CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int main() {
    void *f1, *f2; cudaDriverEntryPointQueryResult q;
    cudaGetDriverEntryPoint("cuTensorMapEncodeIm2col", &f1, cudaEnableDefault, &q);
    cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f2, cudaEnableDefault, &q);
    PFN_im2col enc_i = (PFN_im2col)f1; PFN_tiled enc_t = (PFN_tiled)f2;
    const int N = 8, H = 64, W = 64, Cmax = 256;
    uint8_t *x; cudaMalloc(&x, (size_t)N * H * W * Cmax);
    cudaMemset(x, 1, (size_t)N * H * W * Cmax);
    long long *out; cudaMalloc(&out, 148 * sizeof(long long));
    int nloads = 2000, ns = 6;
    auto run = [&](auto kern, CUtensorMap &m, int bytes, const char *name, int nw) {
        cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 220 * 1024);
        int stage_b = (bytes + 1023) / 1024 * 1024;
        int smem = nw * ns * stage_b;
        if (smem > 220 * 1024) { printf("%-32s nw=%d ns=%d skip\n", name, nw, ns); return; }
        kern<<<148, 32 * nw, smem>>>(m, nloads, bytes, ns, W, H, out);
        cudaError_t e = cudaDeviceSynchronize();
        std::vector<long long> h(148); cudaMemcpy(h.data(), out, 148 * 8, cudaMemcpyDeviceToHost);
        double avg = 0; for (auto v : h) avg += v; avg /= 148;
        printf("%-32s nw=%d ns=%2d bytes/load %6d  cycles/load(per issuer) %7.1f  B/cyc/SM %6.1f  %s\n", name, nw, ns, bytes, avg / nloads, nw * (double)bytes * nloads / avg, e ? cudaGetErrorString(e) : "");
    };
    for (int nw : {1, 2, 4}) {
      ns = 4;
      for (int C : {32, 64, 128}) {
        int box = C;
        CUtensorMap m;
        cuuint64_t dims[4] = {(cuuint64_t)C, W, H, N}, str[3] = {(cuuint64_t)C, (cuuint64_t)C * W, (cuuint64_t)C * W * H};
        int lo[2] = {-1, -1}, up[2] = {-1, -1}; cuuint32_t es[4] = {1, 1, 1, 1};
        CUtensorMapSwizzle sw = box == 128 ? CU_TENSOR_MAP_SWIZZLE_128B : box == 64 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_32B;
        enc_i(&m, CU_TENSOR_MAP_DATA_TYPE_UINT8, 4, x, dims, str, lo, up, box, 128, es, CU_TENSOR_MAP_INTERLEAVE_NONE, sw, CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        char nm[64]; snprintf(nm, 64, "im2col 128px x %dB", box);
        run(bench<1>, m, 128 * box, nm, nw);
        cuuint64_t d2[2] = {(cuuint64_t)C, (cuuint64_t)N * H * W}, s2[1] = {(cuuint64_t)C};
        cuuint32_t bx[2] = {(cuuint32_t)box, 128}, e2[2] = {1, 1};
        enc_t(&m, CU_TENSOR_MAP_DATA_TYPE_UINT8, 2, x, d2, s2, bx, e2, CU_TENSOR_MAP_INTERLEAVE_NONE, sw, CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        snprintf(nm, 64, "tiled2d 128rows x %dB", box);
        run(bench<0>, m, 128 * box, nm, nw);
      }
    }
    return 0;
}
