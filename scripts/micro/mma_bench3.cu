// Microbenchmark: what paces the halo kernels' M128 x N64 x K32 int8 MMAs?  Back-to-back
// tcgen05.mma.kind::i8 from one warp per CTA (warp-uniform loop, elected issue) (one CTA per SM), operand layouts as the
// kernels use them:
//   plane   : no-swizzle K-major, A as separate 16-byte channel planes (LBO = plane stride),
//             start addresses 16-byte aligned and varying per MMA (the halo tap offsets)
//   pair    : no-swizzle, LBO = 16 (the stem's tap pair: K half 1 = next pixel)
//   aligned : no-swizzle, every start 1024-byte aligned
//   sw128   : 128-byte swizzle K-major (a plain GEMM tile), start advanced 32 B per K step
//   ts      : A from TMEM, B no-swizzle
// and N = 64 / 128 / 256; one accumulator (dependent chain) or two alternating.
// Usage: nvcc -gencode arch=compute_100a,code=sm_100a -I ... mma_bench3.cu && ./a.out
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <vector>
#include "../../paper_conf_icpp_hanhyylhgwwlq20_b200/csrc/ptx.cuh"
using namespace qc;

__device__ __forceinline__ void mma_ts(uint32_t d, uint32_t a, uint64_t bd, uint32_t idesc, uint32_t acc) {
    asm volatile(
        "{\n\t.reg .pred p, e;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "elect.sync _|e, 0xffffffff;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %3, p;\n\t}" ::"r"(d),
        "r"(a), "l"(bd), "r"(idesc), "r"(acc)
        : "memory");
}

template <int MODE, int N>
__global__ void bench(int n_iter, int nacc, long long *out) {
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    __shared__ uint32_t tslot;
    __shared__ __align__(8) uint64_t bar;
    const int warp = threadIdx.x / 32, lane = threadIdx.x & 31;
    for (int i = threadIdx.x; i < 160 * 1024; i += blockDim.x) smem[i] = (uint8_t)(i * 7);
    if (threadIdx.x == 0) { mbar_init(&bar, 1); fence_mbar_init(); }
    fence_proxy_async_smem();
    if (warp == 0) tmem_alloc(&tslot, 512);
    tc_fence_before(); __syncthreads(); tc_fence_after();
    const uint32_t tm = tslot;
    const uint32_t idesc = make_idesc_i8(128, N, false, true);
    const uint32_t a = smem_u32(smem), b = smem_u32(smem + 96 * 1024);
    long long t0 = clock64(), t1 = 0;
    if (warp == 0) {   // the whole warp runs the (uniform) loop, one elected lane issues
        const uint64_t bd = MODE == 3 ? make_smem_desc(b, 16, 1024, 2) : make_smem_desc(b, N * 16u, 128, 0);
        uint64_t ad;
        if (MODE == 0) ad = make_smem_desc(a, 58 * 8 * 16, 128, 0);
        else if (MODE == 1) ad = make_smem_desc(a, 16, 128, 0);
        else if (MODE == 2) ad = make_smem_desc(a, 2048, 128, 0);
        else ad = make_smem_desc(a, 16, 1024, 2);
        for (int it = 0; it < n_iter; ++it) {
            const uint32_t d = tm + static_cast<uint32_t>(((it % nacc) * N));
#pragma unroll
            for (int k = 0; k < 8; ++k) {
                // descriptor offsets in 16-byte units (compile-time per k)
                const uint32_t ao = MODE == 0 ? (k / 3) * 58 + k % 3
                                  : MODE == 1 ? (k >> 1) * 115 + 2 * (k & 1)
                                  : MODE == 2 ? 256 * k
                                  : 2 * (k & 3) + 1024 * (k >> 2);
                const uint32_t bo = MODE == 3 ? 2 * (k & 3) + 1024 * (k >> 2) : 0;
                const uint32_t acc = (it > 0 || k > 0) ? 1u : 0u;
                if (MODE == 4) mma_ts(d, tm + 256u + 8u * k, bd + bo, idesc, acc);
                else mma_i8_warp(d, ad + ao, bd + bo, idesc, acc);
            }
        }
        mma_commit_warp(&bar);
        t1 = clock64();
    }
    if (warp == 0) {
        mbar_wait(&bar, 0);
        if (lane == 0) { out[blockIdx.x * 2] = t1 - t0; out[blockIdx.x * 2 + 1] = clock64() - t0; }
    }
    tc_fence_before(); __syncthreads();
    if (warp == 0) { tc_fence_after(); tmem_dealloc(tm, 512); }
}

long long *g_out;
template <int MODE, int N>
void run(const char *name, int nacc) {
    cudaFuncSetAttribute(bench<MODE, N>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    const int n_iter = 500;
    bench<MODE, N><<<148, 128, 200 * 1024>>>(n_iter, nacc, g_out);
    cudaError_t e = cudaDeviceSynchronize();
    std::vector<long long> h(296);
    cudaMemcpy(h.data(), g_out, 296 * 8, cudaMemcpyDeviceToHost);
    double is = 0, ex = 0;
    for (int i = 0; i < 148; ++i) { is += h[2 * i]; ex += h[2 * i + 1]; }
    is /= 148; ex /= 148;
    const double n = 8.0 * n_iter;
    printf("%-8s N=%3d nacc=%d  issue %6.1f  cycles/mma %7.1f  MAC/cyc/SM %6.0f  %s\n", name, N, nacc, is / n, ex / n,
           128.0 * N * 32 / (ex / n), e ? cudaGetErrorString(e) : "");
}

int main() {
    cudaMalloc(&g_out, 148 * 2 * sizeof(long long));
    for (int nacc : {1, 2}) {
        run<0, 64>("plane", nacc); run<0, 128>("plane", nacc); run<0, 256>("plane", nacc);
        run<1, 64>("pair", nacc); run<1, 128>("pair", nacc); run<1, 256>("pair", nacc);
        run<2, 64>("aligned", nacc); run<2, 128>("aligned", nacc); run<2, 256>("aligned", nacc);
        run<3, 64>("sw128", nacc); run<3, 128>("sw128", nacc); run<3, 256>("sw128", nacc);
        run<4, 64>("ts", nacc); run<4, 128>("ts", nacc);
    }
    return 0;
}
