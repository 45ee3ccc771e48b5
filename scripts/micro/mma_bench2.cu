// Microbenchmark: tcgen05.mma.kind::i8 throughput vs shape (M, N) and the number of distinct
// accumulators the MMAs rotate through (is the ~75-cycle floor of small-N MMAs a per-
// accumulator dependency or a per-instruction cost?).  One CTA per SM, lane 0 issues.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <vector>
#include "../../paper_conf_icpp_hanhyylhgwwlq20_b200/csrc/ptx.cuh"
using namespace qc;

__global__ void bench(int n_mma, int M, int N, int nacc, int accum, long long *out) {
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ uint32_t tslot;
    __shared__ __align__(8) uint64_t bar;
    const int warp = threadIdx.x / 32, lane = threadIdx.x & 31;
    for (int i = threadIdx.x; i < 64 * 1024; i += blockDim.x) smem[i] = (uint8_t)(i * 7);
    if (threadIdx.x == 0) { mbar_init(&bar, 1); fence_mbar_init(); }
    fence_proxy_async_smem();
    if (warp == 0) tmem_alloc(&tslot, 512);
    tc_fence_before(); __syncthreads(); tc_fence_after();
    const uint32_t tm = tslot;
    const uint32_t idesc = make_idesc_i8(M, N, false, true);
    const uint32_t a = smem_u32(smem), b = smem_u32(smem + 32768);
    long long t0 = clock64(), t1 = 0;
    if (warp == 0) {
        if (lane == 0) {
            const uint64_t ad = make_smem_desc(a, 2048, 128, 0);
            const uint64_t bd = make_smem_desc(b, 4096, 128, 0);
            for (int i = 0; i < n_mma; ++i) {
                const uint32_t d = tm + static_cast<uint32_t>((i % nacc) * N);
                mma_i8(d, ad + (i & 7) * 2, bd, idesc, (accum && i >= nacc) ? 1u : 0u);
            }
            mma_commit(&bar);
        }
        t1 = clock64();
        mbar_wait(&bar, 0);
        if (lane == 0) { out[blockIdx.x * 2] = t1 - t0; out[blockIdx.x * 2 + 1] = clock64() - t0; }
    }
    tc_fence_before(); __syncthreads();
    if (warp == 0) { tc_fence_after(); tmem_dealloc(tm, 512); }
}

int main() {
    long long *out; cudaMalloc(&out, 148 * 2 * sizeof(long long));
    struct Cfg { int M, N, nacc, accum; };
    std::vector<Cfg> cfgs = {{128, 64, 1, 1}, {128, 64, 2, 1}, {128, 64, 4, 1}, {128, 64, 1, 0},
                             {128, 128, 1, 1}, {128, 128, 2, 1}, {128, 128, 1, 0}, {128, 256, 1, 1},
                             {128, 256, 2, 1}, {64, 256, 1, 1}, {64, 256, 2, 1}, {64, 128, 1, 1},
                             {128, 192, 1, 1}, {128, 96, 1, 1}, {128, 32, 1, 1}};
    cudaFuncSetAttribute(bench, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
    for (auto c : cfgs) {
        int n = 4000;
        bench<<<148, 128, 96 * 1024>>>(n, c.M, c.N, c.nacc, c.accum, out);
        cudaError_t e = cudaDeviceSynchronize();
        std::vector<long long> h(296); cudaMemcpy(h.data(), out, 296 * 8, cudaMemcpyDeviceToHost);
        double is = 0, ex = 0; for (int i = 0; i < 148; ++i) { is += h[2*i]; ex += h[2*i+1]; }
        is /= 148; ex /= 148;
        const double macs = 1.0 * c.M * c.N * 32;
        printf("M=%3d N=%3d nacc=%d accum=%d  cycles/mma %7.1f  MAC/cyc/SM %6.0f  (peak 8192)  %s\n", c.M, c.N,
               c.nacc, c.accum, ex / n, macs / (ex / n), e ? cudaGetErrorString(e) : "");
    }
    return 0;
}
