// Microbenchmark: cost of tcgen05.commit (mbarrier arrive on MMA completion) inside an MMA
// issue loop: M=128 N=256 K=32 i8 MMAs, a commit every `every` MMAs (0 = only at the end).
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <vector>
#include "../../paper_conf_icpp_hanhyylhgwwlq20_b200/csrc/ptx.cuh"
using namespace qc;

__global__ void bench(int n_mma, int N, int every, int warpwide, long long *out) {
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ uint32_t tslot;
    __shared__ __align__(8) uint64_t bar[2];
    const int warp = threadIdx.x / 32, lane = threadIdx.x & 31;
    for (int i = threadIdx.x; i < 64 * 1024; i += blockDim.x) smem[i] = (uint8_t)(i * 7);
    if (threadIdx.x == 0) { mbar_init(&bar[0], 1); mbar_init(&bar[1], 1); fence_mbar_init(); }
    fence_proxy_async_smem();
    if (warp == 0) tmem_alloc(&tslot, 256);
    tc_fence_before(); __syncthreads(); tc_fence_after();
    const uint32_t tm = tslot;
    const uint32_t idesc = make_idesc_i8(128, N, false, true);
    const uint32_t a = smem_u32(smem), b = smem_u32(smem + 32768);
    long long t0 = clock64(), t1 = 0;
    if (warp == 0) {
        const uint64_t ad = make_smem_desc(a, 2048, 128, 0);
        const uint64_t bd = make_smem_desc(b, 4096, 128, 0);
        if (warpwide) {
            int c = 0;
            for (int i = 0; i < n_mma; ++i) {
                mma_i8_warp(tm, ad + (i & 7) * 2, bd, idesc, i > 0 ? 1u : 0u);
                if (++c == every) { c = 0; mma_commit_warp(&bar[1]); }
            }
            mma_commit_warp(&bar[0]);
        } else if (lane == 0) {
            int c = 0;
            for (int i = 0; i < n_mma; ++i) {
                mma_i8(tm, ad + (i & 7) * 2, bd, idesc, i > 0 ? 1u : 0u);
                if (++c == every) { c = 0; mma_commit(&bar[1]); }
            }
            mma_commit(&bar[0]);
        }
        __syncwarp();
        t1 = clock64();
        mbar_wait(&bar[0], 0);
        if (lane == 0) { out[blockIdx.x * 2] = t1 - t0; out[blockIdx.x * 2 + 1] = clock64() - t0; }
    }
    tc_fence_before(); __syncthreads();
    if (warp == 0) { tc_fence_after(); tmem_dealloc(tm, 256); }
}

int main() {
    long long *out; cudaMalloc(&out, 148 * 2 * sizeof(long long));
    cudaFuncSetAttribute(bench, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
    for (int ww = 0; ww < 2; ++ww)
    for (int N : {64, 256})
    for (int every : {0, 1, 2, 4, 8}) {
        int n = 4000;
        bench<<<148, 128, 96 * 1024>>>(n, N, every, ww, out);
        cudaError_t e = cudaDeviceSynchronize();
        std::vector<long long> h(296); cudaMemcpy(h.data(), out, 296 * 8, cudaMemcpyDeviceToHost);
        double is = 0, ex = 0; for (int i = 0; i < 148; ++i) { is += h[2*i]; ex += h[2*i+1]; }
        is /= 148; ex /= 148;
        printf("warpwide=%d N=%3d commit every %d: issue cycles/mma %7.1f total cycles/mma %7.1f %s\n", ww, N, every,
               is / n, ex / n, e ? cudaGetErrorString(e) : "");
    }
    return 0;
}
