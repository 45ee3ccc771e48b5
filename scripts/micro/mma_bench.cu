// Microbenchmark: tcgen05.mma.kind::i8 issue/execution rate for one CTA per SM.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <vector>
#include "../../paper_conf_icpp_hanhyylhgwwlq20_b200/csrc/ptx.cuh"
using namespace qc;

template <int MODE>   // 0: lane 0 issues inside if(lane==0); 1: uniform loop, elect
__global__ void bench(int n_mma, int N, int layout, int pre, long long *out) {
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ uint32_t tslot;
    __shared__ __align__(8) uint64_t bar;
    const int warp = threadIdx.x / 32, lane = threadIdx.x & 31;
    for (int i = threadIdx.x; i < 64 * 1024; i += blockDim.x) smem[i] = (uint8_t)(i * 7);
    if (threadIdx.x == 0) { mbar_init(&bar, 1); fence_mbar_init(); }
    fence_proxy_async_smem();
    if (warp == 0) tmem_alloc(&tslot, 256);
    tc_fence_before(); __syncthreads(); tc_fence_after();
    const uint32_t tm = tslot;
    const uint32_t idesc = make_idesc_i8(128, N, false, true);
    const uint32_t a = smem_u32(smem), b = smem_u32(smem + 32768);
    long long t0 = clock64(), t1 = 0;
    if (warp == 0) {
        if (MODE == 0) {
            if (lane == 0) {
                for (int i = 0; i < n_mma; ++i) {
                    uint32_t ao = pre ? 0u : (uint32_t)(i & 7) * 32u;
                    uint64_t ad = layout ? make_smem_desc(a + ao, 16, 1024, 2) : make_smem_desc(a + ao, 2048, 128, 0);
                    uint64_t bd = layout ? make_smem_desc(b, 16, 1024, 2) : make_smem_desc(b, 2048, 128, 0);
                    mma_i8(tm, ad, bd, idesc, i > 0);
                }
                mma_commit(&bar);
            }
        } else {
            const uint64_t ad0 = layout ? make_smem_desc(a, 16, 1024, 2) : make_smem_desc(a, 2048, 128, 0);
            const uint64_t bd = layout ? make_smem_desc(b, 16, 1024, 2) : make_smem_desc(b, 2048, 128, 0);
            for (int i = 0; i < n_mma; ++i) {
                uint64_t ad = ad0 + (pre ? 0 : (uint64_t)((i & 7) * 2));
                if (elect_one()) mma_i8(tm, ad, bd, idesc, i > 0);
                __syncwarp();
            }
            if (elect_one()) mma_commit(&bar);
            __syncwarp();
        }
        t1 = clock64();
        mbar_wait(&bar, 0);
        if (lane == 0) { out[blockIdx.x * 2] = t1 - t0; out[blockIdx.x * 2 + 1] = clock64() - t0; }
    }
    tc_fence_before(); __syncthreads();
    if (warp == 0) { tc_fence_after(); tmem_dealloc(tm, 256); }
}

int main() {
    long long *out; cudaMalloc(&out, 148 * 2 * sizeof(long long));
    for (int mode = 0; mode < 2; ++mode)
    for (int layout = 0; layout < 2; ++layout)
    for (int N : {64, 128, 256}) {
        int n = 2000;
        auto k = mode == 0 ? bench<0> : bench<1>;
        cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
        k<<<148, 128, 96 * 1024>>>(n, N, layout, 0, out);
        cudaError_t e = cudaDeviceSynchronize();
        std::vector<long long> h(296); cudaMemcpy(h.data(), out, 296 * 8, cudaMemcpyDeviceToHost);
        double is = 0, ex = 0; for (int i = 0; i < 148; ++i) { is += h[2*i]; ex += h[2*i+1]; }
        is /= 148; ex /= 148;
        printf("mode=%d layout=%s N=%3d  issue cycles/mma %7.1f  total cycles/mma %7.1f  (ideal %d)  %s\n", mode, layout ? "sw128" : "none ", N, is / n, ex / n, 128 * N / 256, e ? cudaGetErrorString(e) : "");
    }
    return 0;
}
