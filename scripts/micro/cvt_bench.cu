// Microbenchmark: int4->int8 widening of one staged tile (widen_stage) by the 4 converter
// warps, in isolation (no TMA / MMA traffic).  Cycles per stage for the trans and im2col shapes.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include "../../paper_conf_icpp_hanhyylhgwwlq20_b200/csrc/conv_fwd.cuh"
using namespace qc;

__global__ void bench(int reps, int nchunks, int cshift, int bkb, int sw, long long *out) {
    extern __shared__ __align__(1024) uint8_t smem[];
    const uint32_t stg = smem_u32(smem), adst = smem_u32(smem + 32768);
    for (int i = threadIdx.x; i < 32768 / 4; i += blockDim.x) reinterpret_cast<uint32_t *>(smem)[i] = i * 2654435761u;
    __syncthreads();
    long long t0 = clock64();
    for (int r = 0; r < reps; ++r) {
        widen_stage(stg, adst, threadIdx.x, nchunks, cshift, static_cast<uint32_t>(bkb), static_cast<uint32_t>(sw), 0u);
        fence_proxy_async_smem();
        __syncthreads();
    }
    long long t1 = clock64();
    if (threadIdx.x == 0) out[blockIdx.x] = (t1 - t0) / reps;
}

int main() {
    long long *out; cudaMalloc(&out, 148 * sizeof(long long));
    cudaFuncSetAttribute(bench, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
    struct { const char *name; int nchunks, cshift, bkb, sw; } cases[] = {
        {"trans 256px x BK128", 1024, 2, 128, 7},
        {"im2col 128px x BK128", 512, 2, 128, 7},
        {"trans 256px x BK64", 512, 1, 64, 3},
    };
    for (auto &c : cases) {
        bench<<<148, kNumCvtWarps * 32, 100 * 1024>>>(200, c.nchunks, c.cshift, c.bkb, c.sw, out);
        bench<<<148, kNumCvtWarps * 32, 100 * 1024>>>(200, c.nchunks, c.cshift, c.bkb, c.sw, out);
        cudaError_t e = cudaDeviceSynchronize();
        if (e != cudaSuccess) { printf("err %s\n", cudaGetErrorString(e)); return 1; }
        long long h; cudaMemcpy(&h, out, 8, cudaMemcpyDeviceToHost);
        printf("%-24s cycles/stage=%lld  (%.2f cyc per 16B chunk per warp-slot)\n", c.name, h, (double)h / (c.nchunks / 128.0));
    }
    return 0;
}
