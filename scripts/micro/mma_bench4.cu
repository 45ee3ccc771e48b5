// Microbenchmark: does other warps' shared-memory or TMEM traffic slow the tensor pipe?  Warp 0
// issues back-to-back M128 x N64 x K32 int8 MMAs (shared-memory A/B, the stem's tap-pair
// layout) while warps 4..11 run a load loop: none, broadcast LDS.128 (the epilogue's column
// constants), strided LDS.32 (the fused stem's fp32 reads), LDTM.x32 (accumulator reads), or
// STS.128.  Prints cycles per MMA.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <vector>
#include "../../paper_conf_icpp_hanhyylhgwwlq20_b200/csrc/ptx.cuh"
using namespace qc;

template <int LOAD>
__global__ void bench(int n_iter, long long *out, int *sink) {
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    __shared__ uint32_t tslot;
    __shared__ __align__(8) uint64_t bar;
    __shared__ volatile int stop;
    const int warp = threadIdx.x / 32, lane = threadIdx.x & 31;
    for (int i = threadIdx.x; i < 160 * 1024; i += blockDim.x) smem[i] = (uint8_t)(i * 7);
    if (threadIdx.x == 0) { mbar_init(&bar, 1); fence_mbar_init(); stop = 0; }
    fence_proxy_async_smem();
    if (warp == 0) tmem_alloc(&tslot, 512);
    tc_fence_before(); __syncthreads(); tc_fence_after();
    const uint32_t tm = tslot;
    const uint32_t idesc = make_idesc_i8(128, 64, false, true);
    const uint32_t a = smem_u32(smem), b = smem_u32(smem + 96 * 1024);
    if (warp == 0) {
        const long long t0 = clock64();
        const uint64_t bd = make_smem_desc(b, 64 * 16u, 128, 0);
        const uint64_t ad = make_smem_desc(a, 16, 128, 0);
        for (int it = 0; it < n_iter; ++it) {
            const uint32_t d = tm + static_cast<uint32_t>((it & 1) * 64);
#pragma unroll
            for (int k = 0; k < 8; ++k)
                mma_i8_warp(d, ad + (k >> 1) * 115 + 2 * (k & 1), bd + k * 128, idesc, k > 0 ? 1u : 0u);
        }
        mma_commit_warp(&bar);
        mbar_wait(&bar, 0);
        if (lane == 0) { out[blockIdx.x] = clock64() - t0; stop = 1; }
    } else if (warp >= 4 && warp < 12 && LOAD > 0) {
        uint32_t acc = 0;
        const uint32_t base = smem_u32(smem + 64 * 1024);
        int i = 0;
        while (!stop) {
#pragma unroll 4
            for (int u = 0; u < 64; ++u, ++i) {
                if (LOAD == 1) {
                    const uint4 v = lds128u(base + 16u * (i & 63));
                    acc += v.x ^ v.y ^ v.z ^ v.w;
                } else if (LOAD == 2) {
                    uint32_t v;
                    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(base + 24u * lane + 4u * (i & 7)));
                    acc += v;
                } else if (LOAD == 3) {
                    uint32_t v[32];
                    tmem_ld_32x32b_x32(tm + (static_cast<uint32_t>((warp & 3) * 32) << 16) + 256u + 32u * (warp >> 3), v);
                    tmem_wait_ld();
                    acc += v[0] ^ v[31];
                } else {
                    sts128(base + 16u * ((i * 32 + lane) & 2047), acc, i, lane, warp);
                }
            }
        }
        if (acc == 0x12345678u) sink[0] = acc;
    }
    tc_fence_before(); __syncthreads();
    if (warp == 0) { tc_fence_after(); tmem_dealloc(tm, 512); }
}

long long *g_out;
int *g_sink;
template <int LOAD>
void run(const char *name) {
    cudaFuncSetAttribute(bench<LOAD>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    const int n_iter = 500;
    bench<LOAD><<<148, 384, 200 * 1024>>>(n_iter, g_out, g_sink);
    cudaError_t e = cudaDeviceSynchronize();
    std::vector<long long> h(148);
    cudaMemcpy(h.data(), g_out, 148 * 8, cudaMemcpyDeviceToHost);
    double ex = 0;
    for (int i = 0; i < 148; ++i) ex += h[i];
    ex /= 148;
    printf("%-12s cycles/mma %7.1f  %s\n", name, ex / (8.0 * n_iter), e ? cudaGetErrorString(e) : "");
}

int main() {
    cudaMalloc(&g_out, 148 * sizeof(long long));
    cudaMalloc(&g_sink, 4);
    run<0>("none"); run<1>("lds128_bc"); run<2>("lds32_str"); run<3>("ldtm_x32"); run<4>("sts128");
    return 0;
}
