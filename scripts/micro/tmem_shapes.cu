// tcgen05.ld shapes on sm_100a: (1) which (lane, column) each thread gets for 16x64b / 16x128b,
// (2) read throughput per SM of 16x64b.x32, 16x128b.x16, 16x256b.x8, 32x32b.x32 (32 regs each).
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include "../../paper_conf_icpp_hanhyylhgwwlq20_b200/csrc/ptx.cuh"
using namespace qc;
#define R32 "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
#define O32(v) "=r"(v[0]),"=r"(v[1]),"=r"(v[2]),"=r"(v[3]),"=r"(v[4]),"=r"(v[5]),"=r"(v[6]),"=r"(v[7]),"=r"(v[8]),"=r"(v[9]),"=r"(v[10]),"=r"(v[11]),"=r"(v[12]),"=r"(v[13]),"=r"(v[14]),"=r"(v[15]),"=r"(v[16]),"=r"(v[17]),"=r"(v[18]),"=r"(v[19]),"=r"(v[20]),"=r"(v[21]),"=r"(v[22]),"=r"(v[23]),"=r"(v[24]),"=r"(v[25]),"=r"(v[26]),"=r"(v[27]),"=r"(v[28]),"=r"(v[29]),"=r"(v[30]),"=r"(v[31])
template <int S> __device__ __forceinline__ void ld32(uint32_t a, uint32_t (&v)[32]) {
    if (S == 0) asm volatile("tcgen05.ld.sync.aligned.32x32b.x32.b32 " R32 : O32(v) : "r"(a));
    if (S == 1) asm volatile("tcgen05.ld.sync.aligned.16x256b.x8.b32 " R32 : O32(v) : "r"(a));
    if (S == 2) asm volatile("tcgen05.ld.sync.aligned.16x128b.x16.b32 " R32 : O32(v) : "r"(a));
    if (S == 3) asm volatile("tcgen05.ld.sync.aligned.16x64b.x32.b32 " R32 : O32(v) : "r"(a));
}
template <int S>
__global__ void rd(int iters, long long *out, uint32_t *tags) {
    __shared__ uint32_t tslot;
    const int warp = threadIdx.x / 32, lane = threadIdx.x & 31;
    if (warp == 0) tmem_alloc(&tslot, 512);
    tc_fence_before(); __syncthreads(); tc_fence_after();
    // tag every cell: (lane << 16) | column
    if (warp < 4) {
        for (int c0 = 0; c0 < 512; c0 += 16) {
            uint32_t v[16];
            for (int c = 0; c < 16; ++c) v[c] = (static_cast<uint32_t>(warp * 32 + lane) << 16) | (c0 + c);
            const uint32_t tm = tslot + (static_cast<uint32_t>(warp * 32) << 16) + c0;
            asm volatile("tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};"
                         :: "r"(tm), "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7]),
                            "r"(v[8]), "r"(v[9]), "r"(v[10]), "r"(v[11]), "r"(v[12]), "r"(v[13]), "r"(v[14]), "r"(v[15]) : "memory");
        }
        asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
    }
    tc_fence_before(); __syncthreads(); tc_fence_after();
    const uint32_t tm = tslot + (static_cast<uint32_t>((warp & 3) * 32 + (S != 0 ? ((warp >> 2) & 1) * 16 : 0)) << 16);
    uint32_t v[32];
    if (blockIdx.x == 0 && warp == 0) {
        ld32<S>(tslot, v); asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
        for (int i = 0; i < 32; ++i) tags[lane * 32 + i] = v[i];
    }
    uint32_t acc = 0;
    __syncthreads();
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
        ld32<S>(tm + (((i + warp) * 32) & 255), v);
        tmem_wait_ld_regs(v);
        acc ^= v[0] ^ v[31];
    }
    __syncthreads();
    long long t1 = clock64();
    if (threadIdx.x == 0) out[blockIdx.x] = t1 - t0;
    if (acc == 0x9u) tags[4096] = acc;
    tc_fence_before(); __syncthreads();
    if (warp == 0) { tc_fence_after(); tmem_dealloc(tslot, 512); }
}
int main() {
    long long *out; cudaMalloc(&out, 148 * 8);
    uint32_t *tags; cudaMalloc(&tags, 8192 * 4);
    const char *nm[] = {"32x32b.x32", "16x256b.x8", "16x128b.x16", "16x64b.x32"};
    for (int s = 0; s < 4; ++s) {
        for (int warps : {4, 8, 16}) {
            const int iters = 4096;
            for (int rep = 0; rep < 2; ++rep) {
                if (s == 0) rd<0><<<148, warps * 32>>>(iters, out, tags);
                if (s == 1) rd<1><<<148, warps * 32>>>(iters, out, tags);
                if (s == 2) rd<2><<<148, warps * 32>>>(iters, out, tags);
                if (s == 3) rd<3><<<148, warps * 32>>>(iters, out, tags);
            }
            cudaError_t e = cudaDeviceSynchronize();
            if (e != cudaSuccess) { printf("err %s\n", cudaGetErrorString(e)); return 1; }
            long long h; cudaMemcpy(&h, out, 8, cudaMemcpyDeviceToHost);
            printf("%-12s warps=%2d  accumulators/cycle/SM = %.1f\n", nm[s], warps, (double)warps * iters * 1024 / h);
        }
        uint32_t t[1024]; cudaMemcpy(t, tags, 4096, cudaMemcpyDeviceToHost);
        for (int th : {0, 1, 2, 3, 4, 5}) {
            printf("  %s thread %d:", nm[s], th);
            for (int i = 0; i < 8; ++i) printf(" (l%u,c%u)", t[th * 32 + i] >> 16, t[th * 32 + i] & 0xffff);
            printf("\n");
        }
    }
    return 0;
}
