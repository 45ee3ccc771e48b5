// Microbenchmarks: (1) tcgen05.ld 32x32b read bandwidth of TMEM per SM versus the number of
// reading warps; (2) legacy mma.sync m16n8k32 s8 (IMMA) throughput on sm_100a.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include "../../paper_conf_icpp_hanhyylhgwwlq20_b200/csrc/ptx.cuh"
using namespace qc;

// every warp reads `iters` x (32 lanes x 32 columns x 4 B) from its lane quarter
template <int BATCH>
__global__ void tmem_read(int iters, long long *out, unsigned *sink) {
    __shared__ uint32_t tslot;
    const int warp = threadIdx.x / 32;
    if (warp == 0) tmem_alloc(&tslot, 512);
    tc_fence_before(); __syncthreads(); tc_fence_after();
    const uint32_t tm = tslot + (static_cast<uint32_t>((warp & 3) * 32) << 16);
    uint32_t acc = 0;
    __syncthreads();
    long long t0 = clock64();
    for (int i = 0; i < iters; i += BATCH) {
        uint32_t v[BATCH][32];
#pragma unroll
        for (int b = 0; b < BATCH; ++b) tmem_ld_32x32b_x32(tm + (((i + b + warp) * 32) & 511), v[b]);
        tmem_wait_ld();
#pragma unroll
        for (int b = 0; b < BATCH; ++b)
#pragma unroll
            for (int j = 0; j < 32; ++j) acc += v[b][j];
    }
    __syncthreads();
    long long t1 = clock64();
    if (threadIdx.x == 0) out[blockIdx.x] = t1 - t0;
    if (acc == 0x9u) sink[0] = acc;
    tc_fence_before(); __syncthreads();
    if (warp == 0) { tc_fence_after(); tmem_dealloc(tslot, 512); }
}


__device__ __forceinline__ void tmem_ld_32x32b_x32_p16(uint32_t taddr, uint32_t (&v)[16]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.pack::16b.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, "
        "%11, %12, %13, %14, %15}, [%16];"
        : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
          "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15])
        : "r"(taddr));
}
// SHAPE 0: 32x32b.x32 (32 cols), 1: 16x256b.x8 (16 lanes x 64 cols... 32 regs), 2: 32x32b.x16.pack::16b (32 cols -> 16 regs)
template <int SHAPE>
__global__ void tmem_read2(int iters, long long *out, unsigned *sink) {
    __shared__ uint32_t tslot;
    const int warp = threadIdx.x / 32;
    if (warp == 0) tmem_alloc(&tslot, 512);
    tc_fence_before(); __syncthreads(); tc_fence_after();
    const uint32_t tm = tslot + (static_cast<uint32_t>((warp & 3) * 32 + (SHAPE == 1 ? ((warp >> 2) & 1) * 16 : 0)) << 16);
    uint32_t acc = 0;
    __syncthreads();
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
        uint32_t v[32];
        if (SHAPE == 0) tmem_ld_32x32b_x32(tm + (((i + warp) * 32) & 511), v);
        else if (SHAPE == 1) tmem_ld_16x256b_x8(tm + (((i + warp) * 64) & 511), v);
        else { uint32_t u[16]; tmem_ld_32x32b_x32_p16(tm + (((i + warp) * 32) & 511), u);
#pragma unroll
               for (int j = 0; j < 16; ++j) v[j] = u[j], v[j + 16] = 0; }
        tmem_wait_ld();
#pragma unroll
        for (int j = 0; j < 32; ++j) acc += v[j];
    }
    __syncthreads();
    long long t1 = clock64();
    if (threadIdx.x == 0) out[blockIdx.x] = t1 - t0;
    if (acc == 0x9u) sink[0] = acc;
    tc_fence_before(); __syncthreads();
    if (warp == 0) { tc_fence_after(); tmem_dealloc(tslot, 512); }
}

template <int SHAPE>
__global__ void tmem_read3(int iters, long long *out, unsigned *sink) {
    __shared__ uint32_t tslot;
    const int warp = threadIdx.x / 32;
    if (warp == 0) tmem_alloc(&tslot, 512);
    tc_fence_before(); __syncthreads(); tc_fence_after();
    const uint32_t tm = tslot + (static_cast<uint32_t>((warp & 3) * 32 + (SHAPE == 1 ? ((warp >> 2) & 1) * 16 : 0)) << 16);
    uint32_t acc = 0;
    __syncthreads();
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
        uint32_t v[32];
        if (SHAPE == 0) tmem_ld_32x32b_x32(tm + (((i + warp) * 32) & 511), v);
        else tmem_ld_16x256b_x8(tm + (((i + warp) * 64) & 511), v);
        tmem_wait_ld_regs(v);
        acc ^= v[0] ^ v[31];
    }
    __syncthreads();
    long long t1 = clock64();
    if (threadIdx.x == 0) out[blockIdx.x] = t1 - t0;
    if (acc == 0x9u) sink[0] = acc;
    tc_fence_before(); __syncthreads();
    if (warp == 0) { tc_fence_after(); tmem_dealloc(tslot, 512); }
}

__global__ void imma(int iters, long long *out, int *sink) {
    int a0 = threadIdx.x * 3 + 1, a1 = a0 ^ 0x55, a2 = a0 * 7, a3 = a0 + 9;
    int b0 = threadIdx.x + 5, b1 = b0 * 3;
    int d[8][4] = {};
    __syncthreads();
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int k = 0; k < 8; ++k)
            asm volatile("mma.sync.aligned.m16n8k32.row.col.s32.s8.s8.s32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};"
                         : "+r"(d[k][0]), "+r"(d[k][1]), "+r"(d[k][2]), "+r"(d[k][3])
                         : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1));
    }
    __syncthreads();
    long long t1 = clock64();
    if (threadIdx.x == 0) out[blockIdx.x] = t1 - t0;
    int s = 0;
    for (int k = 0; k < 8; ++k) s += d[k][0] + d[k][1] + d[k][2] + d[k][3];
    if (s == 0x12345) sink[0] = s;
}

int main() {
    long long *out; cudaMalloc(&out, 148 * sizeof(long long));
    unsigned *sink; cudaMalloc(&sink, 64);
    long long h[148];
    int clk_khz = 0; cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0);
    for (int warps : {4, 8, 12, 16}) {
        for (int batch : {1, 2}) {
            const int iters = 4096;
            for (int rep = 0; rep < 2; ++rep) {
                if (batch == 1) tmem_read<1><<<148, warps * 32>>>(iters, out, sink);
                else tmem_read<2><<<148, warps * 32>>>(iters, out, sink);
            }
            cudaError_t e = cudaDeviceSynchronize();
            if (e != cudaSuccess) { printf("err %s\n", cudaGetErrorString(e)); return 1; }
            cudaMemcpy(h, out, sizeof(h), cudaMemcpyDeviceToHost);
            const double bytes = static_cast<double>(warps) * iters * 32 * 32 * 4;
            printf("tmem_read warps=%2d batch=%d  cycles=%lld  B/cyc/SM=%.1f\n", warps, batch, h[0],
                   bytes / h[0]);
        }
    }

    for (int shape : {0, 1, 2}) for (int warps : {4, 8, 16}) {
        const int iters = 4096;
        for (int rep = 0; rep < 2; ++rep) {
            if (shape == 0) tmem_read2<0><<<148, warps * 32>>>(iters, out, sink);
            else if (shape == 1) tmem_read2<1><<<148, warps * 32>>>(iters, out, sink);
            else tmem_read2<2><<<148, warps * 32>>>(iters, out, sink);
        }
        cudaError_t e = cudaDeviceSynchronize();
        if (e != cudaSuccess) { printf("err %s\n", cudaGetErrorString(e)); return 1; }
        cudaMemcpy(h, out, sizeof(h), cudaMemcpyDeviceToHost);
        const double bytes = static_cast<double>(warps) * iters * 32 * 32 * 4;   // accumulator bytes covered
        printf("tmem_read2 shape=%d warps=%2d cycles=%lld  acc-B/cyc/SM=%.1f  (32-bit accumulators/cyc/SM=%.1f)\n", shape, warps, h[0], bytes / h[0], bytes / 4 / h[0]);
    }
    for (int warps : {4, 8, 16, 32}) {
        const int iters = 2048;
        for (int rep = 0; rep < 2; ++rep) imma<<<148, warps * 32>>>(iters, out, reinterpret_cast<int *>(sink));
        cudaError_t e = cudaDeviceSynchronize();
        if (e != cudaSuccess) { printf("err %s\n", cudaGetErrorString(e)); return 1; }
        cudaMemcpy(h, out, sizeof(h), cudaMemcpyDeviceToHost);
        const double macs = static_cast<double>(warps) * iters * 8 * 16 * 8 * 32;
        printf("imma m16n8k32 warps=%2d cycles=%lld  MAC/cyc/SM=%.0f  (x148 SMs x %.2f GHz = %.0f TOPS)\n",
               warps, h[0], macs / h[0], clk_khz / 1e6, 2 * macs / h[0] * 148 * clk_khz * 1e3 / 1e12);
    }

    for (int shape : {0, 1}) for (int warps : {4, 8, 16}) {
        const int iters = 4096;
        for (int rep = 0; rep < 2; ++rep) {
            if (shape == 0) tmem_read3<0><<<148, warps * 32>>>(iters, out, sink);
            else tmem_read3<1><<<148, warps * 32>>>(iters, out, sink);
        }
        cudaDeviceSynchronize();
        cudaMemcpy(h, out, sizeof(h), cudaMemcpyDeviceToHost);
        const double accs = static_cast<double>(warps) * iters * 32 * 32;
        printf("tmem_read3 (no ALU) shape=%d warps=%2d cycles=%lld  accumulators/cyc/SM=%.1f\n", shape, warps, h[0], accs / h[0]);
    }
    return 0;
}
