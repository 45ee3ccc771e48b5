// Learn the register layout of tcgen05.ld.16x256b: write lane/column tags with 32x32b stores,
// read back with 16x256b.x2 at lane offsets 0 and 16, print what each thread of warp 0 got.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include "../../paper_conf_icpp_hanhyylhgwwlq20_b200/csrc/ptx.cuh"
using namespace qc;

__global__ void k(uint32_t *out) {
    __shared__ uint32_t tslot;
    const int warp = threadIdx.x / 32, lane = threadIdx.x & 31;
    if (warp == 0) tmem_alloc(&tslot, 32);
    tc_fence_before(); __syncthreads(); tc_fence_after();
    const uint32_t tm = tslot + (static_cast<uint32_t>(warp * 32) << 16);
    uint32_t v[16];
    for (int c = 0; c < 16; ++c) v[c] = (static_cast<uint32_t>(warp * 32 + lane) << 16) | c;
    asm volatile("tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};"
                 :: "r"(tm), "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7]),
                    "r"(v[8]), "r"(v[9]), "r"(v[10]), "r"(v[11]), "r"(v[12]), "r"(v[13]), "r"(v[14]), "r"(v[15]) : "memory");
    asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
    tc_fence_before(); __syncthreads(); tc_fence_after();
    if (warp == 1) {
        uint32_t r[8];
        const uint32_t ta = tslot + (static_cast<uint32_t>(32 + 16) << 16);   // quarter 1, lanes 16..31
        asm volatile("tcgen05.ld.sync.aligned.16x256b.x2.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                     : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7])
                     : "r"(ta));
        asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
        for (int i = 0; i < 8; ++i) out[lane * 8 + i] = r[i];
    }
    tc_fence_before(); __syncthreads();
    if (warp == 0) { tc_fence_after(); tmem_dealloc(tslot, 32); }
}

int main() {
    uint32_t *d; cudaMalloc(&d, 32 * 8 * 4);
    k<<<1, 128>>>(d);
    cudaError_t e = cudaDeviceSynchronize();
    if (e) { printf("err %s\n", cudaGetErrorString(e)); return 1; }
    uint32_t h[256]; cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    for (int t = 0; t < 32; ++t) {
        printf("t%2d:", t);
        for (int i = 0; i < 8; ++i) printf(" (l%u,c%u)", h[t * 8 + i] >> 16, h[t * 8 + i] & 0xFFFF);
        printf("\n");
    }
    return 0;
}
