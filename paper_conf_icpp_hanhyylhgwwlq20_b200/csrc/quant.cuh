// quant.cuh -- the quantization step of the QNN layer sequence, reading Z4:
// q = clamp(rne(x * fl32(1/s)) + z, qmin, qmax), NaN -> z.  Shared by the quantize kernels
// (prep.cuh) and the fused-quantization stem (halo.cuh).
#pragma once
#include <cstdint>
#include <cuda_bf16.h>

namespace qc {

struct QuantParams {
    const void *x;
    void *y;
    int64_t npix;
    int32_t c, c_pad;
    float inv_s;        // fl32(1/scale), computed on the host in fp32
    float flo, fhi;     // qmin - z - 1, qmax - z + 1 (pre-clamp keeps the int conversion exact)
    int32_t z, qmin, qmax;
    int32_t bf16, bits;
    int32_t fast;       // c == c_pad, c % 16 == 0, 16-byte aligned rows
};

__device__ __forceinline__ int32_t quantize_one(float x, const QuantParams &p) {
    float t = __fmul_rn(x, p.inv_s);                 // one IEEE fp32 multiply, RNE
    if (isnan(t)) return p.z;
    t = fminf(fmaxf(t, p.flo), p.fhi);
    const int32_t q = __float2int_rn(t) + p.z;       // round half to even
    return min(p.qmax, max(p.qmin, q));
}

__device__ __forceinline__ float load_x(const QuantParams &p, int64_t i) {
    if (p.bf16) {
        const uint16_t b = static_cast<const uint16_t *>(p.x)[i];
        return __uint_as_float(static_cast<uint32_t>(b) << 16);
    }
    return static_cast<const float *>(p.x)[i];
}

}  // namespace qc
