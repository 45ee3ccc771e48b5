// prep.cuh -- memory-bound kernels around the convolution:
//   quantize_pack_kernel : fp32/bf16 NHWC -> packed int8/int4 NHWC (Z4)
//   widen_w4_kernel      : packed int4 KRSC weights -> nibble-plane int8 KRSC (once per layer)
//   widen_w4_pad_kernel  : the same with channel padding (c not a multiple of 32)
//   wsum_w4_kernel       : per-channel weight sums (signed 4-bit activation offset)
//   weights_plain_kernel : 4/8-bit KRSC -> int8 KRSC with channel padding (A8W4, 8-bit padding)
//   repack_pad_kernel    : activation codes with channels padded by x_zero codes
//   repack_s2d_kernel    : activation codes -> 2x2 space-to-depth byte codes (stride-2 stems)
//   zx_table_kernel      : 2-D prefix sums of sum_c w[k,r,s,c] for x_zero != 0 borders (Z2)
//   chsum_kernel, x1_kernel : per-output-pixel sums of (x - x_zero) over in-bounds taps, the
//                          correction term of per-channel weight zero points (Z1)
#pragma once
#include <cstdint>
#include <cuda_bf16.h>
#include "ptx.cuh"
#include "quant.cuh"

namespace qc {

// One thread = 16 consecutive output elements (16 B of int8 or 8 B of int4).
__global__ void __launch_bounds__(256) quantize_pack_kernel(const __grid_constant__ QuantParams p) {
    const int64_t total = p.npix * p.c_pad;
    const int64_t ngroups = (total + 15) / 16;
    for (int64_t g = blockIdx.x * static_cast<int64_t>(blockDim.x) + threadIdx.x; g < ngroups;
         g += static_cast<int64_t>(gridDim.x) * blockDim.x) {
        const int64_t e0 = g * 16;
        int32_t q[16];
        if (p.fast && e0 + 16 <= total) {
            if (p.bf16) {
                const uint4 *src = reinterpret_cast<const uint4 *>(static_cast<const uint16_t *>(p.x) + e0);
                const uint4 a = __ldg(src), b = __ldg(src + 1);
                const uint32_t w[8] = {a.x, a.y, a.z, a.w, b.x, b.y, b.z, b.w};
#pragma unroll
                for (int j = 0; j < 8; ++j) {
                    q[2 * j] = quantize_one(__uint_as_float(w[j] << 16), p);
                    q[2 * j + 1] = quantize_one(__uint_as_float(w[j] & 0xFFFF0000u), p);
                }
            } else {
                const float4 *src = reinterpret_cast<const float4 *>(static_cast<const float *>(p.x) + e0);
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    const float4 v = __ldg(src + j);
                    q[4 * j] = quantize_one(v.x, p);
                    q[4 * j + 1] = quantize_one(v.y, p);
                    q[4 * j + 2] = quantize_one(v.z, p);
                    q[4 * j + 3] = quantize_one(v.w, p);
                }
            }
        } else if (p.c_pad % 16 == 0) {
            // one group = 16 channels of one pixel: a single division per group
            const int32_t gpp = p.c_pad / 16;
            const int64_t pix = g / gpp;
            const int32_t ch0 = static_cast<int32_t>(g - pix * gpp) * 16;
            const int64_t base = pix * p.c;
#pragma unroll
            for (int j = 0; j < 16; ++j) {
                const int32_t ch = ch0 + j;
                q[j] = ch < p.c ? quantize_one(load_x(p, base + ch), p) : p.z;
            }
        } else {
#pragma unroll 1
            for (int j = 0; j < 16; ++j) {
                const int64_t e = e0 + j;
                if (e < total) {
                    const int64_t pix = e / p.c_pad;
                    const int32_t ch = static_cast<int32_t>(e - pix * p.c_pad);
                    q[j] = ch < p.c ? quantize_one(load_x(p, pix * p.c + ch), p) : p.z;
                } else {
                    q[j] = 0;
                }
            }
        }
        if (p.bits == 8) {
            uint32_t w[4];
#pragma unroll
            for (int j = 0; j < 4; ++j)
                w[j] = (q[4 * j] & 0xFF) | ((q[4 * j + 1] & 0xFF) << 8) | ((q[4 * j + 2] & 0xFF) << 16) |
                       (static_cast<uint32_t>(q[4 * j + 3] & 0xFF) << 24);
            uint8_t *dst = static_cast<uint8_t *>(p.y) + e0;
            if (e0 + 16 <= total && (reinterpret_cast<uintptr_t>(dst) & 15u) == 0) {
                *reinterpret_cast<uint4 *>(dst) = make_uint4(w[0], w[1], w[2], w[3]);
            } else {
                for (int j = 0; j < 16 && e0 + j < total; ++j) dst[j] = static_cast<uint8_t>(q[j] & 0xFF);
            }
        } else {
            uint32_t w[2];
#pragma unroll
            for (int j = 0; j < 2; ++j) {
                uint32_t acc = 0;
#pragma unroll
                for (int i = 0; i < 8; ++i) acc |= static_cast<uint32_t>(q[8 * j + i] & 0xF) << (4 * i);
                w[j] = acc;
            }
            uint8_t *dst = static_cast<uint8_t *>(p.y) + e0 / 2;
            if (e0 + 16 <= total && (reinterpret_cast<uintptr_t>(dst) & 7u) == 0) {
                *reinterpret_cast<uint2 *>(dst) = make_uint2(w[0], w[1]);
            } else {
                for (int j = 0; 2 * j < 16 && e0 + 2 * j < total; ++j)
                    dst[j] = static_cast<uint8_t>((q[2 * j] & 0xF) | ((q[2 * j + 1] & 0xF) << 4));
            }
        }
    }
}

// packed int4 KRSC -> prepared int8 KRSC in the "nibble-plane" order the on-chip activation
// widening produces (conv_fwd.cuh widen_word): for every 16-byte packed group (32 channels
// c0..c0+31 of one (k,r,s)), byte p < 16 holds 16 * w[c0 + 2p] and byte 16 + p holds
// w[c0 + 2p + 1] (sign- or zero-extended; 16 w of a 4-bit code fits 8 bits).  Requires
// C % 32 == 0.  n_groups = packed bytes / 16.
__global__ void __launch_bounds__(256) widen_w4_kernel(const uint8_t *__restrict__ w4,
                                                       int8_t *__restrict__ w8, int64_t n_groups,
                                                       int32_t is_signed) {
    for (int64_t i = blockIdx.x * static_cast<int64_t>(blockDim.x) + threadIdx.x; i < n_groups;
         i += static_cast<int64_t>(gridDim.x) * blockDim.x) {
        const uint4 pk = reinterpret_cast<const uint4 *>(w4)[i];
        const uint32_t wd[4] = {pk.x, pk.y, pk.z, pk.w};
        uint32_t out[8];
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            uint32_t lo = 0, hi = 0;
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                int e = (wd[q] >> (8 * j)) & 0xF, o = (wd[q] >> (8 * j + 4)) & 0xF;
                if (is_signed) {
                    e = e >= 8 ? e - 16 : e;
                    o = o >= 8 ? o - 16 : o;
                }
                lo |= (static_cast<uint32_t>(16 * e) & 0xFFu) << (8 * j);
                hi |= (static_cast<uint32_t>(o) & 0xFFu) << (8 * j);
            }
            out[q] = lo;
            out[4 + q] = hi;
        }
        uint4 *dst = reinterpret_cast<uint4 *>(w8) + 2 * i;
        dst[0] = make_uint4(out[0], out[1], out[2], out[3]);
        dst[1] = make_uint4(out[4], out[5], out[6], out[7]);
    }
}

// wsum[k] = sum over (r,s,c) of the true 4-bit weight values of output channel k (row of
// row_bytes packed bytes): the offset correction of signed 4-bit activations (widen_word).
__global__ void __launch_bounds__(256) wsum_w4_kernel(const uint8_t *__restrict__ w4,
                                                      int32_t *__restrict__ wsum, int64_t row_bytes,
                                                      int32_t is_signed) {
    const uint8_t *row = w4 + static_cast<int64_t>(blockIdx.x) * row_bytes;
    int32_t s = 0;
    for (int64_t i = threadIdx.x; i < row_bytes; i += blockDim.x) {
        const int b = row[i];
        int e = b & 0xF, o = b >> 4;
        if (is_signed) {
            e = e >= 8 ? e - 16 : e;
            o = o >= 8 ? o - 16 : o;
        }
        s += e + o;
    }
    __shared__ int32_t red[8];
    for (int off = 16; off > 0; off >>= 1) s += __shfl_xor_sync(0xffffffffu, s, off);
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = s;
    __syncthreads();
    if (threadIdx.x == 0) {
        int32_t t = 0;
        for (int w = 0; w < static_cast<int>(blockDim.x >> 5); ++w) t += red[w];
        wsum[blockIdx.x] = t;
    }
}

// table[k][i][j] = sum_{r<i, s<j} sum_c w8[k,r,s,c]  (i in [0,R], j in [0,S]).
// For an output pixel whose in-bounds taps are r in [r0,r1), s in [s0,s1) the
// padded taps' contribution to subtract is x_zero * (T[r1][s1]-T[r0][s1]-T[r1][s0]+T[r0][s0]).
__global__ void zx_table_kernel(const int8_t *__restrict__ w8, int32_t *__restrict__ table, int K,
                                int R, int S, int C, int is_unsigned, int nib) {
    const int k = blockIdx.x * blockDim.x + threadIdx.x;
    if (k >= K) return;
    int32_t *t = table + static_cast<int64_t>(k) * (R + 1) * (S + 1);
    for (int j = 0; j <= S; ++j) t[j] = 0;
    for (int i = 1; i <= R; ++i) {
        t[i * (S + 1)] = 0;
        int32_t rowsum = 0;
        for (int j = 1; j <= S; ++j) {
            const int8_t *src = w8 + ((static_cast<int64_t>(k) * R + (i - 1)) * S + (j - 1)) * C;
            int32_t s = 0;
            for (int c = 0; c < C; ++c) {
                int32_t v = is_unsigned ? static_cast<int32_t>(static_cast<uint8_t>(src[c]))
                                        : static_cast<int32_t>(src[c]);
                if (nib && (c & 31) < 16) v /= 16;       // nibble-plane prepared 4-bit weights
                s += v;
            }
            rowsum += s;
            t[i * (S + 1) + j] = t[(i - 1) * (S + 1) + j] + rowsum;
        }
    }
}

// ---------------------------------------------------------------------------
// Space-to-depth (2x2) form of a stride-2 convolution (the C=3 stem).
// X2[n,i,j,(2b+b')*c+cc] = q(x[n, 2i+b-pad_h, 2j+b'-pad_w, cc]) (code z outside the image
// or beyond 4c), one code per byte, so that a 7x7/s2 conv over C=3 becomes a 4x4/s1 conv over
// C2=16 with W2[k,a,a',(2b+b')*c+cc] = w[k, 2a+b, 2a'+b', cc] (0 beyond R, S): the same sums.
struct QuantS2DParams {
    const void *x;
    uint8_t *y;
    int32_t n, h, w, c, hs, ws, cs, pad_h, pad_w;
    float inv_s, flo, fhi;
    int32_t z, qmin, qmax, bf16;
};

template <int C>   // C > 0: compile-time channel count (stem: 3); C == 0: runtime p.c
__global__ void __launch_bounds__(256) quantize_s2d_kernel(const __grid_constant__ QuantS2DParams p) {
    QuantParams qp;
    qp.x = p.x; qp.inv_s = p.inv_s; qp.flo = p.flo; qp.fhi = p.fhi;
    qp.z = p.z; qp.qmin = p.qmin; qp.qmax = p.qmax; qp.bf16 = p.bf16;
    const int32_t c = C > 0 ? C : p.c;
    const int64_t total = static_cast<int64_t>(p.n) * p.hs * p.ws;
    const int32_t c4 = 4 * c;
    for (int64_t t = blockIdx.x * static_cast<int64_t>(blockDim.x) + threadIdx.x; t < total;
         t += static_cast<int64_t>(gridDim.x) * blockDim.x) {
        const int64_t img = t / (static_cast<int64_t>(p.hs) * p.ws);
        const int32_t rem = static_cast<int32_t>(t - img * p.hs * p.ws);
        const int32_t i = rem / p.ws, j = rem - (rem / p.ws) * p.ws;
        uint8_t *dst = p.y + t * p.cs;
        for (int32_t ch0 = 0; ch0 < p.cs; ch0 += 16) {
            uint32_t w[4] = {0u, 0u, 0u, 0u};
#pragma unroll
            for (int jj = 0; jj < 16; ++jj) {
                const int32_t ch = ch0 + jj;
                int32_t code = p.z;
                if (ch < c4) {
                    const int32_t blk = ch / c, cc = ch - blk * c;
                    const int32_t hh = 2 * i + (blk >> 1) - p.pad_h;
                    const int32_t ww = 2 * j + (blk & 1) - p.pad_w;
                    if (hh >= 0 && hh < p.h && ww >= 0 && ww < p.w)
                        code = quantize_one(load_x(qp, ((img * p.h + hh) * p.w + ww) * c + cc), qp);
                }
                w[jj >> 2] |= static_cast<uint32_t>(code & 0xFF) << (8 * (jj & 3));
            }
            *reinterpret_cast<uint4 *>(dst + ch0) = make_uint4(w[0], w[1], w[2], w[3]);
        }
    }
}

// Code of element `idx` of a packed row-major 4/8-bit buffer (Z7 nibble order), as int.
__device__ __forceinline__ int32_t get_code(const uint8_t *__restrict__ buf, int64_t idx, int32_t bits,
                                            int32_t is_signed) {
    if (bits == 8) return is_signed ? static_cast<int32_t>(static_cast<int8_t>(buf[idx])) : static_cast<int32_t>(buf[idx]);
    const uint8_t b = buf[idx >> 1];
    int32_t v = (idx & 1) ? (b >> 4) : (b & 0xF);
    if (is_signed && v >= 8) v -= 16;
    return v;
}

// Nibble-plane prepared weights (widen_w4_kernel's layout) of 4-bit KRSC weights whose rows
// of c_src channels are padded with zero weights to c_dst (a multiple of 32) channels.
__global__ void __launch_bounds__(256) widen_w4_pad_kernel(const uint8_t *__restrict__ w4,
                                                           int8_t *__restrict__ w8, int64_t rows,
                                                           int32_t c_src, int32_t c_dst, int32_t is_signed) {
    const int32_t gpr = c_dst / 32;
    const int64_t n_groups = rows * gpr;
    for (int64_t i = blockIdx.x * static_cast<int64_t>(blockDim.x) + threadIdx.x; i < n_groups;
         i += static_cast<int64_t>(gridDim.x) * blockDim.x) {
        const int64_t row = i / gpr;
        const int32_t c0 = static_cast<int32_t>(i - row * gpr) * 32;
        int8_t *dst = w8 + row * c_dst + c0;
        for (int p = 0; p < 16; ++p) {
            const int32_t ce = c0 + 2 * p, co = ce + 1;
            const int32_t e = ce < c_src ? get_code(w4, row * c_src + ce, 4, is_signed) : 0;
            const int32_t o = co < c_src ? get_code(w4, row * c_src + co, 4, is_signed) : 0;
            dst[p] = static_cast<int8_t>(16 * e);
            dst[16 + p] = static_cast<int8_t>(o);
        }
    }
}

// int8 KRSC from 4- or 8-bit packed KRSC, rows of c_src channels padded to c_dst with zero
// weights (A8W4 weights; 8-bit channel padding).
// rows = K*R*s_dst output filter rows; filter columns s >= s_src and channels c >= c_src are 0.
__global__ void __launch_bounds__(256) weights_plain_kernel(const uint8_t *__restrict__ w, int8_t *__restrict__ w8,
                                                            int64_t rows, int32_t c_src, int32_t c_dst,
                                                            int32_t bits, int32_t is_signed, int32_t s_src,
                                                            int32_t s_dst) {
    const int64_t total = rows * c_dst;
    for (int64_t e = blockIdx.x * static_cast<int64_t>(blockDim.x) + threadIdx.x; e < total;
         e += static_cast<int64_t>(gridDim.x) * blockDim.x) {
        const int64_t row = e / c_dst;
        const int32_t c = static_cast<int32_t>(e - row * c_dst);
        const int64_t kr = row / s_dst;
        const int32_t sc = static_cast<int32_t>(row - kr * s_dst);
        w8[e] = static_cast<int8_t>(c < c_src && sc < s_src ? get_code(w, (kr * s_src + sc) * c_src + c, bits, is_signed) : 0);
    }
}

// Activation codes [npix][c_src] -> [npix][c_dst] (same packing), pad channels = zx.
// One thread = one pixel: its c_src codes, then x_zero codes up to c_dst channels, written as
// 16-byte vectors (c_dst * bits / 8 is a multiple of 16 for every padded shape qconv.cu makes).
// npix output pixels of rows w_dst wide; output columns >= w_src are all zx codes.
__global__ void __launch_bounds__(256) repack_pad_kernel(const uint8_t *__restrict__ x, uint8_t *__restrict__ y,
                                                         int64_t npix, int32_t c_src, int32_t c_dst,
                                                         int32_t bits, int32_t zx, int32_t w_src, int32_t w_dst) {
    const int32_t ob = c_dst * bits / 8;      // output bytes per pixel
    const uint32_t z8 = static_cast<uint32_t>(zx) & 0xFFu;
    const uint32_t z4 = static_cast<uint32_t>(zx) & 0xFu;
    for (int64_t pix = blockIdx.x * static_cast<int64_t>(blockDim.x) + threadIdx.x; pix < npix;
         pix += static_cast<int64_t>(gridDim.x) * blockDim.x) {
        const int64_t row = pix / w_dst;
        const int32_t col = static_cast<int32_t>(pix - row * w_dst);
        const int32_t c_in = col < w_src ? c_src : 0;  // codes taken from x (the rest are zx)
        const int64_t base = (row * w_src + col) * c_src;   // first code of the pixel (element index)
        uint4 *dst = reinterpret_cast<uint4 *>(y + pix * ob);
        for (int32_t q = 0; q < ob / 16; ++q) {
            uint32_t w[4];
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                uint32_t v = 0;
#pragma unroll
                for (int b = 0; b < 4; ++b) {
                    const int32_t j = 16 * q + 4 * k + b;       // output byte
                    uint32_t byte;
                    if (bits == 8) {
                        byte = j < c_in ? static_cast<uint32_t>(__ldg(x + base + j)) : z8;
                    } else {
                        byte = 0;
#pragma unroll
                        for (int h = 0; h < 2; ++h) {
                            const int32_t c = 2 * j + h;
                            const int64_t idx = base + c;
                            const uint32_t nib = c < c_in ? ((static_cast<uint32_t>(__ldg(x + (idx >> 1))) >> (4 * (idx & 1))) & 0xFu) : z4;
                            byte |= nib << (4 * h);
                        }
                    }
                    v |= byte << (8 * b);
                }
                w[k] = v;
            }
            dst[q] = make_uint4(w[0], w[1], w[2], w[3]);
        }
    }
}

// Activation codes (4/8-bit packed, c channels) -> space-to-depth byte codes X2 [n][hs][ws][cs]:
// X2[n,i,j,(2b+b')*c+cc] = code(x[n, 2i+b-pad_h, 2j+b'-pad_w, cc]), zx outside the image or
// beyond 4c; 4-bit codes sign/zero-extended to a byte.
__global__ void __launch_bounds__(256) repack_s2d_kernel(const uint8_t *__restrict__ x, uint8_t *__restrict__ y,
                                                         int32_t n, int32_t h, int32_t w, int32_t c,
                                                         int32_t hs, int32_t ws, int32_t cs, int32_t pad_h,
                                                         int32_t pad_w, int32_t bits, int32_t is_signed,
                                                         int32_t zx) {
    const int64_t total = static_cast<int64_t>(n) * hs * ws * cs;
    for (int64_t e = blockIdx.x * static_cast<int64_t>(blockDim.x) + threadIdx.x; e < total;
         e += static_cast<int64_t>(gridDim.x) * blockDim.x) {
        int64_t rest = e;
        const int32_t ch = static_cast<int32_t>(rest % cs); rest /= cs;
        const int32_t j = static_cast<int32_t>(rest % ws); rest /= ws;
        const int32_t i = static_cast<int32_t>(rest % hs); rest /= hs;
        const int64_t img = rest;
        int32_t code = zx;
        if (ch < 4 * c) {
            const int32_t blk = ch / c, cc = ch - blk * c;
            const int32_t hh = 2 * i + (blk >> 1) - pad_h;
            const int32_t ww = 2 * j + (blk & 1) - pad_w;
            if (hh >= 0 && hh < h && ww >= 0 && ww < w)
                code = get_code(x, ((img * h + hh) * w + ww) * c + cc, bits, is_signed);
        }
        y[e] = static_cast<uint8_t>(code & 0xFF);
    }
}

// chsum[pix] = sum_c (x[pix, c] - zx) over the true channels of every input pixel.
__global__ void __launch_bounds__(256) chsum_kernel(const uint8_t *__restrict__ x, int32_t *__restrict__ chsum,
                                                    int64_t npix, int32_t c, int32_t bits, int32_t is_signed,
                                                    int32_t zx) {
    const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    const int64_t nwarps = (static_cast<int64_t>(gridDim.x) * blockDim.x) >> 5;
    for (int64_t pix = warp; pix < npix; pix += nwarps) {
        int32_t s = 0;
        for (int32_t ch = lane; ch < c; ch += 32) s += get_code(x, pix * c + ch, bits, is_signed) - zx;
        for (int off = 16; off > 0; off >>= 1) s += __shfl_xor_sync(0xffffffffu, s, off);
        if (lane == 0) chsum[pix] = s;
    }
}

// x1[m] = sum over the in-bounds taps (r, s) of output pixel m of chsum[input pixel]:
// sum_{taps, c} (x - zx) with padded taps contributing nothing (Z2).
__global__ void __launch_bounds__(256) x1_kernel(const int32_t *__restrict__ chsum, int32_t *__restrict__ x1,
                                                 int32_t n, int32_t h, int32_t w, int32_t P, int32_t Q,
                                                 int32_t R, int32_t S, int32_t sh, int32_t sw, int32_t ph,
                                                 int32_t pw, int32_t dh, int32_t dw) {
    const int64_t M = static_cast<int64_t>(n) * P * Q;
    for (int64_t m = blockIdx.x * static_cast<int64_t>(blockDim.x) + threadIdx.x; m < M;
         m += static_cast<int64_t>(gridDim.x) * blockDim.x) {
        const int64_t img = m / (static_cast<int64_t>(P) * Q);
        const int32_t rem = static_cast<int32_t>(m - img * P * Q);
        const int32_t p = rem / Q, q = rem - (rem / Q) * Q;
        int32_t s = 0;
        for (int32_t r = 0; r < R; ++r) {
            const int32_t hh = p * sh - ph + r * dh;
            if (hh < 0 || hh >= h) continue;
            for (int32_t t = 0; t < S; ++t) {
                const int32_t ww = q * sw - pw + t * dw;
                if (ww < 0 || ww >= w) continue;
                s += chsum[(img * h + hh) * w + ww];
            }
        }
        x1[m] = s;
    }
}

// W2 (int8 KRSC of the transformed conv) from packed w (4- or 8-bit codes).
__global__ void __launch_bounds__(256) weights_s2d_kernel(const uint8_t *__restrict__ w,
                                                          int8_t *__restrict__ w2, int32_t k, int32_t r,
                                                          int32_t s, int32_t c, int32_t r2, int32_t s2,
                                                          int32_t cs, int32_t bits, int32_t is_signed) {
    const int64_t total = static_cast<int64_t>(k) * r2 * s2 * cs;
    for (int64_t e = blockIdx.x * static_cast<int64_t>(blockDim.x) + threadIdx.x; e < total;
         e += static_cast<int64_t>(gridDim.x) * blockDim.x) {
        int64_t rest = e;
        const int32_t ch = static_cast<int32_t>(rest % cs); rest /= cs;
        const int32_t a2 = static_cast<int32_t>(rest % s2); rest /= s2;
        const int32_t a1 = static_cast<int32_t>(rest % r2); rest /= r2;
        const int32_t kk = static_cast<int32_t>(rest);
        int32_t v = 0;
        if (ch < 4 * c) {
            const int32_t blk = ch / c, cc = ch - blk * c;
            const int32_t rr = 2 * a1 + (blk >> 1), ss = 2 * a2 + (blk & 1);
            if (rr < r && ss < s) {
                const int64_t idx = ((static_cast<int64_t>(kk) * r + rr) * s + ss) * c + cc;
                if (bits == 8) {
                    v = is_signed ? static_cast<int32_t>(static_cast<int8_t>(w[idx])) : static_cast<int32_t>(w[idx]);
                } else {
                    const uint8_t b = w[idx >> 1];
                    v = (idx & 1) ? (b >> 4) : (b & 0xF);
                    if (is_signed && v >= 8) v -= 16;
                }
            }
        }
        w2[e] = static_cast<int8_t>(v);
    }
}

// Debug: one im2col TMA tile straight to global memory (no swizzle).
__global__ void qconv_debug_im2col_kernel(const __grid_constant__ CUtensorMap xmap, int32_t c,
                                          int32_t w, int32_t h, int32_t n, uint16_t ow,
                                          uint16_t oh, uint32_t bytes, uint8_t *out) {
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    // 1024-byte aligned base by pointer arithmetic on the shared array itself (no integer round
    // trip): the compiler keeps it in the shared window, so every smem_u32() below is one add
    uint8_t *smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
    __shared__ __align__(8) uint64_t bar;
    if (threadIdx.x == 0) {
        mbar_init(&bar, 1);
        fence_mbar_init();
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        mbar_arrive_expect_tx(&bar, bytes);
        tma_load_im2col_4d(smem, &xmap, &bar, c, w, h, n, ow, oh);
    }
    mbar_wait(&bar, 0);
    for (uint32_t i = threadIdx.x; i < bytes; i += blockDim.x) out[i] = smem[i];
}

}  // namespace qc
