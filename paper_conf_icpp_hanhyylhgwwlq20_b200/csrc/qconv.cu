// qconv.cu -- host side of libqconv.so: the C ABI declared in include/qconv.h.
//
// Validation, the overflow bound, the per-shape launch plan (tile sizes,
// pipeline depth, shared-memory carve-up), TMA descriptor encoding (im2col
// for activations, tiled for weights) and kernel launches.  All device work
// is in conv_fwd.cuh / prep.cuh.  Nothing here allocates device memory.
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdint>
#include <cstring>
#include <mutex>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "qconv.h"
#include "conv_fwd.cuh"
#include "prep.cuh"
#include "halo.cuh"
#include "trans.cuh"
#include "fwd2.cuh"

namespace {

thread_local int g_last_cuda_error = 0;

qc_status cuda_fail(cudaError_t e) {
    g_last_cuda_error = static_cast<int>(e);
    return QC_ERR_CUDA;
}

bool is_int_input(qc_dtype t) { return t == QC_U4 || t == QC_S4 || t == QC_U8 || t == QC_S8; }
bool is_valid_dtype(qc_dtype t) { return is_int_input(t) || t == QC_S32; }
int dtype_bits(qc_dtype t) { return (t == QC_U4 || t == QC_S4) ? 4 : (t == QC_S32 ? 32 : 8); }
bool dtype_signed(qc_dtype t) { return t == QC_S4 || t == QC_S8 || t == QC_S32; }
int64_t dtype_min(qc_dtype t) {
    switch (t) {
        case QC_U4: return 0;
        case QC_S4: return -8;
        case QC_U8: return 0;
        case QC_S8: return -128;
        default: return INT32_MIN;
    }
}
int64_t dtype_max(qc_dtype t) {
    switch (t) {
        case QC_U4: return 15;
        case QC_S4: return 7;
        case QC_U8: return 255;
        case QC_S8: return 127;
        default: return INT32_MAX;
    }
}
bool aligned16(const void *p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }
size_t align_up(size_t v, size_t a) { return (v + a - 1) / a * a; }
// MMA operand signedness of the activations: 4-bit codes are widened to unsigned bytes
// (nibble-plane widening, conv_fwd.cuh widen_word); 8-bit codes are used as they are.
bool act_signed(const qconv_desc *d) { return dtype_bits(d->x_t) == 8 && dtype_signed(d->x_t); }

// ------------------------------------------------------------------ driver entry points
typedef CUresult (*PFN_encodeIm2col)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *,
                                     const cuuint64_t *, const cuuint64_t *, const int *,
                                     const int *, cuuint32_t, cuuint32_t, const cuuint32_t *,
                                     CUtensorMapInterleave, CUtensorMapSwizzle,
                                     CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
typedef CUresult (*PFN_encodeTiled)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *,
                                    const cuuint64_t *, const cuuint64_t *, const cuuint32_t *,
                                    const cuuint32_t *, CUtensorMapInterleave, CUtensorMapSwizzle,
                                    CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

struct Driver {
    PFN_encodeIm2col im2col = nullptr;
    PFN_encodeTiled tiled = nullptr;
    int driver_version = 0;
    cudaError_t err = cudaSuccess;
};

const Driver &driver() {
    static Driver d;
    static std::once_flag once;
    std::call_once(once, [] {
        void *f1 = nullptr, *f2 = nullptr;
        cudaDriverEntryPointQueryResult q1, q2;
        cudaError_t e1 = cudaGetDriverEntryPoint("cuTensorMapEncodeIm2col", &f1, cudaEnableDefault, &q1);
        cudaError_t e2 = cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f2, cudaEnableDefault, &q2);
        if (e1 != cudaSuccess || e2 != cudaSuccess || q1 != cudaDriverEntryPointSuccess ||
            q2 != cudaDriverEntryPointSuccess) {
            d.err = e1 != cudaSuccess ? e1 : (e2 != cudaSuccess ? e2 : cudaErrorSymbolNotFound);
            return;
        }
        d.im2col = reinterpret_cast<PFN_encodeIm2col>(f1);
        d.tiled = reinterpret_cast<PFN_encodeTiled>(f2);
        cudaDriverGetVersion(&d.driver_version);
    });
    return d;
}

// Driver releases up to 13.1 mis-handle a descriptor flag for tensors under
// 128 KiB; clearing bit 21 of the second descriptor word is the documented
// workaround used by NVIDIA's own TMA helpers.
void small_tensor_fixup(CUtensorMap *m, uint64_t tensor_bytes) {
    if (driver().driver_version <= 13010 && tensor_bytes < 131072)
        reinterpret_cast<uint64_t *>(m)[1] &= ~(1ull << 21);
}

int num_sms() {
    static int cache[64] = {0};
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 0 || dev >= 64) dev = 0;
    if (cache[dev] == 0) {
        int n = 0;
        cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
        cache[dev] = n > 0 ? n : 148;
    }
    return cache[dev];
}

// ------------------------------------------------------------------ descriptor validation
struct Geometry {
    int P, Q;
    int64_t M;
    int bits;
    int c_bytes;        // packed bytes per input pixel
    int64_t x_bytes, w_bytes, w8_bytes, y_bytes;
};

qc_status validate_desc(const qconv_desc *d, Geometry *g) {
    if (!d) return QC_ERR_INVALID_ARG;
    if (d->n < 1 || d->h < 1 || d->w < 1 || d->c < 1 || d->k < 1 || d->r < 1 || d->s < 1)
        return QC_ERR_INVALID_ARG;
    if (d->stride_h < 1 || d->stride_w < 1 || d->dil_h < 1 || d->dil_w < 1 || d->pad_h < 0 ||
        d->pad_w < 0)
        return QC_ERR_INVALID_ARG;
    if (!is_int_input(d->x_t) || !is_int_input(d->w_t) || !is_valid_dtype(d->y_t))
        return QC_ERR_INVALID_ARG;
    const int P = (d->h + 2 * d->pad_h - d->dil_h * (d->r - 1) - 1) / d->stride_h + 1;
    const int Q = (d->w + 2 * d->pad_w - d->dil_w * (d->s - 1) - 1) / d->stride_w + 1;
    if (d->h + 2 * d->pad_h - d->dil_h * (d->r - 1) - 1 < 0 ||
        d->w + 2 * d->pad_w - d->dil_w * (d->s - 1) - 1 < 0 || P < 1 || Q < 1)
        return QC_ERR_INVALID_ARG;
    if (d->x_zero < dtype_min(d->x_t) || d->x_zero > dtype_max(d->x_t)) return QC_ERR_INVALID_ARG;
    if (d->y_t != QC_S32) {
        if (d->y_zero < dtype_min(d->y_t) || d->y_zero > dtype_max(d->y_t)) return QC_ERR_INVALID_ARG;
        if (d->clamp_lo > d->clamp_hi || d->clamp_lo < dtype_min(d->y_t) ||
            d->clamp_hi > dtype_max(d->y_t))
            return QC_ERR_INVALID_ARG;
    }
    const int bits = dtype_bits(d->x_t);
    if (bits == 4 && (d->c % 2)) return QC_ERR_INVALID_ARG;
    const int64_t M = static_cast<int64_t>(d->n) * P * Q;
    g->P = P;
    g->Q = Q;
    g->M = M;
    g->bits = bits;
    g->c_bytes = d->c * bits / 8;
    g->x_bytes = static_cast<int64_t>(d->n) * d->h * d->w * g->c_bytes;
    g->w8_bytes = static_cast<int64_t>(d->k) * d->r * d->s * d->c;
    g->w_bytes = g->w8_bytes * dtype_bits(d->w_t) / 8;
    const int yb = dtype_bits(d->y_t);
    if (yb == 4 && (d->k % 2)) return QC_ERR_UNSUPPORTED;
    g->y_bytes = M * d->k * yb / 8;
    return QC_OK;
}

// Support + overflow checks for the GPU path (after validate_desc).
qc_status check_supported(const qconv_desc *d, const Geometry &g) {
    if (dtype_bits(d->x_t) != dtype_bits(d->w_t)) return QC_ERR_UNSUPPORTED;   // mixed widths: NEXT
    const bool pair = dtype_bits(d->x_t) == 8 && d->c == 16;   // 2 taps per 32-byte K-stage
    if (d->c % 32 && !pair) return QC_ERR_UNSUPPORTED;   // MMA K granularity / 16-byte TMA strides
    if (d->stride_h > 8 || d->stride_w > 8) return QC_ERR_UNSUPPORTED;   // TMA traversal stride
    const int lw = -d->pad_w, lh = -d->pad_h;
    const int uw = d->pad_w - d->dil_w * (d->s - 1), uh = d->pad_h - d->dil_h * (d->r - 1);
    if (lw < -128 || lh < -128 || uw < -128 || uh < -128 || uw > 127 || uh > 127)
        return QC_ERR_UNSUPPORTED;                     // rank-4 im2col corner range
    if (d->dil_w * (d->s - 1) > 255 || d->dil_h * (d->r - 1) > 255) return QC_ERR_UNSUPPORTED;
    if (g.M > INT32_MAX - 256 || d->n > 65535) return QC_ERR_UNSUPPORTED;
    if (static_cast<int64_t>(d->r) * d->s * d->c > INT32_MAX / 2) return QC_ERR_UNSUPPORTED;
    // int32 accumulation bound ("overflow well addressed"): both the raw MMA sum and the
    // zero-point-centred sum must stay inside int32 for any codes of these dtypes.
    const int64_t T = static_cast<int64_t>(d->r) * d->s * d->c;
    const int64_t wmax = std::max(-dtype_min(d->w_t), dtype_max(d->w_t));
    const int64_t xraw = std::max(-dtype_min(d->x_t), dtype_max(d->x_t));
    const int64_t xctr = std::max(d->x_zero - dtype_min(d->x_t), dtype_max(d->x_t) - d->x_zero);
    // 4-bit activations are widened to 16 x (x [+ 8]) (nibble-plane widening): the MMA sum
    // is 16 x larger and must stay below 2^30 (the epilogue adds 16 * bias inside int32)
    const double lim = dtype_bits(d->x_t) == 4 ? 67108864.0 /* 2^30 / 16 */ : 2147483647.0;
    const double xw = dtype_bits(d->x_t) == 4 ? 15.0 : static_cast<double>(std::max(xraw, xctr));
    if (static_cast<double>(T) * xraw * wmax > lim || static_cast<double>(T) * xctr * wmax > lim ||
        static_cast<double>(T) * xw * wmax > lim)
        return QC_ERR_OVERFLOW_RISK;
    return QC_OK;
}

// ------------------------------------------------------------------ launch plan
struct Plan {
    int BK, bkp, chunks, BN, n_tiles_n, num_tiles, num_kb, stages, grid, threads;
    uint32_t tmem_cols, smem_bytes;
    qc::ConvParams cp;
};

int choose_bk(int c) { return (c % 128 == 0) ? 128 : (c % 64 == 0 ? 64 : 32); }
uint32_t pow2_cols(int n) {
    uint32_t c = 32;
    while (c < static_cast<uint32_t>(n)) c <<= 1;
    return c;
}

qc_status make_plan(const qconv_desc *d, const Geometry &g, Plan *pl) {
    const bool is4 = g.bits == 4;
    const bool pair = !is4 && d->c == 16;
    pl->BK = pair ? 32 : choose_bk(d->c);
    pl->bkp = is4 ? pl->BK / 2 : (pair ? 16 : pl->BK);
    pl->chunks = pair ? 1 : d->c / pl->BK;
    pl->num_kb = pair ? (d->r * d->s + 1) / 2 : d->r * d->s * pl->chunks;
    const int m_tiles = static_cast<int>((g.M + qc::kBM - 1) / qc::kBM);
    const int sms = num_sms();
    int BN = std::min(qc::kMaxBN, ((d->k + 15) / 16) * 16);
    // smaller N tiles when the grid would not fill the GPU (paper P:L321: at small batch the
    // tiling decides how well the machine is filled)
    while (BN > 64 && static_cast<int64_t>(m_tiles) * ((d->k + BN - 1) / BN) < sms) {
        BN = std::max(64, ((BN / 2 + 15) / 16) * 16);
    }
    pl->BN = BN;
    pl->n_tiles_n = (d->k + BN - 1) / BN;
    pl->num_tiles = m_tiles * pl->n_tiles_n;
    pl->tmem_cols = pow2_cols(2 * BN);
    const uint32_t a_bytes = static_cast<uint32_t>(qc::kBM * pl->BK);
    const uint32_t b_bytes = static_cast<uint32_t>(align_up(static_cast<size_t>(BN) * pl->BK, 1024));
    const uint32_t stg_bytes = is4 ? static_cast<uint32_t>(qc::kBM * pl->bkp) : 0u;
    const uint32_t per_stage = a_bytes + b_bytes + stg_bytes;
    const int ybits = dtype_bits(d->y_t);
    const int tile_row_bytes = BN * ybits / 8;
    const int y_gw = tile_row_bytes >= 128 ? 128 : tile_row_bytes;
    const bool y_tma = d->y_t != QC_S32 && BN % 32 == 0 &&
                       (static_cast<int64_t>(d->k) * ybits / 8) % 16 == 0 &&
                       (y_gw == 32 || y_gw == 64 || (y_gw == 128 && tile_row_bytes % 128 == 0));
    const uint32_t ystg_one = y_tma ? 128u * static_cast<uint32_t>(tile_row_bytes) : 0u;
    const uint32_t ystg_bytes = 2u * ystg_one;   // double-buffered
    const uint32_t fixed = static_cast<uint32_t>(qc::kMaxBN) * 16u + 128u + 1024u + ystg_bytes;
    const uint32_t budget = 227u * 1024u - 1024u - fixed;
    int stages = static_cast<int>(budget / per_stage);
    stages = std::min(stages, 32);     // deep rings: TMA latency is ~1-3 us under load
    if (stages < 2) return QC_ERR_UNSUPPORTED;
    pl->stages = stages;
    qc::ConvParams &p = pl->cp;
    std::memset(&p, 0, sizeof(p));
    p.off_a = 0;
    p.off_b = p.off_a + a_bytes * stages;
    p.off_stg = p.off_b + b_bytes * stages;
    p.off_ystg = static_cast<uint32_t>(align_up(p.off_stg + stg_bytes * stages, 1024));
    p.ystg_bytes = ystg_one;
    p.y_tma = y_tma ? 1 : 0;
    p.y_gw = y_gw;
    p.y_gmask = y_gw == 128 ? 7 : (y_gw == 64 ? 3 : 1);
    p.n_ygroups = y_tma ? tile_row_bytes / y_gw : 0;
    p.off_par = static_cast<uint32_t>(align_up(p.off_ystg + ystg_bytes, 16));
    p.off_bar = static_cast<uint32_t>(align_up(p.off_par + static_cast<uint32_t>(qc::kMaxBN) * 16u + 128u, 8));
    const uint32_t bar_bytes = static_cast<uint32_t>((3 * stages + 4) * 8 + 16);
    pl->smem_bytes = p.off_bar + bar_bytes + 1024u;       // + alignment slack for the 1024-B base
    pl->grid = std::min(pl->num_tiles, sms);
    pl->threads = is4 ? 512 : 384;
    p.a_stage_bytes = a_bytes;
    p.b_stage_bytes = b_bytes;
    p.stg_stage_bytes = stg_bytes;
    p.M = static_cast<int32_t>(g.M);
    p.P = g.P;
    p.Q = g.Q;
    p.PQ = g.P * g.Q;
    p.K = d->k;
    p.BN = BN;
    p.n_tiles_n = pl->n_tiles_n;
    p.num_tiles = pl->num_tiles;
    p.num_kb = pl->num_kb;
    p.chunks = pl->chunks;
    p.S = d->s;
    p.R = d->r;
    p.stride_h = d->stride_h;
    p.stride_w = d->stride_w;
    p.pad_h = d->pad_h;
    p.pad_w = d->pad_w;
    p.dil_h = d->dil_h;
    p.dil_w = d->dil_w;
    p.H = d->h;
    p.W = d->w;
    p.C8 = d->c;
    p.BK = pl->BK;
    p.bkp = pl->bkp;
    p.stages = stages;
    p.sw_layout = pl->BK == 128 ? 2 : (pl->BK == 64 ? 4 : 6);
    p.pair = pair ? 1 : 0;
    p.cvt_shift = pl->bkp >= 64 ? 2 : (pl->bkp >= 32 ? 1 : 0);
    p.need_clamp = (d->y_t != QC_S32 && (d->clamp_lo > dtype_min(d->y_t) || d->clamp_hi < dtype_max(d->y_t))) ? 1 : 0;
    p.sw_mask = pl->BK == 128 ? 7 : (pl->BK == 64 ? 3 : 1);
    p.idesc = qc::make_idesc_i8(qc::kBM, static_cast<uint32_t>(BN), act_signed(d), dtype_signed(d->w_t));
    p.tmem_cols = pl->tmem_cols;
    p.y_zero = d->y_t == QC_S32 ? 0 : d->y_zero;
    p.clamp_lo = d->y_t == QC_S32 ? INT32_MIN : d->clamp_lo;
    p.clamp_hi = d->y_t == QC_S32 ? INT32_MAX : d->clamp_hi;
    p.x_zero = d->x_zero;
    p.y_row_bytes = static_cast<int64_t>(d->k) * dtype_bits(d->y_t) / 8;
    return QC_OK;
}

CUtensorMapSwizzle swizzle_for(int bk) {
    return bk == 128 ? CU_TENSOR_MAP_SWIZZLE_128B
                     : (bk == 64 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_32B);
}

// Packed 4-bit staging rows of `bytes` per pixel are loaded swizzled whenever the row width
// allows (32/64/128 B): SWIZZLE_NONE boxes are moved in 16-byte requests, several times slower
// (measured: conv1/halo ablations, r1).  The converter reads the swizzled layout (widen_stage).
CUtensorMapSwizzle packed_swizzle(int bytes) {
    return bytes == 128 ? CU_TENSOR_MAP_SWIZZLE_128B
                        : (bytes == 64 ? CU_TENSOR_MAP_SWIZZLE_64B
                                       : (bytes == 32 ? CU_TENSOR_MAP_SWIZZLE_32B : CU_TENSOR_MAP_SWIZZLE_NONE));
}
int packed_sw_mask(int bytes) { return bytes == 128 ? 7 : (bytes == 64 ? 3 : (bytes == 32 ? 1 : 0)); }

qc_status encode_x_map(const qconv_desc *d, const Geometry &g, const void *x, int box_bytes,
                       CUtensorMapSwizzle sw, CUtensorMap *map, int pixels = qc::kBM) {
    const Driver &drv = driver();
    if (!drv.im2col) return cuda_fail(drv.err);
    const cuuint64_t cb = static_cast<cuuint64_t>(g.c_bytes);
    cuuint64_t dims[4] = {cb, static_cast<cuuint64_t>(d->w), static_cast<cuuint64_t>(d->h),
                          static_cast<cuuint64_t>(d->n)};
    cuuint64_t strides[3] = {cb, cb * d->w, cb * d->w * d->h};
    int lower[2] = {-d->pad_w, -d->pad_h};
    int upper[2] = {d->pad_w - d->dil_w * (d->s - 1), d->pad_h - d->dil_h * (d->r - 1)};
    cuuint32_t estr[4] = {1, static_cast<cuuint32_t>(d->stride_w), static_cast<cuuint32_t>(d->stride_h), 1};
    CUresult r = drv.im2col(map, CU_TENSOR_MAP_DATA_TYPE_UINT8, 4, const_cast<void *>(x), dims,
                            strides, lower, upper, static_cast<cuuint32_t>(box_bytes),
                            static_cast<cuuint32_t>(pixels), estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                            sw, CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) return cuda_fail(cudaErrorInvalidValue);
    small_tensor_fixup(map, static_cast<uint64_t>(g.x_bytes));
    return QC_OK;
}

qc_status encode_w_map(const qconv_desc *d, const Geometry &g, const void *w8, int bk, int bn,
                       CUtensorMapSwizzle sw, CUtensorMap *map) {
    const Driver &drv = driver();
    if (!drv.tiled) return cuda_fail(drv.err);
    const cuuint64_t kg = static_cast<cuuint64_t>(d->r) * d->s * d->c;
    cuuint64_t dims[2] = {kg, static_cast<cuuint64_t>(d->k)};
    cuuint64_t strides[1] = {kg};
    cuuint32_t box[2] = {static_cast<cuuint32_t>(bk), static_cast<cuuint32_t>(bn)};
    cuuint32_t estr[2] = {1, 1};
    CUresult r = drv.tiled(map, CU_TENSOR_MAP_DATA_TYPE_UINT8, 2, const_cast<void *>(w8), dims,
                           strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE, sw,
                           CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) return cuda_fail(cudaErrorInvalidValue);
    small_tensor_fixup(map, static_cast<uint64_t>(g.w8_bytes));
    return QC_OK;
}

// Weights of the channel-major kernel (trans.cuh): a 4-D view {kg bytes, 8, 2, k/16} with
// strides {2 kg, kg, 16 kg} so that the tile's shared-memory row r = pl + 8 par + 16 ph holds
// channel 2 pl + par + 16 ph -- TMEM lanes l and l+8 of every 16-lane group then hold the
// channel pair (2i, 2i+1).  Requires k % 16 == 0.
qc_status encode_w_map_pairs(const qconv_desc *d, const Geometry &g, const void *w8, int bk, int bm,
                             CUtensorMapSwizzle sw, CUtensorMap *map) {
    const Driver &drv = driver();
    if (!drv.tiled) return cuda_fail(drv.err);
    const cuuint64_t kg = static_cast<cuuint64_t>(d->r) * d->s * d->c;
    cuuint64_t dims[4] = {kg, 8, 2, static_cast<cuuint64_t>(d->k / 16)};
    cuuint64_t strides[3] = {2 * kg, kg, 16 * kg};
    cuuint32_t box[4] = {static_cast<cuuint32_t>(bk), 8, 2, static_cast<cuuint32_t>(bm / 16)};
    cuuint32_t estr[4] = {1, 1, 1, 1};
    CUresult r = drv.tiled(map, CU_TENSOR_MAP_DATA_TYPE_UINT8, 4, const_cast<void *>(w8), dims,
                           strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE, sw,
                           CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) return cuda_fail(cudaErrorInvalidValue);
    small_tensor_fixup(map, static_cast<uint64_t>(g.w8_bytes));
    return QC_OK;
}

qc_status encode_y_map(const qconv_desc *d, const Geometry &g, void *y, int gw, CUtensorMap *map,
                       int rows = qc::kBM, bool swizzle = true) {
    const Driver &drv = driver();
    if (!drv.tiled) return cuda_fail(drv.err);
    const int yb = dtype_bits(d->y_t);
    const cuuint64_t row = static_cast<cuuint64_t>(d->k) * yb / 8;
    cuuint64_t dims[2] = {row, static_cast<cuuint64_t>(g.M)};
    cuuint64_t strides[1] = {row};
    cuuint32_t box[2] = {static_cast<cuuint32_t>(gw), static_cast<cuuint32_t>(rows)};
    cuuint32_t estr[2] = {1, 1};
    CUresult r = drv.tiled(map, CU_TENSOR_MAP_DATA_TYPE_UINT8, 2, y, dims, strides, box, estr,
                           CU_TENSOR_MAP_INTERLEAVE_NONE, swizzle ? swizzle_for(gw) : CU_TENSOR_MAP_SWIZZLE_NONE,
                           CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) return cuda_fail(cudaErrorInvalidValue);
    small_tensor_fixup(map, static_cast<uint64_t>(g.y_bytes));
    return QC_OK;
}

// Programmatic dependent launch (see ptx.cuh griddep_wait): the conv kernels may start while
// the previous kernel of the stream drains; QC_NO_PDL=1 disables it (debug).
void set_pdl(cudaLaunchConfig_t &cfg, cudaLaunchAttribute *attr) {
    static const bool off = std::getenv("QC_NO_PDL") != nullptr;
    if (off) return;
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
}

// Debug hooks (never set in normal use): QC_EXPERIMENT=<flags> ablations, and
// QC_TRACE=<file> timestamps of CTA 0's pipeline events, appended to the file after a sync.
qc::ConvParams debug_params(const qc::ConvParams &base, cudaStream_t stream) {
    static const char *trace_file = std::getenv("QC_TRACE");
    static const char *exp_env = std::getenv("QC_EXPERIMENT");
    qc::ConvParams cp = base;
    cp.exp_flags = exp_env ? std::atoi(exp_env) : 0;
    cp.trace = nullptr;
    if (trace_file) {
        unsigned long long *tbuf = nullptr;
        cudaMalloc(&tbuf, 16 * 1024 * sizeof(unsigned long long));
        cudaMemsetAsync(tbuf, 0, 16 * 1024 * sizeof(unsigned long long), stream);
        cp.trace = tbuf;
    }
    return cp;
}

void debug_dump(const qc::ConvParams &cp, cudaStream_t stream) {
    if (!cp.trace) return;
    std::vector<unsigned long long> h(16 * 1024);
    cudaMemcpyAsync(h.data(), cp.trace, h.size() * 8, cudaMemcpyDeviceToHost, stream);
    cudaStreamSynchronize(stream);
    cudaFree(cp.trace);
    if (FILE *f = std::fopen(std::getenv("QC_TRACE"), "ab")) {
        std::fwrite(h.data(), 8, h.size(), f);
        std::fclose(f);
    }
}

template <bool IS4, int OUT, bool ZX>
qc_status launch_conv_t(const Plan &pl, const CUtensorMap &xm, const CUtensorMap &wm,
                        const CUtensorMap &ym, cudaStream_t stream) {
    auto kern = qc::qconv_fwd_kernel<IS4, OUT, ZX>;
    static int configured_smem = 0;   // per instantiation; max over calls is safe to keep
    if (configured_smem < static_cast<int>(pl.smem_bytes)) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                             227 * 1024);
        if (e != cudaSuccess) return cuda_fail(e);
        configured_smem = 227 * 1024;
    }
    cudaLaunchConfig_t cfg;
    std::memset(&cfg, 0, sizeof(cfg));
    cfg.gridDim = dim3(static_cast<unsigned>(pl.grid));
    cfg.blockDim = dim3(static_cast<unsigned>(pl.threads));
    cfg.dynamicSmemBytes = pl.smem_bytes;
    cfg.stream = stream;
    cudaLaunchAttribute pdl[1];
    set_pdl(cfg, pdl);
    qc::ConvParams cp = debug_params(pl.cp, stream);
    cudaError_t e = cudaLaunchKernelEx(&cfg, kern, xm, wm, ym, cp);
    if (e != cudaSuccess) return cuda_fail(e);
    debug_dump(cp, stream);
    return QC_OK;
}

template <bool IS4, int OUT>
qc_status launch_conv(const Plan &pl, const CUtensorMap &xm, const CUtensorMap &wm,
                      const CUtensorMap &ym, cudaStream_t stream) {
    return pl.cp.x_zero != 0 ? launch_conv_t<IS4, OUT, true>(pl, xm, wm, ym, stream)
                             : launch_conv_t<IS4, OUT, false>(pl, xm, wm, ym, stream);
}

// ------------------------------------------------------------------ CTA-pair im2col (experimental)
// The CTA-pair kernel (fwd2.cuh) runs im2col layers with R*S > 1 and a full N = 256 tile
// (measured faster there: res4/res5 3x3 -6 to -13 % at 4 and 8 bits; no gain for 1x1 layers,
// slower for N = 128 tiles).  QC_CTA2=1 forces it for every eligible layer (tests),
// QC_NO_CTA2=1 disables it.
bool make_plan2(const qconv_desc *d, const Geometry &g, const Plan &pl1, Plan *pl) {
    static const bool force = std::getenv("QC_CTA2") != nullptr;
    static const bool off = std::getenv("QC_NO_CTA2") != nullptr;
    if (off) return false;
    if (pl1.cp.pair || d->x_zero != 0 || d->y_t == QC_S32 || !pl1.cp.y_tma) return false;
    const int BN = pl1.BN;
    if (BN % 32 || BN < 64) return false;
    if (!force && !(BN == 256 && d->r * d->s > 1)) return false;
    *pl = pl1;
    qc::ConvParams &p = pl->cp;
    const bool is4 = g.bits == 4;
    const int m_tiles2 = static_cast<int>((g.M + 2 * qc::kBM - 1) / (2 * qc::kBM));
    pl->num_tiles = m_tiles2 * pl1.n_tiles_n;
    const uint32_t a_bytes = static_cast<uint32_t>(qc::kBM * pl1.BK);
    const uint32_t b_bytes = static_cast<uint32_t>(align_up(static_cast<size_t>(BN / 2) * pl1.BK, 1024));
    const uint32_t stg_bytes = is4 ? static_cast<uint32_t>(qc::kBM * pl1.bkp) : 0u;
    const uint32_t per_stage = a_bytes + b_bytes + stg_bytes;
    const uint32_t ystg_bytes = p.ystg_bytes;                 // one staging buffer (fwd2.cuh)
    const uint32_t fixed = static_cast<uint32_t>(qc::kMaxBN) * 16u + 128u + 1024u + ystg_bytes;
    int stages = static_cast<int>((227u * 1024u - 1024u - fixed) / per_stage);
    stages = std::min(stages, 24);
    if (stages < 2) return false;
    pl->stages = stages;
    p.stages = stages;
    p.num_tiles = pl->num_tiles;
    p.a_stage_bytes = a_bytes;
    p.b_stage_bytes = b_bytes;
    p.stg_stage_bytes = stg_bytes;
    p.off_a = 0;
    p.off_b = a_bytes * stages;
    p.off_stg = p.off_b + b_bytes * stages;
    p.off_ystg = static_cast<uint32_t>(align_up(p.off_stg + stg_bytes * stages, 1024));
    p.off_par = static_cast<uint32_t>(align_up(p.off_ystg + ystg_bytes, 16));
    p.off_bar = static_cast<uint32_t>(align_up(p.off_par + static_cast<uint32_t>(qc::kMaxBN) * 16u + 128u, 8));
    const uint32_t bar_bytes = static_cast<uint32_t>((4 * stages + 4) * 8 + 16);
    pl->smem_bytes = p.off_bar + bar_bytes + 1024u;
    if (pl->smem_bytes > 227u * 1024u) return false;
    p.idesc = qc::make_idesc_i8(2 * qc::kBM, static_cast<uint32_t>(BN), act_signed(d), dtype_signed(d->w_t));
    const int pairs = std::min(pl->num_tiles, num_sms() / 2);
    pl->grid = 2 * pairs;
    return true;
}

template <bool IS4, int OUT>
qc_status launch_fwd2(const Plan &pl, const CUtensorMap &xm, const CUtensorMap &wm, const CUtensorMap &ym,
                      cudaStream_t stream) {
    auto kern = qc::qconv_fwd2_kernel<IS4, OUT>;
    static int configured = 0;
    if (!configured) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
        if (e != cudaSuccess) return cuda_fail(e);
        configured = 1;
    }
    cudaLaunchConfig_t cfg;
    std::memset(&cfg, 0, sizeof(cfg));
    cfg.gridDim = dim3(static_cast<unsigned>(pl.grid));
    cfg.blockDim = dim3(static_cast<unsigned>(pl.threads));
    cfg.dynamicSmemBytes = pl.smem_bytes;
    cfg.stream = stream;
    cudaLaunchAttribute attr[2];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = 2;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    qc::ConvParams cp = debug_params(pl.cp, stream);
    cudaError_t e = cudaLaunchKernelEx(&cfg, kern, xm, wm, ym, cp);
    if (e != cudaSuccess) return cuda_fail(e);
    debug_dump(cp, stream);
    return QC_OK;
}

// ------------------------------------------------------------------ halo mode (stride 1)
bool halo_disabled() {
    static const bool off = std::getenv("QC_NO_HALO") != nullptr;
    return off;
}

// Decide whether the stride-1 halo kernel applies and fill its plan.
bool make_halo_plan(const qconv_desc *d, const Geometry &g, Plan *pl) {
    if (halo_disabled()) return false;
    if (d->stride_h != 1 || d->stride_w != 1 || d->dil_h != 1 || d->dil_w != 1) return false;
    if (d->x_zero != 0 || d->y_t == QC_S32) return false;
    const bool is4 = g.bits == 4;
    const int C8 = d->c;                                 // int8 bytes per pixel after widening
    const bool tap_pair = !is4 && C8 == 16;
    if (tap_pair) {
        if (d->s % 2) return false;
    } else if (C8 % 32) {
        return false;
    }
    const int Wh = d->w + 2 * d->pad_w;
    if (Wh > qc::kBM || Wh > 256) return false;
    if (d->r * d->s == 1) return false;                 // no tap reuse: the im2col GEMM path is better
    const int Rt = qc::kBM / Wh;
    const int tpi = (g.P + Rt - 1) / Rt;
    if (static_cast<double>(g.P) * g.Q / (static_cast<double>(tpi) * qc::kBM) < 0.7) return false;
    const int HR = Rt + d->r - 1;
    const int nplanes = C8 / 16;
    const int nch = g.c_bytes / 16;                      // TMA channel chunks (packed for 4-bit)
    if (nch < 1 || nch > 256 || HR > 256) return false;
    const int KG8 = d->r * d->s * C8;
    const int nK = KG8 / 16;
    if (nK > 256) return false;
    // N tile: largest of {round_up(K,32) <= 256, 128, 64, 32} whose weight slab fits in 100 KB
    // the whole weight slab stays resident (one N tile): MMA issue costs ~75 cycles per
    // instruction (measured), so narrower N tiles would be issue-bound
    if (d->k > 256) return false;
    const int BN = (d->k + 31) / 32 * 32;
    if (static_cast<int64_t>(BN) * KG8 > 100 * 1024) return false;
    const int ybits = dtype_bits(d->y_t);
    const int tile_row_bytes = BN * ybits / 8;
    const int y_gw = tile_row_bytes >= 128 ? 128 : tile_row_bytes;
    if (!((static_cast<int64_t>(d->k) * ybits / 8) % 16 == 0 &&
          (y_gw == 32 || y_gw == 64 || (y_gw == 128 && tile_row_bytes % 128 == 0))))
        return false;
    const int n_tiles_n = (d->k + BN - 1) / BN;
    const int tiles_per_img = (g.P + Rt - 1) / Rt;
    const int64_t num_tiles = static_cast<int64_t>(d->n) * tiles_per_img * n_tiles_n;
    if (num_tiles > INT32_MAX) return false;
    const uint32_t plane = static_cast<uint32_t>(HR * Wh * 16);
    const uint32_t hx = static_cast<uint32_t>(align_up(static_cast<size_t>(nplanes) * plane, 1024));
    const uint32_t hp = is4 ? static_cast<uint32_t>(align_up(static_cast<size_t>(nch) * plane, 1024)) : 0u;
    const uint32_t bres = static_cast<uint32_t>(align_up(static_cast<size_t>(BN) * KG8, 1024));
    const uint32_t ystg = 2u * 128u * static_cast<uint32_t>(tile_row_bytes);   // double-buffered
    const uint32_t fixed = bres + ystg + static_cast<uint32_t>(qc::kMaxBN) * 16u + 128u + 2048u +
                           8u * static_cast<uint32_t>(d->r * d->s * nplanes);
    if (fixed + 2 * (hx + hp) > 227u * 1024u) return false;
    int stages = static_cast<int>((227u * 1024u - fixed) / (hx + hp));
    stages = std::min(stages, 24);   // deep ring: the halo loads are latency-bound (~6 us each under load)
    qc::ConvParams &p = pl->cp;
    std::memset(&p, 0, sizeof(p));
    p.M = static_cast<int32_t>(g.M);
    p.P = g.P; p.Q = g.Q; p.PQ = g.P * g.Q; p.K = d->k;
    p.BN = BN; p.n_tiles_n = n_tiles_n; p.num_tiles = static_cast<int32_t>(num_tiles);
    p.S = d->s; p.R = d->r; p.H = d->h; p.W = d->w; p.C8 = C8;
    p.stride_h = p.stride_w = 1; p.dil_h = p.dil_w = 1; p.pad_h = d->pad_h; p.pad_w = d->pad_w;
    p.stages = stages;
    p.Wh = Wh; p.Rt = Rt; p.HR = HR; p.tiles_per_img = tiles_per_img; p.nplanes = nplanes;
    p.nk_planes = nK; p.tap_pair = tap_pair ? 1 : 0; p.h_plane_bytes = plane;
    p.off_bres = 0;
    p.b_res_bytes = static_cast<uint32_t>(BN) * static_cast<uint32_t>(KG8);
    p.off_hx = bres;
    p.hx_stage_bytes = hx;
    p.off_hp = bres + hx * stages;
    p.hp_stage_bytes = hp;
    p.halo_tx = static_cast<uint32_t>(nch) * plane;
    // whole-row loads when one box row (Wh pixels) fits the 256-element limit as int64s and the
    // staged layout works without planes: the C = 16 stem (one plane) or 4-bit inputs (the
    // converter re-lays the packed pixels into planes)
    p.c_px = g.c_bytes;
    p.halo_flat = ((tap_pair || is4) && (Wh * g.c_bytes) % 8 == 0 && Wh * g.c_bytes / 8 <= 256) ? 1 : 0;
    p.off_ystg = static_cast<uint32_t>(align_up(p.off_hp + hp * stages, 1024));
    p.ystg_bytes = ystg / 2;
    p.y_tma = 1;
    p.y_gw = y_gw;
    p.y_gmask = y_gw == 128 ? 7 : (y_gw == 64 ? 3 : 1);
    p.n_ygroups = tile_row_bytes / y_gw;
    p.off_par = static_cast<uint32_t>(align_up(p.off_ystg + ystg, 16));
    p.n_mma = tap_pair ? d->r * (d->s / 2) : d->r * d->s * (nplanes / 2);
    if (p.n_mma > qc::kHaloMaxMMA) return false;
    p.off_mtab = static_cast<uint32_t>(align_up(p.off_par + static_cast<uint32_t>(qc::kMaxBN) * 16u + 128u, 16));
    p.off_bar = static_cast<uint32_t>(align_up(p.off_mtab + 8u * static_cast<uint32_t>(p.n_mma), 8));
    const uint32_t bar_bytes = static_cast<uint32_t>((3 * stages + 9) * 8 + 16);
    pl->smem_bytes = p.off_bar + bar_bytes + 1024u;
    if (pl->smem_bytes > 227u * 1024u) return false;
    p.idesc = qc::make_idesc_i8(qc::kBM, static_cast<uint32_t>(BN), act_signed(d), dtype_signed(d->w_t));
    pl->tmem_cols = pow2_cols(2 * BN);
    p.tmem_cols = pl->tmem_cols;
    p.y_zero = d->y_zero; p.clamp_lo = d->clamp_lo; p.clamp_hi = d->clamp_hi; p.x_zero = 0;
    p.need_clamp = (d->clamp_lo > dtype_min(d->y_t) || d->clamp_hi < dtype_max(d->y_t)) ? 1 : 0;
    p.y_row_bytes = static_cast<int64_t>(d->k) * ybits / 8;
    const int sms = num_sms();
    int grid = std::min<int64_t>(num_tiles, sms / n_tiles_n * n_tiles_n);
    grid = std::max(grid / n_tiles_n * n_tiles_n, n_tiles_n);
    pl->grid = grid;
    pl->threads = is4 ? 512 : 384;
    pl->BN = BN;
    pl->n_tiles_n = n_tiles_n;
    pl->num_tiles = static_cast<int>(num_tiles);
    pl->stages = stages;
    return true;
}

qc_status encode_halo_maps(const qconv_desc *d, const Geometry &g, const qc::ConvParams &p,
                           const void *x, const void *w8, void *y, CUtensorMap *hm, CUtensorMap *bm,
                           CUtensorMap *ym) {
    const Driver &drv = driver();
    if (!drv.tiled) return cuda_fail(drv.err);
    const cuuint64_t cb = static_cast<cuuint64_t>(g.c_bytes);
    if (p.halo_flat) {   // input halo: [n][h][w * c_bytes / 8] int64 view of NHWC, whole rows
        cuuint64_t dims[3] = {static_cast<cuuint64_t>(d->w) * cb / 8, static_cast<cuuint64_t>(d->h),
                              static_cast<cuuint64_t>(d->n)};
        cuuint64_t strides[2] = {cb * d->w, cb * d->w * d->h};
        cuuint32_t box[3] = {static_cast<cuuint32_t>(p.Wh * cb / 8), static_cast<cuuint32_t>(p.HR), 1};
        cuuint32_t es[3] = {1, 1, 1};
        CUresult r = drv.tiled(hm, CU_TENSOR_MAP_DATA_TYPE_INT64, 3, const_cast<void *>(x), dims, strides,
                               box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                               CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        if (r != CUDA_SUCCESS) return cuda_fail(cudaErrorInvalidValue);
        small_tensor_fixup(hm, static_cast<uint64_t>(g.x_bytes));
    } else {   // input halo: [chunk][n][h][w][16 B] view of NHWC
        cuuint64_t dims[5] = {16, static_cast<cuuint64_t>(d->w), static_cast<cuuint64_t>(d->h),
                              static_cast<cuuint64_t>(d->n), cb / 16};
        cuuint64_t strides[4] = {cb, cb * d->w, cb * d->w * d->h, 16};
        cuuint32_t box[5] = {16, static_cast<cuuint32_t>(p.Wh), static_cast<cuuint32_t>(p.HR), 1,
                             static_cast<cuuint32_t>(cb / 16)};
        cuuint32_t es[5] = {1, 1, 1, 1, 1};
        CUresult r = drv.tiled(hm, CU_TENSOR_MAP_DATA_TYPE_UINT8, 5, const_cast<void *>(x), dims, strides,
                               box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                               CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        if (r != CUDA_SUCCESS) return cuda_fail(cudaErrorInvalidValue);
        small_tensor_fixup(hm, static_cast<uint64_t>(g.x_bytes));
    }
    {   // weights: [K-chunk][k][16 B] view of int8 KRSC
        const cuuint64_t kg = static_cast<cuuint64_t>(d->r) * d->s * d->c;
        cuuint64_t dims[3] = {16, static_cast<cuuint64_t>(d->k), kg / 16};
        cuuint64_t strides[2] = {kg, 16};
        cuuint32_t box[3] = {16, static_cast<cuuint32_t>(p.BN), static_cast<cuuint32_t>(kg / 16)};
        cuuint32_t es[3] = {1, 1, 1};
        CUresult r = drv.tiled(bm, CU_TENSOR_MAP_DATA_TYPE_UINT8, 3, const_cast<void *>(w8), dims, strides,
                               box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                               CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        if (r != CUDA_SUCCESS) return cuda_fail(cudaErrorInvalidValue);
        small_tensor_fixup(bm, static_cast<uint64_t>(g.w8_bytes));
    }
    {   // output: [n][p][q][k bytes], box [1][Rt][Q][y_gw]
        const int yb = dtype_bits(d->y_t);
        const cuuint64_t row = static_cast<cuuint64_t>(d->k) * yb / 8;
        cuuint64_t dims[4] = {row, static_cast<cuuint64_t>(g.Q), static_cast<cuuint64_t>(g.P),
                              static_cast<cuuint64_t>(d->n)};
        cuuint64_t strides[3] = {row, row * g.Q, row * g.Q * g.P};
        cuuint32_t box[4] = {static_cast<cuuint32_t>(p.y_gw), static_cast<cuuint32_t>(g.Q),
                             static_cast<cuuint32_t>(p.Rt), 1};
        cuuint32_t es[4] = {1, 1, 1, 1};
        CUresult r = drv.tiled(ym, CU_TENSOR_MAP_DATA_TYPE_UINT8, 4, y, dims, strides, box, es,
                               CU_TENSOR_MAP_INTERLEAVE_NONE, swizzle_for(p.y_gw),
                               CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        if (r != CUDA_SUCCESS) return cuda_fail(cudaErrorInvalidValue);
        small_tensor_fixup(ym, static_cast<uint64_t>(g.y_bytes));
    }
    return QC_OK;
}

template <bool IS4, int OUT>
qc_status launch_halo(const Plan &pl, const CUtensorMap &hm, const CUtensorMap &bm,
                      const CUtensorMap &ym, cudaStream_t stream) {
    auto kern = qc::qconv_halo_kernel<IS4, OUT>;
    static int configured = 0;
    if (!configured) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
        if (e != cudaSuccess) return cuda_fail(e);
        configured = 1;
    }
    cudaLaunchConfig_t cfg;
    std::memset(&cfg, 0, sizeof(cfg));
    cfg.gridDim = dim3(static_cast<unsigned>(pl.grid));
    cfg.blockDim = dim3(static_cast<unsigned>(pl.threads));
    cfg.dynamicSmemBytes = pl.smem_bytes;
    cfg.stream = stream;
    cudaLaunchAttribute pdl[1];
    set_pdl(cfg, pdl);
    qc::ConvParams cp = debug_params(pl.cp, stream);
    cudaError_t e = cudaLaunchKernelEx(&cfg, kern, hm, bm, ym, cp);
    if (e != cudaSuccess) return cuda_fail(e);
    debug_dump(cp, stream);
    return QC_OK;
}

// ------------------------------------------------------------------ channel-major 1x1 kernel
bool trans_disabled() {
    static const bool off = std::getenv("QC_NO_TRANS") != nullptr;
    return off;
}

bool make_trans_plan(const qconv_desc *d, const Geometry &g, Plan *pl) {
    if (trans_disabled()) return false;
    if (d->r != 1 || d->s != 1 || d->x_zero != 0 || d->y_t == QC_S32) return false;
    if (d->c % 32 || d->k % 64) return false;
    const bool is4 = g.bits == 4;
    // With 4-bit activations the 256-pixel operand tile doubles the on-chip widening per
    // MAC; for deep inputs (C > 512) that outweighs the cheaper epilogue (measured, r1).
    if (is4 && d->c > 512) return false;
    const int ybits = dtype_bits(d->y_t);
    if ((static_cast<int64_t>(d->k) * ybits / 8) % 16) return false;
    const int BMc = d->k % 128 == 0 ? 128 : 64;
    const int BNp = 256;
    const int BK = choose_bk(d->c);
    const int bkp = is4 ? BK / 2 : BK;
    const int n_tiles_n = d->k / BMc;
    const int64_t m_tiles = (g.M + BNp - 1) / BNp;
    const int64_t num_tiles = m_tiles * n_tiles_n;
    if (num_tiles > INT32_MAX) return false;
    const int row_bytes = BMc * ybits / 8;                 // 32 .. 128
    const uint32_t ystg_one = static_cast<uint32_t>(BNp * row_bytes);
    const uint32_t a_bytes = static_cast<uint32_t>(BNp * BK);      // activations
    const uint32_t b_bytes = static_cast<uint32_t>(BMc * BK);      // weights
    const uint32_t stg_bytes = is4 ? static_cast<uint32_t>(BNp * bkp) : 0u;
    const uint32_t per_stage = a_bytes + b_bytes + stg_bytes;
    const uint32_t fixed = 2u * ystg_one + 2048u;
    if (fixed + 2 * per_stage > 227u * 1024u) return false;
    int stages = std::min(static_cast<int>((227u * 1024u - fixed) / per_stage), 16);
    qc::ConvParams &p = pl->cp;
    std::memset(&p, 0, sizeof(p));
    p.M = static_cast<int32_t>(g.M);
    p.P = g.P; p.Q = g.Q; p.PQ = g.P * g.Q; p.K = d->k;
    p.BN = BMc;                  // channels per tile (UMMA M)
    p.Wh = BNp;                  // pixels per tile (UMMA N)
    p.n_tiles_n = n_tiles_n;
    p.num_tiles = static_cast<int32_t>(num_tiles);
    p.chunks = d->c / BK;
    p.num_kb = p.chunks;
    p.S = 1; p.R = 1; p.H = d->h; p.W = d->w; p.C8 = d->c;
    p.stride_h = d->stride_h; p.stride_w = d->stride_w; p.pad_h = d->pad_h; p.pad_w = d->pad_w;
    p.dil_h = p.dil_w = 1;
    p.BK = BK; p.bkp = bkp; p.stages = stages;
    p.sw_layout = BK == 128 ? 2 : (BK == 64 ? 4 : 6);
    p.sw_mask = BK == 128 ? 7 : (BK == 64 ? 3 : 1);
    p.cvt_shift = bkp >= 64 ? 2 : (bkp >= 32 ? 1 : 0);
    p.off_a = 0;
    p.a_stage_bytes = a_bytes;
    p.off_b = a_bytes * stages;
    p.b_stage_bytes = b_bytes;
    p.off_stg = p.off_b + b_bytes * stages;
    p.stg_stage_bytes = stg_bytes;
    p.off_ystg = static_cast<uint32_t>(align_up(p.off_stg + stg_bytes * stages, 1024));
    p.ystg_bytes = ystg_one;
    p.y_tma = 1;
    p.y_gw = row_bytes;
    p.y_gmask = row_bytes >= 128 ? 7 : (row_bytes == 64 ? 3 : 1);   // staging swizzled like the TMA store
    p.n_ygroups = 1;
    p.off_par = static_cast<uint32_t>(align_up(p.off_ystg + 2u * ystg_one, 16));
    p.off_bar = static_cast<uint32_t>(align_up(p.off_par, 8));
    const uint32_t bar_bytes = static_cast<uint32_t>((3 * stages + 8) * 8 + 16);
    pl->smem_bytes = p.off_bar + bar_bytes + 1024u;
    if (pl->smem_bytes > 227u * 1024u) return false;
    p.idesc = qc::make_idesc_i8(static_cast<uint32_t>(BMc), static_cast<uint32_t>(BNp),
                                dtype_signed(d->w_t), act_signed(d));
    pl->tmem_cols = pow2_cols(2 * BNp);
    p.tmem_cols = pl->tmem_cols;
    p.y_zero = d->y_zero; p.clamp_lo = d->clamp_lo; p.clamp_hi = d->clamp_hi;
    p.need_clamp = (d->clamp_lo > dtype_min(d->y_t) || d->clamp_hi < dtype_max(d->y_t)) ? 1 : 0;
    p.y_row_bytes = static_cast<int64_t>(d->k) * ybits / 8;
    const int sms = num_sms();
    int grid = static_cast<int>(std::min<int64_t>(num_tiles, sms / n_tiles_n * n_tiles_n));
    grid = std::max(grid, 1);
    pl->grid = grid;
    pl->threads = is4 ? qc::kTThreads4 : qc::kTThreads8;
    pl->BK = BK; pl->bkp = bkp; pl->BN = BMc; pl->n_tiles_n = n_tiles_n;
    pl->num_tiles = static_cast<int>(num_tiles); pl->stages = stages; pl->chunks = p.chunks;
    pl->num_kb = p.num_kb;
    return true;
}

template <bool IS4, int OUT, bool M64>
qc_status launch_trans_m(const Plan &pl, const CUtensorMap &xm, const CUtensorMap &wm,
                         const CUtensorMap &ym, cudaStream_t stream) {
    auto kern = qc::qconv_t_kernel<IS4, OUT, M64>;
    static int configured = 0;
    if (!configured) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
        if (e != cudaSuccess) return cuda_fail(e);
        configured = 1;
    }
    cudaLaunchConfig_t cfg;
    std::memset(&cfg, 0, sizeof(cfg));
    cfg.gridDim = dim3(static_cast<unsigned>(pl.grid));
    cfg.blockDim = dim3(static_cast<unsigned>(pl.threads));
    cfg.dynamicSmemBytes = pl.smem_bytes;
    cfg.stream = stream;
    cudaLaunchAttribute pdl[1];
    set_pdl(cfg, pdl);
    qc::ConvParams cp = debug_params(pl.cp, stream);
    cudaError_t e = cudaLaunchKernelEx(&cfg, kern, xm, wm, ym, cp);
    if (e != cudaSuccess) return cuda_fail(e);
    debug_dump(cp, stream);
    return QC_OK;
}

template <bool IS4, int OUT>
qc_status launch_trans(const Plan &pl, const CUtensorMap &xm, const CUtensorMap &wm,
                       const CUtensorMap &ym, cudaStream_t stream) {
    return pl.BN == 64 ? launch_trans_m<IS4, OUT, true>(pl, xm, wm, ym, stream)
                       : launch_trans_m<IS4, OUT, false>(pl, xm, wm, ym, stream);
}

}  // namespace

// ====================================================================== C ABI
extern "C" {

const char *qconv_status_string(qc_status s) {
    switch (s) {
        case QC_OK: return "ok";
        case QC_ERR_INVALID_ARG: return "invalid argument";
        case QC_ERR_UNSUPPORTED: return "unsupported configuration";
        case QC_ERR_OVERFLOW_RISK: return "int32 accumulator overflow risk";
        case QC_ERR_MISALIGNED: return "device pointer not 16-byte aligned";
        case QC_ERR_WORKSPACE: return "workspace missing or too small";
        case QC_ERR_CUDA: return "CUDA error";
    }
    return "unknown status";
}

int qconv_last_cuda_error(void) { return g_last_cuda_error; }
int qconv_version(void) { return 100; }

qc_status qconv_requant_params(float in_scale, const float *w_scale, float out_scale, int32_t k,
                               int32_t *multiplier, int32_t *shift) {
    if (!w_scale || !multiplier || !shift || k < 1) return QC_ERR_INVALID_ARG;
    if (!(in_scale > 0.0f) || !(out_scale > 0.0f) || !std::isfinite(in_scale) ||
        !std::isfinite(out_scale))
        return QC_ERR_INVALID_ARG;
    for (int32_t i = 0; i < k; ++i) {
        const float ws = w_scale[i];
        if (!(ws >= 0.0f) || !std::isfinite(ws)) return QC_ERR_INVALID_ARG;
        // exact product of two binary32 values in binary64, then one RNE division
        const double M = (static_cast<double>(in_scale) * static_cast<double>(ws)) /
                         static_cast<double>(out_scale);
        if (M == 0.0) {
            multiplier[i] = 0;
            shift[i] = 31;
            continue;
        }
        int e = 0;
        const double f = std::frexp(M, &e);                   // M = f * 2^e, f in [0.5, 1)
        const double scaled = std::ldexp(f, 31);              // exact
        int64_t m = static_cast<int64_t>(scaled);             // floor (scaled > 0)
        if (scaled - static_cast<double>(m) >= 0.5) m += 1;   // round half up
        if (m == (int64_t(1) << 31)) {
            m = int64_t(1) << 30;
            e += 1;
        }
        const int n = 31 - e;
        if (n < 1 || n > 62) return QC_ERR_INVALID_ARG;
        multiplier[i] = static_cast<int32_t>(m);
        shift[i] = n;
    }
    return QC_OK;
}

qc_status qconv_quantize_pack(const void *x, qc_ftype xt, int64_t npix, int32_t c, int32_t c_pad,
                              float scale, int32_t zero_point, qc_dtype yt, void *y, void *stream) {
    if (!x || !y || npix < 0 || c < 1 || c_pad < c) return QC_ERR_INVALID_ARG;
    if (xt != QC_F32 && xt != QC_BF16) return QC_ERR_INVALID_ARG;
    if (!is_int_input(yt)) return QC_ERR_INVALID_ARG;
    if (!(scale > 0.0f) || !std::isfinite(scale)) return QC_ERR_INVALID_ARG;
    if (zero_point < dtype_min(yt) || zero_point > dtype_max(yt)) return QC_ERR_INVALID_ARG;
    const int bits = dtype_bits(yt);
    if (bits == 4 && (c_pad % 2)) return QC_ERR_INVALID_ARG;
    if (!aligned16(x) || !aligned16(y)) return QC_ERR_MISALIGNED;
    if (npix == 0) return QC_OK;
    qc::QuantParams p;
    p.x = x;
    p.y = y;
    p.npix = npix;
    p.c = c;
    p.c_pad = c_pad;
    p.inv_s = 1.0f / scale;
    p.z = zero_point;
    p.qmin = static_cast<int32_t>(dtype_min(yt));
    p.qmax = static_cast<int32_t>(dtype_max(yt));
    p.flo = static_cast<float>(p.qmin - p.z - 1);
    p.fhi = static_cast<float>(p.qmax - p.z + 1);
    p.bf16 = xt == QC_BF16;
    p.bits = bits;
    p.fast = (c == c_pad) && (c % 16 == 0);
    const int64_t groups = (npix * c_pad + 15) / 16;
    const int64_t blocks_needed = (groups + 255) / 256;
    const int grid = static_cast<int>(std::min<int64_t>(blocks_needed, static_cast<int64_t>(num_sms()) * 8));
    qc::quantize_pack_kernel<<<grid, 256, 0, static_cast<cudaStream_t>(stream)>>>(p);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e);
    return QC_OK;
}

// Prepared weights: int8 KRSC (8-bit: the codes as they are; 4-bit: nibble-plane order,
// prep.cuh widen_w4_kernel), then for 4-bit a 16-byte aligned int32 wsum[K].
static size_t prepared_bytes(const qconv_desc *d, const Geometry &g) {
    if (dtype_bits(d->w_t) == 8) return static_cast<size_t>(g.w8_bytes);
    return align_up(static_cast<size_t>(g.w8_bytes), 16) + 4 * static_cast<size_t>(d->k);
}
static const int32_t *prepared_wsum(const qconv_desc *d, const Geometry &g, const void *w8) {
    if (dtype_bits(d->w_t) != 4) return nullptr;
    return reinterpret_cast<const int32_t *>(static_cast<const uint8_t *>(w8) +
                                             align_up(static_cast<size_t>(g.w8_bytes), 16));
}

size_t qconv_prepared_weight_bytes(const qconv_desc *d) {
    Geometry g;
    if (validate_desc(d, &g) != QC_OK) return 0;
    return prepared_bytes(d, g);
}

static qc_status prepare_weights_impl(const qconv_desc *d, const Geometry &g, const void *w,
                                      void *w_prep, cudaStream_t st) {
    if (dtype_bits(d->w_t) == 8) {
        cudaError_t e = cudaMemcpyAsync(w_prep, w, static_cast<size_t>(g.w8_bytes),
                                        cudaMemcpyDeviceToDevice, st);
        if (e != cudaSuccess) return cuda_fail(e);
        return QC_OK;
    }
    if (d->c % 32) return QC_ERR_UNSUPPORTED;            // nibble planes are 32-channel groups
    const int64_t ngroups = g.w_bytes / 16;
    const int grid = static_cast<int>(std::min<int64_t>((ngroups + 255) / 256, 4096));
    const int sgn = d->w_t == QC_S4 ? 1 : 0;
    qc::widen_w4_kernel<<<grid, 256, 0, st>>>(static_cast<const uint8_t *>(w),
                                              static_cast<int8_t *>(w_prep), ngroups, sgn);
    qc::wsum_w4_kernel<<<d->k, 256, 0, st>>>(
        static_cast<const uint8_t *>(w), const_cast<int32_t *>(prepared_wsum(d, g, w_prep)),
        static_cast<int64_t>(d->r) * d->s * d->c / 2, sgn);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e);
    return QC_OK;
}

qc_status qconv_prepare_weights(const qconv_desc *d, const void *w, void *w_prep, void *stream) {
    Geometry g;
    qc_status s = validate_desc(d, &g);
    if (s != QC_OK) return s;
    if (!w || !w_prep) return QC_ERR_INVALID_ARG;
    if (!aligned16(w) || !aligned16(w_prep)) return QC_ERR_MISALIGNED;
    return prepare_weights_impl(d, g, w, w_prep, static_cast<cudaStream_t>(stream));
}

static size_t ws_weights_bytes(const qconv_desc *d, const Geometry &g) {
    return (dtype_bits(d->w_t) == 4 && !d->w_prepared) ? align_up(prepared_bytes(d, g), 256) : 0;
}
static size_t ws_zx_bytes(const qconv_desc *d) {
    return d->x_zero != 0 ? align_up(static_cast<size_t>(d->k) * (d->r + 1) * (d->s + 1) * 4, 256) : 0;
}

size_t qconv2d_workspace_size(const qconv_desc *d) {
    Geometry g;
    if (validate_desc(d, &g) != QC_OK) return 0;
    return ws_weights_bytes(d, g) + ws_zx_bytes(d);
}

// Accumulator scale and signed-offset correction of 4-bit activations (widen_word).
static void set_act_params(const qconv_desc *d, const Geometry &g, const void *w8, qc::ConvParams &p) {
    p.acc_lg = g.bits == 4 ? 4 : 0;
    p.x_sgn4 = (g.bits == 4 && d->x_t == QC_S4) ? 1 : 0;
    p.wsum = p.x_sgn4 ? prepared_wsum(d, g, w8) : nullptr;
}

qc_status qconv2d_forward(const qconv_desc *d, const void *x, const void *w, const int32_t *bias,
                          const int32_t *multiplier, const int32_t *shift, void *y, void *workspace,
                          size_t ws_bytes, void *stream) {
    Geometry g;
    qc_status s = validate_desc(d, &g);
    if (s != QC_OK) return s;
    if (!x || !w || !y) return QC_ERR_INVALID_ARG;
    if (d->y_t != QC_S32 && (!multiplier || !shift)) return QC_ERR_INVALID_ARG;
    s = check_supported(d, g);
    if (s != QC_OK) return s;
    if (!aligned16(x) || !aligned16(w) || !aligned16(y) || (bias && !aligned16(bias)) ||
        (multiplier && !aligned16(multiplier)) || (shift && !aligned16(shift)) ||
        (workspace && !aligned16(workspace)))
        return QC_ERR_MISALIGNED;
    const size_t need_w = ws_weights_bytes(d, g), need_z = ws_zx_bytes(d);
    if (need_w + need_z > 0 && (!workspace || ws_bytes < need_w + need_z)) return QC_ERR_WORKSPACE;
    cudaStream_t st = static_cast<cudaStream_t>(stream);

    Plan pl;
    s = make_plan(d, g, &pl);
    if (s != QC_OK) return s;

    const void *w8 = w;
    if (need_w) {
        s = prepare_weights_impl(d, g, w, workspace, st);
        if (s != QC_OK) return s;
        w8 = workspace;
    }
    {   // stride-1 convolutions: halo kernel (one tiled TMA per tile, resident weights)
        Plan hp;
        if (need_z == 0 && make_halo_plan(d, g, &hp)) {
            set_act_params(d, g, w8, hp.cp);
            hp.cp.w_early = need_w == 0 ? 1 : 0;
            hp.cp.bias = bias;
            hp.cp.mult = multiplier;
            hp.cp.shift = shift;
            hp.cp.y = y;
            alignas(64) CUtensorMap hm, bm, ym;
            s = encode_halo_maps(d, g, hp.cp, x, w8, y, &hm, &bm, &ym);
            if (s != QC_OK) return s;
            const bool is4 = g.bits == 4;
            switch (d->y_t) {
                case QC_U8: return is4 ? launch_halo<true, qc::OUT_U8>(hp, hm, bm, ym, st) : launch_halo<false, qc::OUT_U8>(hp, hm, bm, ym, st);
                case QC_S8: return is4 ? launch_halo<true, qc::OUT_S8>(hp, hm, bm, ym, st) : launch_halo<false, qc::OUT_S8>(hp, hm, bm, ym, st);
                case QC_U4: return is4 ? launch_halo<true, qc::OUT_U4>(hp, hm, bm, ym, st) : launch_halo<false, qc::OUT_U4>(hp, hm, bm, ym, st);
                case QC_S4: return is4 ? launch_halo<true, qc::OUT_S4>(hp, hm, bm, ym, st) : launch_halo<false, qc::OUT_S4>(hp, hm, bm, ym, st);
                default: break;
            }
        }
    }
    {   // 1x1 convolutions: channel-major kernel (per-channel constants in registers)
        Plan tp;
        if (need_z == 0 && make_trans_plan(d, g, &tp)) {
            set_act_params(d, g, w8, tp.cp);
            tp.cp.bias = bias;
            tp.cp.mult = multiplier;
            tp.cp.shift = shift;
            tp.cp.y = y;
            alignas(64) CUtensorMap xm, wm, ym;
            tp.cp.stg_sw = g.bits == 4 ? packed_sw_mask(tp.bkp) : 0;
            s = encode_x_map(d, g, x, tp.bkp, g.bits == 4 ? packed_swizzle(tp.bkp) : swizzle_for(tp.BK), &xm,
                             tp.cp.Wh);
            if (s != QC_OK) return s;
            s = encode_w_map_pairs(d, g, w8, tp.BK, tp.BN, swizzle_for(tp.BK), &wm);
            if (s != QC_OK) return s;
            s = encode_y_map(d, g, y, tp.cp.y_gw, &ym, tp.cp.Wh, true);
            if (s != QC_OK) return s;
            const bool is4 = g.bits == 4;
            switch (d->y_t) {
                case QC_U8: return is4 ? launch_trans<true, qc::OUT_U8>(tp, xm, wm, ym, st) : launch_trans<false, qc::OUT_U8>(tp, xm, wm, ym, st);
                case QC_S8: return is4 ? launch_trans<true, qc::OUT_S8>(tp, xm, wm, ym, st) : launch_trans<false, qc::OUT_S8>(tp, xm, wm, ym, st);
                case QC_U4: return is4 ? launch_trans<true, qc::OUT_U4>(tp, xm, wm, ym, st) : launch_trans<false, qc::OUT_U4>(tp, xm, wm, ym, st);
                case QC_S4: return is4 ? launch_trans<true, qc::OUT_S4>(tp, xm, wm, ym, st) : launch_trans<false, qc::OUT_S4>(tp, xm, wm, ym, st);
                default: break;
            }
        }
    }
    qc::ConvParams &p = pl.cp;
    set_act_params(d, g, w8, p);
    if (need_z) {
        int32_t *table = reinterpret_cast<int32_t *>(static_cast<uint8_t *>(workspace) + need_w);
        qc::zx_table_kernel<<<(d->k + 127) / 128, 128, 0, st>>>(
            static_cast<const int8_t *>(w8), table, d->k, d->r, d->s, d->c, dtype_signed(d->w_t) ? 0 : 1,
            g.bits == 4 ? 1 : 0);
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return cuda_fail(e);
        p.zx_table = table;
    }
    p.bias = bias;
    p.mult = multiplier;
    p.shift = shift;
    p.y = y;

    alignas(64) CUtensorMap xm, wm;
    const bool pair = p.pair != 0;
    p.stg_sw = g.bits == 4 ? packed_sw_mask(pl.bkp) : 0;
    s = encode_x_map(d, g, x, pl.bkp,
                     pair ? CU_TENSOR_MAP_SWIZZLE_NONE : (g.bits == 4 ? packed_swizzle(pl.bkp) : swizzle_for(pl.BK)),
                     &xm);
    if (s != QC_OK) return s;
    s = encode_w_map(d, g, w8, pair ? 16 : pl.BK, pl.BN,
                     pair ? CU_TENSOR_MAP_SWIZZLE_NONE : swizzle_for(pl.BK), &wm);
    if (s != QC_OK) return s;

    alignas(64) CUtensorMap ym;
    std::memset(&ym, 0, sizeof(ym));
    if (p.y_tma) {
        s = encode_y_map(d, g, y, p.y_gw, &ym);
        if (s != QC_OK) return s;
    }
    const bool is4 = g.bits == 4;
    {
        Plan p2;
        if (make_plan2(d, g, pl, &p2)) {
            p2.cp.bias = bias; p2.cp.mult = multiplier; p2.cp.shift = shift; p2.cp.y = y;
            alignas(64) CUtensorMap wm2;
            s = encode_w_map(d, g, w8, pl.BK, pl.BN / 2, swizzle_for(pl.BK), &wm2);
            if (s != QC_OK) return s;
            switch (d->y_t) {
                case QC_U8: return is4 ? launch_fwd2<true, qc::OUT_U8>(p2, xm, wm2, ym, st) : launch_fwd2<false, qc::OUT_U8>(p2, xm, wm2, ym, st);
                case QC_S8: return is4 ? launch_fwd2<true, qc::OUT_S8>(p2, xm, wm2, ym, st) : launch_fwd2<false, qc::OUT_S8>(p2, xm, wm2, ym, st);
                case QC_U4: return is4 ? launch_fwd2<true, qc::OUT_U4>(p2, xm, wm2, ym, st) : launch_fwd2<false, qc::OUT_U4>(p2, xm, wm2, ym, st);
                case QC_S4: return is4 ? launch_fwd2<true, qc::OUT_S4>(p2, xm, wm2, ym, st) : launch_fwd2<false, qc::OUT_S4>(p2, xm, wm2, ym, st);
                default: break;
            }
        }
    }
    switch (d->y_t) {
        case QC_S32: return is4 ? launch_conv<true, qc::OUT_S32>(pl, xm, wm, ym, st) : launch_conv<false, qc::OUT_S32>(pl, xm, wm, ym, st);
        case QC_U8: return is4 ? launch_conv<true, qc::OUT_U8>(pl, xm, wm, ym, st) : launch_conv<false, qc::OUT_U8>(pl, xm, wm, ym, st);
        case QC_S8: return is4 ? launch_conv<true, qc::OUT_S8>(pl, xm, wm, ym, st) : launch_conv<false, qc::OUT_S8>(pl, xm, wm, ym, st);
        case QC_U4: return is4 ? launch_conv<true, qc::OUT_U4>(pl, xm, wm, ym, st) : launch_conv<false, qc::OUT_U4>(pl, xm, wm, ym, st);
        case QC_S4: return is4 ? launch_conv<true, qc::OUT_S4>(pl, xm, wm, ym, st) : launch_conv<false, qc::OUT_S4>(pl, xm, wm, ym, st);
    }
    return QC_ERR_INVALID_ARG;
}

// ------------------------------------------------------------------ space-to-depth stem
static int32_t s2d_channels(int32_t c) {
    const int32_t c4 = 4 * c;
    return c4 <= 16 ? 16 : (c4 + 31) / 32 * 32;
}
static qc_dtype byte_container(qc_dtype t) {
    return (t == QC_U4 || t == QC_U8) ? QC_U8 : QC_S8;
}

qc_status qconv_s2d_desc(const qconv_desc *d, qconv_desc *out) {
    if (!d) return QC_ERR_INVALID_ARG;
    // the original activations are float (quantized by qconv_quantize_pack_s2d), so an odd c
    // with a 4-bit code type is fine: validate the byte-container view
    qconv_desc dv = *d;
    dv.x_t = byte_container(d->x_t);
    Geometry g;
    qc_status s = validate_desc(&dv, &g);
    if (s != QC_OK) return s;
    if (!is_int_input(d->x_t) || d->x_zero < dtype_min(d->x_t) || d->x_zero > dtype_max(d->x_t))
        return QC_ERR_INVALID_ARG;
    if (!out) return QC_ERR_INVALID_ARG;
    if (d->stride_h != 2 || d->stride_w != 2 || d->dil_h != 1 || d->dil_w != 1)
        return QC_ERR_UNSUPPORTED;
    qconv_desc o = *d;
    o.r = (d->r + 1) / 2;
    o.s = (d->s + 1) / 2;
    o.h = g.P + o.r - 1;
    o.w = g.Q + o.s - 1;
    o.c = s2d_channels(d->c);
    o.stride_h = o.stride_w = 1;
    o.pad_h = o.pad_w = 0;
    o.dil_h = o.dil_w = 1;
    o.x_t = byte_container(d->x_t);
    o.w_t = byte_container(d->w_t);
    o.w_prepared = 1;
    *out = o;
    return QC_OK;
}

qc_status qconv_quantize_pack_s2d(const qconv_desc *d, const void *x, qc_ftype xt, float scale,
                                  void *y, void *stream) {
    qconv_desc o;
    qc_status s = qconv_s2d_desc(d, &o);
    if (s != QC_OK) return s;
    if (!x || !y || (xt != QC_F32 && xt != QC_BF16)) return QC_ERR_INVALID_ARG;
    if (!(scale > 0.0f) || !std::isfinite(scale)) return QC_ERR_INVALID_ARG;
    if (!aligned16(x) || !aligned16(y)) return QC_ERR_MISALIGNED;
    qc::QuantS2DParams p;
    p.x = x;
    p.y = static_cast<uint8_t *>(y);
    p.n = d->n; p.h = d->h; p.w = d->w; p.c = d->c;
    p.hs = o.h; p.ws = o.w; p.cs = o.c;
    p.pad_h = d->pad_h; p.pad_w = d->pad_w;
    p.inv_s = 1.0f / scale;
    p.z = d->x_zero;
    p.qmin = static_cast<int32_t>(dtype_min(d->x_t));
    p.qmax = static_cast<int32_t>(dtype_max(d->x_t));
    p.flo = static_cast<float>(p.qmin - p.z - 1);
    p.fhi = static_cast<float>(p.qmax - p.z + 1);
    p.bf16 = xt == QC_BF16;
    {
        const int64_t total = static_cast<int64_t>(p.n) * p.hs * p.ws;
        const int grid = static_cast<int>(std::min<int64_t>((total + 255) / 256, static_cast<int64_t>(num_sms()) * 32));
        if (p.c == 3)
            qc::quantize_s2d_kernel<3><<<grid, 256, 0, static_cast<cudaStream_t>(stream)>>>(p);
        else
            qc::quantize_s2d_kernel<0><<<grid, 256, 0, static_cast<cudaStream_t>(stream)>>>(p);
    }
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e);
    return QC_OK;
}

size_t qconv_prepared_weight_bytes_s2d(const qconv_desc *d) {
    qconv_desc o;
    if (qconv_s2d_desc(d, &o) != QC_OK) return 0;
    return static_cast<size_t>(o.k) * o.r * o.s * o.c;
}

qc_status qconv_prepare_weights_s2d(const qconv_desc *d, const void *w, void *w_prep, void *stream) {
    qconv_desc o;
    qc_status s = qconv_s2d_desc(d, &o);
    if (s != QC_OK) return s;
    if (!w || !w_prep) return QC_ERR_INVALID_ARG;
    if (!aligned16(w) || !aligned16(w_prep)) return QC_ERR_MISALIGNED;
    const int64_t total = static_cast<int64_t>(o.k) * o.r * o.s * o.c;
    const int grid = static_cast<int>(std::min<int64_t>((total + 255) / 256, 4096));
    qc::weights_s2d_kernel<<<grid, 256, 0, static_cast<cudaStream_t>(stream)>>>(
        static_cast<const uint8_t *>(w), static_cast<int8_t *>(w_prep), d->k, d->r, d->s, d->c, o.r,
        o.s, o.c, dtype_bits(d->w_t), dtype_signed(d->w_t) ? 1 : 0);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e);
    return QC_OK;
}

qc_status qconv_debug_im2col_tile(const qconv_desc *d, const void *x, int64_t m0, int32_t r,
                                  int32_t s_, int32_t c_byte, int32_t box_bytes, void *out,
                                  void *stream) {
    Geometry g;
    qc_status s = validate_desc(d, &g);
    if (s != QC_OK) return s;
    if (!x || !out || m0 < 0 || m0 >= g.M || r < 0 || r >= d->r || s_ < 0 || s_ >= d->s ||
        box_bytes < 16 || box_bytes > 256 || box_bytes % 16 || c_byte < 0 ||
        c_byte + box_bytes > g.c_bytes)
        return QC_ERR_INVALID_ARG;
    if (g.c_bytes % 16) return QC_ERR_UNSUPPORTED;
    alignas(64) CUtensorMap xm;
    s = encode_x_map(d, g, x, box_bytes, CU_TENSOR_MAP_SWIZZLE_NONE, &xm);
    if (s != QC_OK) return s;
    const int64_t PQ = static_cast<int64_t>(g.P) * g.Q;
    const int img = static_cast<int>(m0 / PQ);
    const int64_t rem = m0 - img * PQ;
    const int p0 = static_cast<int>(rem / g.Q), q0 = static_cast<int>(rem % g.Q);
    const uint32_t bytes = static_cast<uint32_t>(qc::kBM * box_bytes);
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    cudaError_t e = cudaFuncSetAttribute(qc::qconv_debug_im2col_kernel,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024);
    if (e != cudaSuccess) return cuda_fail(e);
    qc::qconv_debug_im2col_kernel<<<1, 128, bytes + 1024, st>>>(
        xm, c_byte, q0 * d->stride_w - d->pad_w, p0 * d->stride_h - d->pad_h, img,
        static_cast<uint16_t>(s_ * d->dil_w), static_cast<uint16_t>(r * d->dil_h), bytes,
        static_cast<uint8_t *>(out));
    e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e);
    return QC_OK;
}

}  // extern "C"
