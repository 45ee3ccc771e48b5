// qconv.cu -- host side of libqconv.so: the C ABI declared in include/qconv.h.
//
// Validation, the overflow bound, the rewrite of a descriptor into the form the kernels
// take ("exec" descriptor: channel padding / space-to-depth for channel counts the kernels
// cannot take directly), the per-shape launch plan (kernel family, tile sizes, pipeline
// depth, shared-memory carve-up) with the tuning hooks of the paper's profile-run search
// (P:L271-273), TMA descriptor encoding and kernel launches (launch.h, k_*.cu).  All device
// work is in conv_fwd.cuh / halo.cuh / trans.cuh / fwd2.cuh / prep.cuh.  Nothing here
// allocates device memory.
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <mutex>
#include <string>
#include <vector>

#include "qconv.h"
#include "launch.h"
#include "prep.cuh"

#ifndef QC_MAX_YSTG
#define QC_MAX_YSTG 4
#endif

namespace {

thread_local int g_last_cuda_error = 0;

qc_status cuda_fail(cudaError_t e) {
    g_last_cuda_error = static_cast<int>(e);
    return QC_ERR_CUDA;
}

bool is_int_input(qc_dtype t) { return t == QC_U4 || t == QC_S4 || t == QC_U8 || t == QC_S8; }
bool is_float_out(qc_dtype t) { return t == QC_F32_OUT || t == QC_BF16_OUT; }
bool is_packed_out(qc_dtype t) { return is_int_input(t); }
int dtype_bits(qc_dtype t) {
    switch (t) {
        case QC_U4: case QC_S4: return 4;
        case QC_U8: case QC_S8: return 8;
        case QC_BF16_OUT: return 16;
        default: return 32;
    }
}
bool dtype_signed(qc_dtype t) { return t != QC_U4 && t != QC_U8; }
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
int out_kind(qc_dtype t) {
    switch (t) {
        case QC_U8: return qc::OUT_U8;
        case QC_S8: return qc::OUT_S8;
        case QC_U4: return qc::OUT_U4;
        case QC_S4: return qc::OUT_S4;
        case QC_F32_OUT: return qc::OUT_F32;
        case QC_BF16_OUT: return qc::OUT_BF16;
        default: return qc::OUT_S32;
    }
}
qc_dtype byte_container(qc_dtype t) { return (t == QC_U4 || t == QC_U8) ? QC_U8 : QC_S8; }
bool aligned16(const void *p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }
size_t align_up(size_t v, size_t a) { return (v + a - 1) / a * a; }
// MMA operand signedness of the activations: 4-bit codes are widened to unsigned bytes
// (nibble-plane widening, epilogue.cuh widen_word); 8-bit codes are used as they are.
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

// Driver releases up to 13.1 mis-handle a descriptor flag for tensors under 128 KiB;
// clearing bit 21 of the second descriptor word is the workaround CUTLASS applies
// (cute/atom/copy_traits_sm90_im2col.hpp, same version / size constants).
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
    int bits;           // activation bits
    int c_bytes;        // packed bytes per input pixel
    int64_t x_bytes, w_bytes, w8_bytes, y_bytes;
};

qc_status validate_desc(const qconv_desc *d, Geometry *g, bool allow_float) {
    if (!d) return QC_ERR_INVALID_ARG;
    if (d->n < 1 || d->h < 1 || d->w < 1 || d->c < 1 || d->k < 1 || d->r < 1 || d->s < 1)
        return QC_ERR_INVALID_ARG;
    if (d->stride_h < 1 || d->stride_w < 1 || d->dil_h < 1 || d->dil_w < 1 || d->pad_h < 0 ||
        d->pad_w < 0)
        return QC_ERR_INVALID_ARG;
    if (!is_int_input(d->x_t) || !is_int_input(d->w_t)) return QC_ERR_INVALID_ARG;
    if (!(is_packed_out(d->y_t) || d->y_t == QC_S32 || (allow_float && is_float_out(d->y_t))))
        return QC_ERR_INVALID_ARG;
    if (d->rounding != QC_ROUND_SINGLE && d->rounding != QC_ROUND_TFLITE) return QC_ERR_INVALID_ARG;
    if (d->relu != 0 && d->relu != 1) return QC_ERR_INVALID_ARG;
    const int64_t hx = static_cast<int64_t>(d->h) + 2 * d->pad_h - static_cast<int64_t>(d->dil_h) * (d->r - 1) - 1;
    const int64_t wx = static_cast<int64_t>(d->w) + 2 * d->pad_w - static_cast<int64_t>(d->dil_w) * (d->s - 1) - 1;
    if (hx < 0 || wx < 0) return QC_ERR_INVALID_ARG;
    const int P = static_cast<int>(hx / d->stride_h + 1);
    const int Q = static_cast<int>(wx / d->stride_w + 1);
    if (d->x_zero < dtype_min(d->x_t) || d->x_zero > dtype_max(d->x_t)) return QC_ERR_INVALID_ARG;
    if (is_packed_out(d->y_t)) {
        if (d->y_zero < dtype_min(d->y_t) || d->y_zero > dtype_max(d->y_t)) return QC_ERR_INVALID_ARG;
        if (d->clamp_lo > d->clamp_hi || d->clamp_lo < dtype_min(d->y_t) ||
            d->clamp_hi > dtype_max(d->y_t))
            return QC_ERR_INVALID_ARG;
    }
    const int bits = dtype_bits(d->x_t);
    if (bits == 4 && (d->c % 2)) return QC_ERR_INVALID_ARG;   // 4-bit pixel rows must be whole bytes
    const int64_t M = static_cast<int64_t>(d->n) * P * Q;
    g->P = P;
    g->Q = Q;
    g->M = M;
    g->bits = bits;
    g->c_bytes = d->c * bits / 8;
    g->x_bytes = static_cast<int64_t>(d->n) * d->h * d->w * g->c_bytes;
    g->w8_bytes = static_cast<int64_t>(d->k) * d->r * d->s * d->c;
    g->w_bytes = (g->w8_bytes * dtype_bits(d->w_t) + 7) / 8;
    const int yb = dtype_bits(d->y_t);
    if (yb == 4 && (d->k % 2)) return QC_ERR_UNSUPPORTED;
    g->y_bytes = M * d->k * yb / 8;
    return QC_OK;
}

// int32 accumulation bound ("overflow well addressed") on the caller's descriptor:
// both the raw MMA sum and the zero-point-centred sum must stay inside int32 for any codes
// of these dtypes.
qc_status check_overflow(const qconv_desc *d) {
    const int64_t T = static_cast<int64_t>(d->r) * d->s * d->c;
    const int64_t wmax = std::max(-dtype_min(d->w_t), dtype_max(d->w_t));
    const int64_t wctr = dtype_max(d->w_t) - dtype_min(d->w_t);      // |w - w_zero| with any zero point
    const int64_t xraw = std::max(-dtype_min(d->x_t), dtype_max(d->x_t));
    const int64_t xctr = std::max(d->x_zero - dtype_min(d->x_t), dtype_max(d->x_t) - d->x_zero);
    // 4-bit activations are widened to 16 x (x [+ 8]) (nibble-plane widening): the MMA sum
    // is 16 x larger and must stay below 2^30 (the epilogue adds 16 * bias inside int32)
    const bool nib = dtype_bits(d->x_t) == 4;
    const double lim = nib ? 67108864.0 /* 2^30 / 16 */ : 2147483647.0;
    const double xw = nib ? 15.0 : static_cast<double>(std::max(xraw, xctr));
    const double wz = d->w_zero ? static_cast<double>(wctr) : static_cast<double>(wmax);
    if (static_cast<double>(T) * xraw * wmax > lim || static_cast<double>(T) * xctr * wz > lim ||
        static_cast<double>(T) * xw * wmax > lim)
        return QC_ERR_OVERFLOW_RISK;
    return QC_OK;
}

// Structural limits of the kernels on the exec descriptor.
qc_status check_structure(const qconv_desc *e, const Geometry &g) {
    const bool pair = dtype_bits(e->x_t) == 8 && e->c == 16;   // 2 taps per 32-byte K-stage
    if (e->c % 32 && !pair) return QC_ERR_UNSUPPORTED;
    if (e->stride_h > 8 || e->stride_w > 8) return QC_ERR_UNSUPPORTED;   // TMA traversal stride
    const int lw = -e->pad_w, lh = -e->pad_h;
    const int uw = e->pad_w - e->dil_w * (e->s - 1), uh = e->pad_h - e->dil_h * (e->r - 1);
    if (lw < -128 || lh < -128 || uw < -128 || uh < -128 || uw > 127 || uh > 127)
        return QC_ERR_UNSUPPORTED;                     // rank-4 im2col corner range
    if (e->dil_w * (e->s - 1) > 255 || e->dil_h * (e->r - 1) > 255) return QC_ERR_UNSUPPORTED;
    if (g.M > INT32_MAX - 256 || e->n > 65535) return QC_ERR_UNSUPPORTED;
    if (static_cast<int64_t>(e->r) * e->s * e->c > INT32_MAX / 2) return QC_ERR_UNSUPPORTED;
    return QC_OK;
}

// ------------------------------------------------------------------ exec descriptor
enum Xform { XF_NONE = 0, XF_S2D = 1, XF_PAD = 2 };
enum WPrep { WP_COPY = 0, WP_NIBBLE = 1, WP_PLAIN = 2, WP_S2D = 3 };

struct Exec {
    const qconv_desc *d;  // the caller's descriptor
    Geometry gu;          // its geometry
    qconv_desc e;         // what the conv kernel sees
    Geometry g;           // its geometry
    int xform;
    int wprep;            // layout of the prepared weights
    bool wprep_needed;    // unprepared weights that need preparation on this call
    size_t prep_bytes;
    bool zx, zw;
    size_t off_w, off_x, off_zx, off_cs, off_x1, ws_total;
    int prologue;         // qconv_plan.prologue mask
    int s_pad;            // XF_PAD: extra zero-weight filter columns (odd S -> even: halo tap pairs)
};

int32_t s2d_channels(int32_t c) {
    const int32_t c4 = 4 * c;
    return c4 <= 16 ? 16 : (c4 + 31) / 32 * 32;
}

// Space-to-depth descriptor of a stride-2 conv (qconv.h): stride-1, unpadded, ceil(r/2) x
// ceil(s/2) taps over s2d_channels(c) byte codes; same output geometry.
qconv_desc s2d_of(const qconv_desc *d, const Geometry &g) {
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
    return o;
}

bool halo_eligible(const qconv_desc *e, const Geometry &g);   // after make_halo_plan below

qc_status derive_exec(const qconv_desc *d, bool allow_float, Exec *ex) {
    qc_status s = validate_desc(d, &ex->gu, allow_float);
    if (s != QC_OK) return s;
    const int xbits = dtype_bits(d->x_t), wbits = dtype_bits(d->w_t);
    if (xbits == 4 && wbits == 8) return QC_ERR_UNSUPPORTED;   // nibble-plane weights need 4-bit w
    s = check_overflow(d);
    if (s != QC_OK) return s;
    ex->d = d;
    ex->e = *d;
    const bool direct = (d->c % 32 == 0) || (xbits == 8 && d->c == 16);
    if (direct) {
        ex->xform = XF_NONE;
    } else if (d->stride_h == 2 && d->stride_w == 2 && d->dil_h == 1 && d->dil_w == 1 && 4 * d->c <= 16 &&
               d->w_zero == nullptr) {
        // (with weight zero points the s2d zero weights beyond r, s would not contribute 0)
        ex->xform = XF_S2D;
        ex->e = s2d_of(d, ex->gu);
    } else {
        ex->xform = XF_PAD;
        ex->e.c = (xbits == 8 && d->c < 16) ? 16 : (d->c + 31) / 32 * 32;
    }
    ex->s_pad = 0;
    if (ex->xform == XF_PAD && ex->e.c == 16 && xbits == 8 && (d->s % 2) && d->stride_w == 1 &&
        d->stride_h == 1 && d->dil_h == 1 && d->dil_w == 1 && d->x_zero == 0 && d->w_zero == nullptr) {
        // C = 16 byte codes pair two filter taps per K = 32 MMA in the halo kernels, which need
        // an even S: one more filter column of zero weights, one more input column of zero-point
        // codes (the column it would read past the image) -- same products, same P and Q --
        // taken only when a halo plan then exists (the im2col path would just do 1/S more MMAs)
        qconv_desc e2 = ex->e;
        e2.s += 1;
        e2.w += 1;
        e2.x_t = byte_container(d->x_t);
        e2.w_t = byte_container(d->w_t);
        Geometry g2;
        if (validate_desc(&e2, &g2, allow_float) == QC_OK && g2.P == ex->gu.P && g2.Q == ex->gu.Q &&
            halo_eligible(&e2, g2)) {
            ex->e.s = e2.s;
            ex->e.w = e2.w;
            ex->s_pad = 1;
        }
    }
    qconv_desc &e = ex->e;
    if (ex->xform == XF_S2D) ex->wprep = WP_S2D;
    else if (xbits == 4) ex->wprep = WP_NIBBLE;
    else if (wbits == 4 || ex->xform == XF_PAD) ex->wprep = WP_PLAIN;
    else ex->wprep = WP_COPY;
    if (ex->wprep == WP_PLAIN) e.w_t = byte_container(d->w_t);
    s = validate_desc(&e, &ex->g, allow_float);
    if (s != QC_OK) return s;
    s = check_structure(&e, ex->g);
    if (s != QC_OK) return s;
    const size_t w8 = static_cast<size_t>(ex->g.w8_bytes);
    ex->prep_bytes = ex->wprep == WP_NIBBLE ? align_up(w8, 16) + 4 * static_cast<size_t>(e.k) : w8;
    ex->wprep_needed = !d->w_prepared && ex->wprep != WP_COPY;
    ex->zx = e.x_zero != 0;
    ex->zw = d->w_zero != nullptr;
    size_t off = 0;
    ex->off_w = ex->off_x = ex->off_zx = ex->off_cs = ex->off_x1 = 0;
    ex->prologue = 0;
    if (ex->wprep_needed) { ex->off_w = off; off += align_up(ex->prep_bytes, 256); ex->prologue |= 1; }
    if (ex->xform != XF_NONE) { ex->off_x = off; off += align_up(static_cast<size_t>(ex->g.x_bytes), 256); ex->prologue |= 2; }
    if (ex->zx) {
        ex->off_zx = off;
        off += align_up(static_cast<size_t>(e.k) * (e.r + 1) * (e.s + 1) * 4, 256);
        ex->prologue |= 4;
    }
    if (ex->zw) {
        ex->off_cs = off;
        off += align_up(static_cast<size_t>(e.n) * e.h * e.w * 4, 256);
        ex->off_x1 = off;
        off += align_up(static_cast<size_t>(ex->g.M) * 4, 256);
        ex->prologue |= 8;
    }
    ex->ws_total = off;
    return QC_OK;
}

// Weight preparation into the exec layout (qconv_prepare_weights and the prologue).
qc_status prepare_weights_exec(const Exec &ex, const void *w, void *out, cudaStream_t st) {
    const qconv_desc *d = ex.d;
    const qconv_desc &e = ex.e;
    const int64_t rows = static_cast<int64_t>(d->k) * d->r * d->s;
    const int sgn = dtype_signed(d->w_t) ? 1 : 0;
    switch (ex.wprep) {
        case WP_COPY: {
            cudaError_t err = cudaMemcpyAsync(out, w, static_cast<size_t>(ex.g.w8_bytes), cudaMemcpyDeviceToDevice, st);
            if (err != cudaSuccess) return cuda_fail(err);
            break;
        }
        case WP_NIBBLE: {
            if (e.c == d->c) {
                const int64_t ngroups = ex.gu.w_bytes / 16;
                const int grid = static_cast<int>(std::min<int64_t>((ngroups + 255) / 256, 4096));
                qc::widen_w4_kernel<<<grid, 256, 0, st>>>(static_cast<const uint8_t *>(w), static_cast<int8_t *>(out),
                                                          ngroups, sgn);
            } else {
                const int64_t ngroups = rows * (e.c / 32);
                const int grid = static_cast<int>(std::min<int64_t>((ngroups + 255) / 256, 4096));
                qc::widen_w4_pad_kernel<<<grid, 256, 0, st>>>(static_cast<const uint8_t *>(w),
                                                              static_cast<int8_t *>(out), rows, d->c, e.c, sgn);
            }
            int32_t *wsum = reinterpret_cast<int32_t *>(static_cast<uint8_t *>(out) +
                                                        align_up(static_cast<size_t>(ex.g.w8_bytes), 16));
            qc::wsum_w4_kernel<<<d->k, 256, 0, st>>>(static_cast<const uint8_t *>(w), wsum,
                                                     static_cast<int64_t>(d->r) * d->s * d->c / 2, sgn);
            break;
        }
        case WP_PLAIN: {
            const int64_t rows_e = static_cast<int64_t>(e.k) * e.r * e.s;
            const int64_t total = rows_e * e.c;
            const int grid = static_cast<int>(std::min<int64_t>((total + 255) / 256, 4096));
            qc::weights_plain_kernel<<<grid, 256, 0, st>>>(static_cast<const uint8_t *>(w), static_cast<int8_t *>(out),
                                                           rows_e, d->c, e.c, dtype_bits(d->w_t), sgn, d->s, e.s);
            break;
        }
        case WP_S2D: {
            const int64_t total = static_cast<int64_t>(e.k) * e.r * e.s * e.c;
            const int grid = static_cast<int>(std::min<int64_t>((total + 255) / 256, 4096));
            qc::weights_s2d_kernel<<<grid, 256, 0, st>>>(static_cast<const uint8_t *>(w), static_cast<int8_t *>(out),
                                                         d->k, d->r, d->s, d->c, e.r, e.s, e.c,
                                                         dtype_bits(d->w_t), sgn);
            break;
        }
    }
    cudaError_t err = cudaGetLastError();
    if (err != cudaSuccess) return cuda_fail(err);
    return QC_OK;
}

// ------------------------------------------------------------------ launch plans
struct Plan {
    int kernel;       // qc_kernel
    int BK, bkp, chunks, BN, BM, n_tiles_n, num_tiles, num_kb, stages, grid, threads;
    uint32_t tmem_cols, smem_bytes;
    qc::ConvParams cp;
};

int choose_bk(int c) { return (c % 128 == 0) ? 128 : (c % 64 == 0 ? 64 : 32); }
uint32_t pow2_cols(int n) {
    uint32_t c = 32;
    while (c < static_cast<uint32_t>(n)) c <<= 1;
    return c;
}
bool needs_general_only(const Exec &ex) {
    return ex.zx || ex.zw || !is_packed_out(ex.e.y_t);
}

#ifdef QC_NO_A_TMEM          // build-time A/B switch (same bytes): widened A tiles in shared memory
constexpr bool g_no_a_tmem = true;
#else
constexpr bool g_no_a_tmem = false;
#endif

// im2col kernel (conv_fwd.cuh).  bn_req = 0: the default N tile (largest <= 256, halved
// while the grid would not fill the GPU -- P:L321: at small batch the tiling decides how
// well the machine is filled).
bool make_plan(const qconv_desc *d, const Geometry &g, int bn_req, Plan *pl) {
    const bool is4 = g.bits == 4;
    const bool pair = !is4 && d->c == 16;
    pl->kernel = QC_KERNEL_IM2COL;
    pl->BK = pair ? 32 : choose_bk(d->c);
    pl->bkp = is4 ? pl->BK / 2 : (pair ? 16 : pl->BK);
    pl->chunks = pair ? 1 : d->c / pl->BK;
    pl->num_kb = pair ? (d->r * d->s + 1) / 2 : d->r * d->s * pl->chunks;
    const int m_tiles = static_cast<int>((g.M + qc::kBM - 1) / qc::kBM);
    const int sms = num_sms();
    int BN;
    if (bn_req > 0) {
        if (bn_req % 16 || bn_req > qc::kMaxBN) return false;
        BN = bn_req;
    } else {
        BN = std::min(qc::kMaxBN, ((d->k + 15) / 16) * 16);
        while (BN > 64 && static_cast<int64_t>(m_tiles) * ((d->k + BN - 1) / BN) < sms)
            BN = std::max(64, ((BN / 2 + 15) / 16) * 16);
    }
    pl->BN = BN;
    pl->BM = qc::kBM;
    pl->n_tiles_n = (d->k + BN - 1) / BN;
    pl->num_tiles = m_tiles * pl->n_tiles_n;
    pl->tmem_cols = pow2_cols(2 * BN);
    // 4-bit: the widened A tile can live in TMEM (conv_fwd.cuh): one BK/4-column slab per stage
    // after the two accumulators -- no widened copy in shared memory and no A operand reads of
    // it, but the 512 columns cap the ring depth
    const int a_cols = pl->BK / 4;
    const int tmem_stages = is4 && !pair && !g_no_a_tmem ? (512 - 2 * BN) / a_cols : 0;
    const bool a_tmem = tmem_stages >= 4;
    const uint32_t a_bytes = a_tmem ? 0u : static_cast<uint32_t>(qc::kBM * pl->BK);
    const uint32_t b_bytes = static_cast<uint32_t>(align_up(static_cast<size_t>(BN) * pl->BK, 1024));
    const uint32_t stg_bytes = is4 ? static_cast<uint32_t>(qc::kBM * pl->bkp) : 0u;
    const uint32_t per_stage = a_bytes + b_bytes + stg_bytes;
    const bool packed = is_packed_out(d->y_t);
    const int ybits = dtype_bits(d->y_t);
    const int tile_row_bytes = BN * ybits / 8;
    const int y_gw = tile_row_bytes >= 128 ? 128 : tile_row_bytes;
    const bool y_tma = packed && BN % 32 == 0 && (static_cast<int64_t>(d->k) * ybits / 8) % 16 == 0 &&
                       (y_gw == 32 || y_gw == 64 || (y_gw == 128 && tile_row_bytes % 128 == 0));
    const uint32_t ystg_one = y_tma ? 128u * static_cast<uint32_t>(tile_row_bytes) : 0u;
    const uint32_t ystg_bytes = 2u * ystg_one;   // double-buffered
    const uint32_t fixed = static_cast<uint32_t>(qc::kMaxBN) * 16u + 128u + 1024u + ystg_bytes;
    const uint32_t budget = 227u * 1024u - 1024u - fixed;
    int stages = static_cast<int>(budget / per_stage);
    stages = std::min(stages, 32);     // deep rings: TMA latency is ~1-3 us under load
    if (a_tmem) stages = std::min(stages, tmem_stages);
    if (stages < 2) return false;
    pl->stages = stages;
    if (a_tmem) pl->tmem_cols = 512;
    qc::ConvParams &p = pl->cp;
    std::memset(&p, 0, sizeof(p));
    p.a_tmem_col = a_tmem ? 2 * BN : 0;
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
    p.need_clamp = (packed && (d->clamp_lo > dtype_min(d->y_t) || d->clamp_hi < dtype_max(d->y_t))) ? 1 : 0;
    p.sw_mask = pl->BK == 128 ? 7 : (pl->BK == 64 ? 3 : 1);
    p.idesc = qc::make_idesc_i8(qc::kBM, static_cast<uint32_t>(BN), act_signed(d), dtype_signed(d->w_t));
    p.tmem_cols = pl->tmem_cols;
    p.y_zero = packed ? d->y_zero : 0;
    p.clamp_lo = packed ? d->clamp_lo : INT32_MIN;
    p.clamp_hi = packed ? d->clamp_hi : INT32_MAX;
    p.x_zero = d->x_zero;
    p.y_row_bytes = static_cast<int64_t>(d->k) * dtype_bits(d->y_t) / 8;
    return true;
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

// ------------------------------------------------------------------ CTA-pair im2col
// The CTA-pair kernel (fwd2.cuh) by default runs im2col layers with R*S > 1 and a full
// N = 256 tile (measured faster there: res4/res5 3x3 -6 to -13 % at 4 and 8 bits; no gain
// for 1x1 layers, slower for N = 128 tiles); any N tile of 64..256 (multiple of 32) can be
// chosen through the plan API.
bool make_plan2(const qconv_desc *d, const Geometry &g, const Plan &pl1, bool chosen, Plan *pl) {
    if (pl1.cp.pair || d->x_zero != 0 || !is_packed_out(d->y_t) || !pl1.cp.y_tma) return false;
    const int BN = pl1.BN;
    if (BN % 32 || BN < 64) return false;
    if (!chosen && !(BN == 256 && d->r * d->s > 1)) return false;
    *pl = pl1;
    pl->kernel = QC_KERNEL_PAIR;
    pl->BM = 2 * qc::kBM;
    qc::ConvParams &p = pl->cp;
    const bool is4 = g.bits == 4;
    const int m_tiles2 = static_cast<int>((g.M + 2 * qc::kBM - 1) / (2 * qc::kBM));
    pl->num_tiles = m_tiles2 * pl1.n_tiles_n;
    p.a_tmem_col = 0;                                      // (A from TMEM: im2col kernel only)
    pl->tmem_cols = pow2_cols(2 * BN);
    p.tmem_cols = pl->tmem_cols;
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

// ------------------------------------------------------------------ halo mode (stride 1)
// f32_row_bytes > 0: the fused fp32-quantization stem (halo.cuh F32): the staging ring holds
// the tile's 2*HR fp32 input rows of f32_row_bytes each instead of packed codes.
// cm: the channel-major variant (halo.cuh CM): K = 64 output channels on TMEM lanes, N = Rt
// padded rows of Wh = round_up(W + 2 pad, 8) pixels (<= 256), the channel-pair epilogue.
bool make_halo_plan(const qconv_desc *d, const Geometry &g, Plan *pl, uint32_t f32_row_bytes = 0, bool cm = false) {
    if (d->stride_h != 1 || d->stride_w != 1 || d->dil_h != 1 || d->dil_w != 1) return false;
    if (d->x_zero != 0 || !is_packed_out(d->y_t)) return false;
    if (cm && (d->k != 64 || d->rounding == QC_ROUND_TFLITE)) return false;
    const bool is4 = g.bits == 4;
    const int C8 = d->c;                                 // int8 bytes per pixel after widening
    const bool tap_pair = !is4 && C8 == 16;
    if (tap_pair) {
        if (d->s % 2) return false;
    } else if (C8 % 32) {
        return false;
    }
    const int Wh = cm ? (d->w + 2 * d->pad_w + 7) / 8 * 8 : d->w + 2 * d->pad_w;
    const int tile_px = cm ? 256 : qc::kBM;               // accumulator rows (pixels) per tile
    if (Wh > tile_px || Wh > 256) return false;
    if (d->r * d->s == 1) return false;                 // no tap reuse: the im2col GEMM path is better
    const int Rt = tile_px / Wh;
    const int tpi = (g.P + Rt - 1) / Rt;
    if (static_cast<double>(g.P) * g.Q / (static_cast<double>(tpi) * tile_px) < 0.7) return false;
    const int HR = Rt + d->r - 1;
    const int nplanes = C8 / 16;
    const int nch = g.c_bytes / 16;                      // TMA channel chunks (packed for 4-bit)
    if (nch < 1 || nch > 256 || HR > 256) return false;
    const int KG8 = d->r * d->s * C8;
    const int nK = KG8 / 16;
    if (nK > 256) return false;
    // the whole weight slab stays resident (one N tile): MMA issue costs ~75 cycles per
    // instruction (measured), so narrower N tiles would be issue-bound
    if (d->k > 256) return false;
    const int BN = (d->k + 31) / 32 * 32;
    if (static_cast<int64_t>(BN) * KG8 > 100 * 1024) return false;
    const int ybits = dtype_bits(d->y_t);
    const int tile_row_bytes = BN * ybits / 8;
    const int y_gw = tile_row_bytes >= 128 ? 128 : tile_row_bytes;
    const int ystg_rows = cm ? 256 : 128;
    if (!((static_cast<int64_t>(d->k) * ybits / 8) % 16 == 0 &&
          (y_gw == 32 || y_gw == 64 || (y_gw == 128 && tile_row_bytes % 128 == 0))))
        return false;
    const int n_tiles_n = (d->k + BN - 1) / BN;
    const int tiles_per_img = (g.P + Rt - 1) / Rt;
    const int64_t num_tiles = static_cast<int64_t>(d->n) * tiles_per_img * n_tiles_n;
    if (num_tiles > INT32_MAX) return false;
    const uint32_t plane = static_cast<uint32_t>(HR * Wh * 16);
    // the fused fp32 stem keeps one ring of HR + Rt code rows, each stored twice, plus a
    // 64-byte zero area (halo.cuh F32) instead of a code halo per stage
    const uint32_t ringb = f32_row_bytes ? static_cast<uint32_t>(align_up(static_cast<size_t>(2 * (HR + Rt)) * Wh * 16 + 64 + (cm ? 256 : 0), 1024)) : 0u;
    const uint32_t hx = f32_row_bytes ? 0u : static_cast<uint32_t>(align_up(static_cast<size_t>(nplanes) * plane + (cm ? 256 : 0), 1024));
    const uint32_t hp = f32_row_bytes ? static_cast<uint32_t>(align_up(static_cast<size_t>(2 * HR) * f32_row_bytes, 1024))
                        : (is4 ? static_cast<uint32_t>(align_up(static_cast<size_t>(nch) * plane, 1024)) : 0u);
    const uint32_t bres = static_cast<uint32_t>(align_up(static_cast<size_t>(BN) * KG8, 1024));
    // output staging ring: 4 buffers when the halo ring keeps >= 3 stages, else 3, else 2
    int n_ystg = QC_MAX_YSTG;
    uint32_t ystg = 0, fixed = 0;
    for (;; --n_ystg) {
        ystg = static_cast<uint32_t>(n_ystg) * static_cast<uint32_t>(ystg_rows) * static_cast<uint32_t>(tile_row_bytes);
        fixed = bres + ringb + ystg + static_cast<uint32_t>(qc::kMaxBN) * 16u + 128u + 2048u +
                8u * static_cast<uint32_t>(d->r * d->s * nplanes);
        if (n_ystg == 2 || fixed + 3 * (hx + hp) <= 227u * 1024u) break;
    }
    if (fixed + 2 * (hx + hp) > 227u * 1024u) return false;
    int stages = static_cast<int>((227u * 1024u - fixed) / (hx + hp));
    stages = std::min(stages, 24);   // deep ring: the halo loads are latency-bound (~6 us each under load)
    if (f32_row_bytes && (!tap_pair || stages < 3)) return false;   // (the ring reuse needs 3 stages)
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
    p.off_hp = bres + (f32_row_bytes ? ringb : hx * stages);
    p.hp_stage_bytes = hp;
    p.halo_tx = f32_row_bytes ? static_cast<uint32_t>(2 * HR) * f32_row_bytes : static_cast<uint32_t>(nch) * plane;
    // whole-row loads when one box row (Wh pixels) fits the 256-element limit as int64s and the
    // staged layout works without planes: the C = 16 stem (one plane) or 4-bit inputs (the
    // converter re-lays the packed pixels into planes)
    p.c_px = g.c_bytes;
    p.halo_flat = ((tap_pair || is4) && (Wh * g.c_bytes) % 8 == 0 && Wh * g.c_bytes / 8 <= 256) ? 1 : 0;
    p.off_ystg = static_cast<uint32_t>(align_up(p.off_hp + hp * stages, 1024));
    p.ystg_bytes = ystg / static_cast<uint32_t>(n_ystg);
    p.n_ystg = n_ystg;
    p.y_tma = 1;
    p.y_gw = y_gw;
    p.y_gmask = y_gw == 128 ? 7 : (y_gw == 64 ? 3 : 1);
    p.n_ygroups = tile_row_bytes / y_gw;
    p.off_par = static_cast<uint32_t>(align_up(p.off_ystg + ystg, 16));
    p.n_mma = tap_pair ? d->r * (d->s / 2) : d->r * d->s * (nplanes / 2);
    if (p.n_mma > qc::kHaloMaxMMA) return false;
    p.off_mtab = static_cast<uint32_t>(align_up(p.off_par + static_cast<uint32_t>(qc::kMaxBN) * 16u + 128u, 16));
    p.off_bar = static_cast<uint32_t>(align_up(p.off_mtab + 8u * static_cast<uint32_t>(p.n_mma), 8));
    const uint32_t bar_bytes = static_cast<uint32_t>((3 * stages + 5 + 2 * qc::kMaxYstg + 1) * 8 + 16);
    pl->smem_bytes = p.off_bar + bar_bytes + 1024u;
    if (pl->smem_bytes > 227u * 1024u) return false;
    // kind::i8 takes N = 8 or a multiple of 16: the padded columns read halo pixels past the
    // tile (slack below) into accumulator columns nobody stores
    p.idesc = cm ? qc::make_idesc_i8(64u, static_cast<uint32_t>((Rt * Wh + 15) / 16 * 16), dtype_signed(d->w_t), act_signed(d))
                 : qc::make_idesc_i8(qc::kBM, static_cast<uint32_t>(BN), act_signed(d), dtype_signed(d->w_t));
    pl->tmem_cols = cm ? 512u : pow2_cols(2 * BN);
    p.tmem_cols = pl->tmem_cols;
    p.y_zero = d->y_zero; p.clamp_lo = d->clamp_lo; p.clamp_hi = d->clamp_hi; p.x_zero = 0;
    p.need_clamp = (d->clamp_lo > dtype_min(d->y_t) || d->clamp_hi < dtype_max(d->y_t)) ? 1 : 0;
    p.y_row_bytes = static_cast<int64_t>(d->k) * ybits / 8;
    const int sms = num_sms();
    int grid = std::min<int64_t>(num_tiles, sms / n_tiles_n * n_tiles_n);
    grid = std::max(grid / n_tiles_n * n_tiles_n, n_tiles_n);
    pl->kernel = cm ? QC_KERNEL_HALO_T : QC_KERNEL_HALO;
    pl->grid = grid;
    pl->threads = cm ? ((is4 || f32_row_bytes) ? qc::kTThreads4 : qc::kTThreads8)
                     : ((is4 || f32_row_bytes) ? 512 : 384);
    pl->BN = BN;
    pl->BM = cm ? Rt * Wh : qc::kBM;
    pl->n_tiles_n = n_tiles_n;
    pl->num_tiles = static_cast<int>(num_tiles);
    pl->stages = stages;
    return true;
}

bool halo_eligible(const qconv_desc *e, const Geometry &g) {
    Plan tmp;
    return make_halo_plan(e, g, &tmp, 0, true) || make_halo_plan(e, g, &tmp, 0, false);
}

qc_status encode_halo_maps(const qconv_desc *d, const Geometry &g, const qc::ConvParams &p,
                           const void *x, const void *w8, void *y, CUtensorMap *hm, CUtensorMap *bm,
                           CUtensorMap *ym, bool cm = false) {
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
    if (cm) {   // weights: [K-chunk][k / 16][h][i][16 B] view, smem row 16 g + 8 h + i = channel 16 g + 2 i + h
        const cuuint64_t kg = static_cast<cuuint64_t>(d->r) * d->s * d->c;
        cuuint64_t dims[5] = {16, 8, 2, static_cast<cuuint64_t>(d->k / 16), kg / 16};
        cuuint64_t strides[4] = {2 * kg, kg, 16 * kg, 16};
        cuuint32_t box[5] = {16, 8, 2, static_cast<cuuint32_t>(p.BN / 16), static_cast<cuuint32_t>(kg / 16)};
        cuuint32_t es[5] = {1, 1, 1, 1, 1};
        CUresult r = drv.tiled(bm, CU_TENSOR_MAP_DATA_TYPE_UINT8, 5, const_cast<void *>(w8), dims, strides,
                               box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                               CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        if (r != CUDA_SUCCESS) return cuda_fail(cudaErrorInvalidValue);
        small_tensor_fixup(bm, static_cast<uint64_t>(g.w8_bytes));
    } else {   // weights: [K-chunk][k][16 B] view of int8 KRSC
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
                             static_cast<cuuint32_t>(cm ? 1 : p.Rt), 1};
        cuuint32_t es[4] = {1, 1, 1, 1};
        CUresult r = drv.tiled(ym, CU_TENSOR_MAP_DATA_TYPE_UINT8, 4, y, dims, strides, box, es,
                               CU_TENSOR_MAP_INTERLEAVE_NONE, swizzle_for(p.y_gw),
                               CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        if (r != CUDA_SUCCESS) return cuda_fail(cudaErrorInvalidValue);
        small_tensor_fixup(ym, static_cast<uint64_t>(g.y_bytes));
    }
    return QC_OK;
}

// ------------------------------------------------------------------ channel-major 1x1 kernel
// bmc_req = 0: 128 output channels per tile when k % 128 == 0, else 64.  With 4-bit
// activations the 256-pixel operand tile doubles the on-chip widening per MAC; for deep
// inputs (C > 512) that outweighs the cheaper epilogue (measured, r1), so the default
// excludes them (the plan API can still choose it).
bool make_trans_plan(const qconv_desc *d, const Geometry &g, int bmc_req, bool chosen, Plan *pl) {
    if (d->r != 1 || d->s != 1 || d->x_zero != 0 || !is_packed_out(d->y_t)) return false;
    if (d->rounding == QC_ROUND_TFLITE) return false;   // kept out of its epilogue (register budget)
    if (d->c % 32 || d->k % 64) return false;
    const bool is4 = g.bits == 4;
    if (!chosen && is4 && d->c > 512) return false;
    const int ybits = dtype_bits(d->y_t);
    if ((static_cast<int64_t>(d->k) * ybits / 8) % 16) return false;
    int BMc = d->k % 128 == 0 ? 128 : 64;
    if (bmc_req) {
        if (bmc_req != 64 && bmc_req != 128) return false;
        if (d->k % bmc_req) return false;
        BMc = bmc_req;
    }
    const int BNp = qc::kTBNp;                               // pixels per tile (trans.cuh)
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
    const uint32_t fixed = static_cast<uint32_t>(qc::kTGroups) * ystg_one + 2048u;
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
    p.off_par = static_cast<uint32_t>(align_up(p.off_ystg + static_cast<uint32_t>(qc::kTGroups) * ystg_one, 16));
    p.off_bar = static_cast<uint32_t>(align_up(p.off_par, 8));
    const uint32_t bar_bytes = static_cast<uint32_t>((3 * stages + 16) * 8 + 16);
    pl->smem_bytes = p.off_bar + bar_bytes + 1024u;
    if (pl->smem_bytes > 227u * 1024u) return false;
    p.idesc = qc::make_idesc_i8(static_cast<uint32_t>(BMc), static_cast<uint32_t>(BNp),
                                dtype_signed(d->w_t), act_signed(d));
    pl->tmem_cols = pow2_cols(qc::kTGroups * BNp);
    p.tmem_cols = pl->tmem_cols;
    p.y_zero = d->y_zero; p.clamp_lo = d->clamp_lo; p.clamp_hi = d->clamp_hi;
    p.need_clamp = (d->clamp_lo > dtype_min(d->y_t) || d->clamp_hi < dtype_max(d->y_t)) ? 1 : 0;
    p.y_row_bytes = static_cast<int64_t>(d->k) * ybits / 8;
    const int sms = num_sms();
    int grid = static_cast<int>(std::min<int64_t>(num_tiles, sms / n_tiles_n * n_tiles_n));
    grid = std::max(grid, 1);
    pl->kernel = QC_KERNEL_CHANNEL;
    pl->grid = grid;
    pl->threads = is4 ? qc::kTThreads4 : qc::kTThreads8;
    pl->BK = BK; pl->bkp = bkp; pl->BN = BMc; pl->BM = BNp; pl->n_tiles_n = n_tiles_n;
    pl->num_tiles = static_cast<int>(num_tiles); pl->stages = stages; pl->chunks = p.chunks;
    pl->num_kb = p.num_kb;
    return true;
}

// ------------------------------------------------------------------ plan choice
struct Choice {
    int kernel = QC_KERNEL_AUTO;
    int bn = 0;
};

// Resolve a choice to a plan on the exec descriptor; AUTO = the default rule
// (channel-major halo -> halo -> channel-major 1x1 -> CTA pair -> im2col).
bool resolve(const Exec &ex, Choice c, Plan *pl) {
    const qconv_desc *e = &ex.e;
    const Geometry &g = ex.g;
    const bool special_ok = !needs_general_only(ex);       // halo / channel / pair eligibility
    if (c.kernel == QC_KERNEL_AUTO) {
        if (special_ok && make_halo_plan(e, g, pl, 0, true)) return true;   // K = 64: channel-major halo
        if (special_ok && make_halo_plan(e, g, pl)) return true;
        if (special_ok && make_trans_plan(e, g, 0, false, pl)) return true;
        Plan p1;
        if (!make_plan(e, g, 0, &p1)) return false;
        if (special_ok && make_plan2(e, g, p1, false, pl)) return true;
        *pl = p1;
        return true;
    }
    switch (c.kernel) {
        case QC_KERNEL_HALO:
            if (!special_ok || !make_halo_plan(e, g, pl)) return false;
            return c.bn == 0 || c.bn == pl->BN;
        case QC_KERNEL_HALO_T:
            if (!special_ok || !make_halo_plan(e, g, pl, 0, true)) return false;
            return c.bn == 0 || c.bn == pl->BN;
        case QC_KERNEL_CHANNEL:
            return special_ok && make_trans_plan(e, g, c.bn, true, pl);
        case QC_KERNEL_PAIR: {
            Plan p1;
            return special_ok && make_plan(e, g, c.bn, &p1) && make_plan2(e, g, p1, true, pl);
        }
        case QC_KERNEL_IM2COL:
            return make_plan(e, g, c.bn, pl);
        default:
            return false;
    }
}

std::vector<Choice> candidates(const Exec &ex) {
    std::vector<Choice> out;
    Plan pl;
    auto try_add = [&](int kernel, int bn) {
        Choice c;
        c.kernel = kernel;
        c.bn = bn;
        if (resolve(ex, c, &pl)) {
            for (const Choice &o : out)
                if (o.kernel == kernel && o.bn == pl.BN) return;
            c.bn = pl.BN;
            out.push_back(c);
        }
    };
    try_add(QC_KERNEL_HALO, 0);
    try_add(QC_KERNEL_HALO_T, 0);
    try_add(QC_KERNEL_CHANNEL, 64);
    try_add(QC_KERNEL_CHANNEL, 128);
    const int kmax = std::min(qc::kMaxBN, (ex.e.k + 15) / 16 * 16);
    for (int bn : {64, 128, 256})
        if (bn <= std::max(kmax, 64)) try_add(QC_KERNEL_PAIR, bn);
    for (int bn : {32, 64, 128, 256})
        if (bn < kmax * 2) try_add(QC_KERNEL_IM2COL, std::min(bn, kmax));
    return out;
}

// Process-wide choices (qconv_plan_set) keyed by every field of the caller's descriptor
// (w_zero by presence), and the autotuner's per-thread forced choice.
std::mutex g_plan_mu;
std::map<std::string, Choice> g_plans;
thread_local bool g_forced = false;
thread_local Choice g_force;

std::string desc_key(const qconv_desc *d) {
    const int32_t f[] = {d->n, d->h, d->w, d->c, d->k, d->r, d->s, d->stride_h, d->stride_w, d->pad_h,
                         d->pad_w, d->dil_h, d->dil_w, static_cast<int32_t>(d->x_t), static_cast<int32_t>(d->w_t),
                         static_cast<int32_t>(d->y_t), d->x_zero, d->w_zero ? 1 : 0, d->w_prepared, d->y_zero,
                         d->clamp_lo, d->clamp_hi, d->rounding, d->relu};
    return std::string(reinterpret_cast<const char *>(f), sizeof(f));
}

Choice current_choice(const qconv_desc *d) {
    if (g_forced) return g_force;
    std::lock_guard<std::mutex> lk(g_plan_mu);
    if (g_plans.empty()) return Choice();
    auto it = g_plans.find(desc_key(d));
    return it == g_plans.end() ? Choice() : it->second;
}

void fill_plan_out(const Exec &ex, const Plan &pl, qconv_plan *o) {
    std::memset(o, 0, sizeof(*o));
    o->kernel = pl.kernel;
    o->bn = pl.BN;
    o->bm = pl.BM;
    o->stages = pl.stages;
    o->grid = pl.grid;
    o->threads = pl.threads;
    o->num_tiles = pl.num_tiles;
    o->smem_bytes = static_cast<int32_t>(pl.smem_bytes);
    o->tmem_cols = static_cast<int32_t>(pl.kernel == QC_KERNEL_HALO || pl.kernel == QC_KERNEL_HALO_T ||
                                                pl.kernel == QC_KERNEL_CHANNEL
                                            ? pl.cp.tmem_cols : pl.tmem_cols);
    o->prologue = ex.prologue;
    o->epilogue_mode = (needs_general_only(ex) || ex.e.rounding == QC_ROUND_TFLITE) ? 2 : -1;
}

// ------------------------------------------------------------------ the forward call
qc_status run_prologue(const Exec &ex, const void *x, const void *w, void *ws, cudaStream_t st,
                       const void **x_e, const void **w_e) {
    const qconv_desc *d = ex.d;
    const qconv_desc &e = ex.e;
    uint8_t *wsb = static_cast<uint8_t *>(ws);
    *x_e = x;
    *w_e = w;
    if (ex.wprep_needed) {
        qc_status s = prepare_weights_exec(ex, w, wsb + ex.off_w, st);
        if (s != QC_OK) return s;
        *w_e = wsb + ex.off_w;
    }
    if (ex.xform == XF_S2D) {
        const int64_t total = static_cast<int64_t>(e.n) * e.h * e.w * e.c;
        const int grid = static_cast<int>(std::min<int64_t>((total + 255) / 256, static_cast<int64_t>(num_sms()) * 16));
        qc::repack_s2d_kernel<<<grid, 256, 0, st>>>(static_cast<const uint8_t *>(x), wsb + ex.off_x, d->n, d->h,
                                                    d->w, d->c, e.h, e.w, e.c, d->pad_h, d->pad_w,
                                                    dtype_bits(d->x_t), dtype_signed(d->x_t) ? 1 : 0, d->x_zero);
        *x_e = wsb + ex.off_x;
    } else if (ex.xform == XF_PAD) {
        const int64_t npix = static_cast<int64_t>(d->n) * d->h * d->w;
        const int grid = static_cast<int>(std::min<int64_t>((npix + 255) / 256, static_cast<int64_t>(num_sms()) * 16));
        const int64_t npix_e = static_cast<int64_t>(e.n) * e.h * e.w;
        qc::repack_pad_kernel<<<grid, 256, 0, st>>>(static_cast<const uint8_t *>(x), wsb + ex.off_x, npix_e, d->c,
                                                    e.c, dtype_bits(d->x_t), d->x_zero, d->w, e.w);
        *x_e = wsb + ex.off_x;
    }
    if (ex.zx) {
        int32_t *table = reinterpret_cast<int32_t *>(wsb + ex.off_zx);
        qc::zx_table_kernel<<<(e.k + 127) / 128, 128, 0, st>>>(
            static_cast<const int8_t *>(*w_e), table, e.k, e.r, e.s, e.c, dtype_signed(e.w_t) ? 0 : 1,
            ex.wprep == WP_NIBBLE ? 1 : 0);
    }
    if (ex.zw) {
        int32_t *cs = reinterpret_cast<int32_t *>(wsb + ex.off_cs);
        int32_t *x1 = reinterpret_cast<int32_t *>(wsb + ex.off_x1);
        const int64_t npix = static_cast<int64_t>(e.n) * e.h * e.w;
        const int grid = static_cast<int>(std::min<int64_t>((npix * 32 + 255) / 256, static_cast<int64_t>(num_sms()) * 16));
        qc::chsum_kernel<<<grid, 256, 0, st>>>(static_cast<const uint8_t *>(*x_e), cs, npix, e.c,
                                               dtype_bits(e.x_t), dtype_signed(e.x_t) ? 1 : 0, e.x_zero);
        const int grid2 = static_cast<int>(std::min<int64_t>((ex.g.M + 255) / 256, static_cast<int64_t>(num_sms()) * 16));
        qc::x1_kernel<<<grid2, 256, 0, st>>>(cs, x1, e.n, e.h, e.w, ex.g.P, ex.g.Q, e.r, e.s, e.stride_h,
                                             e.stride_w, e.pad_h, e.pad_w, e.dil_h, e.dil_w);
    }
    cudaError_t err = cudaGetLastError();
    if (err != cudaSuccess) return cuda_fail(err);
    return QC_OK;
}

// Accumulator scale and signed-offset correction of 4-bit activations (widen_word).
void set_act_params(const Exec &ex, const void *w8, qc::ConvParams &p) {
    const bool nib = ex.wprep == WP_NIBBLE;
    p.acc_lg = nib ? 4 : 0;
    p.x_sgn4 = (nib && ex.e.x_t == QC_S4) ? 1 : 0;
    p.wsum = p.x_sgn4 ? reinterpret_cast<const int32_t *>(static_cast<const uint8_t *>(w8) +
                                                           align_up(static_cast<size_t>(ex.g.w8_bytes), 16))
                      : nullptr;
}

#ifdef QC_DEBUG
// Debug builds only: QC_TRACE=<file> appends timestamps of CTA 0's pipeline events after a sync.
void debug_attach(qc::ConvParams &cp, cudaStream_t stream) {
    static const char *trace_file = std::getenv("QC_TRACE");
    cp.trace = nullptr;
    if (trace_file) {
        unsigned long long *tbuf = nullptr;
        cudaMalloc(&tbuf, 16 * 1024 * sizeof(unsigned long long));
        cudaMemsetAsync(tbuf, 0, 16 * 1024 * sizeof(unsigned long long), stream);
        cp.trace = tbuf;
    }
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
#else
void debug_attach(qc::ConvParams &, cudaStream_t) {}
void debug_dump(const qc::ConvParams &, cudaStream_t) {}
#endif

qc_status launch_plan(const Exec &ex, Plan &pl, const void *x, const void *w8, const int32_t *bias,
                      const int32_t *mult, const int32_t *shift, const float *dq, void *y, void *ws,
                      cudaStream_t st) {
    const qconv_desc *e = &ex.e;
    const Geometry &g = ex.g;
    const bool is4 = g.bits == 4;
    const int out = out_kind(e->y_t);
    qc::ConvParams &p = pl.cp;
    set_act_params(ex, w8, p);
    p.bias = bias;
    p.mult = mult;
    p.shift = shift;
    p.dq_scale = dq;
    p.y = y;
    p.round_tfl = e->rounding == QC_ROUND_TFLITE ? 1 : 0;
    p.relu = e->relu;
    uint8_t *wsb = static_cast<uint8_t *>(ws);
    p.zx_table = ex.zx ? reinterpret_cast<const int32_t *>(wsb + ex.off_zx) : nullptr;
    p.zw = ex.zw ? ex.d->w_zero : nullptr;
    p.x1 = ex.zw ? reinterpret_cast<const int32_t *>(wsb + ex.off_x1) : nullptr;
    p.fd_pq = qc::make_fastdiv(static_cast<uint32_t>(p.PQ));
    p.fd_q = qc::make_fastdiv(static_cast<uint32_t>(p.Q));
    p.fd_ntn = qc::make_fastdiv(static_cast<uint32_t>(p.n_tiles_n));
    p.fd_tpr = qc::make_fastdiv(static_cast<uint32_t>(std::max(1, p.S * p.chunks)));
    p.fd_chunks = qc::make_fastdiv(static_cast<uint32_t>(std::max(1, p.chunks)));
    p.fd_s = qc::make_fastdiv(static_cast<uint32_t>(std::max(1, p.S)));
    p.fd_tpi = qc::make_fastdiv(static_cast<uint32_t>(std::max(1, p.tiles_per_img)));
    debug_attach(p, st);
    qc::Launch L;
    L.grid = dim3(static_cast<unsigned>(pl.grid));
    L.threads = pl.threads;
    L.smem = pl.smem_bytes;
    L.stream = st;
    static const bool no_pdl = std::getenv("QC_NO_PDL") != nullptr;   // same bytes either way
    L.pdl = !no_pdl;
    cudaError_t err = cudaSuccess;
    qc_status s = QC_OK;
    alignas(64) CUtensorMap m0, m1, m2;
    std::memset(&m2, 0, sizeof(m2));
    switch (pl.kernel) {
        case QC_KERNEL_HALO:
        case QC_KERNEL_HALO_T: {
            const bool cm = pl.kernel == QC_KERNEL_HALO_T;
            s = encode_halo_maps(e, g, p, x, w8, y, &m0, &m1, &m2, cm);
            if (s != QC_OK) return s;
            err = qc::launch_halo(L, is4, out, m0, m1, m2, p, cm);
            break;
        }
        case QC_KERNEL_CHANNEL:
            p.stg_sw = is4 ? packed_sw_mask(pl.bkp) : 0;
            s = encode_x_map(e, g, x, pl.bkp, is4 ? packed_swizzle(pl.bkp) : swizzle_for(pl.BK), &m0, p.Wh);
            if (s != QC_OK) return s;
            s = encode_w_map_pairs(e, g, w8, pl.BK, pl.BN, swizzle_for(pl.BK), &m1);
            if (s != QC_OK) return s;
            s = encode_y_map(e, g, y, p.y_gw, &m2, p.Wh, true);
            if (s != QC_OK) return s;
            err = qc::launch_trans(L, is4, out, pl.BN == 64, m0, m1, m2, p);
            break;
        case QC_KERNEL_PAIR:
        case QC_KERNEL_IM2COL: {
            const bool pair = p.pair != 0;
            p.stg_sw = is4 ? packed_sw_mask(pl.bkp) : 0;
            s = encode_x_map(e, g, x, pl.bkp,
                             pair ? CU_TENSOR_MAP_SWIZZLE_NONE : (is4 ? packed_swizzle(pl.bkp) : swizzle_for(pl.BK)),
                             &m0);
            if (s != QC_OK) return s;
            const int wbn = pl.kernel == QC_KERNEL_PAIR ? pl.BN / 2 : pl.BN;
            s = encode_w_map(e, g, w8, pair ? 16 : pl.BK, wbn, pair ? CU_TENSOR_MAP_SWIZZLE_NONE : swizzle_for(pl.BK),
                             &m1);
            if (s != QC_OK) return s;
            if (p.y_tma) {
                s = encode_y_map(e, g, y, p.y_gw, &m2);
                if (s != QC_OK) return s;
            }
            if (pl.kernel == QC_KERNEL_PAIR) {
                L.cluster = 2;
                err = qc::launch_fwd2(L, is4, out, m0, m1, m2, p);
            } else {
                err = qc::launch_fwd(L, is4, out, ex.zx || ex.zw, m0, m1, m2, p);
            }
            break;
        }
        default:
            return QC_ERR_INVALID_ARG;
    }
    if (err != cudaSuccess) return cuda_fail(err);
    debug_dump(p, st);
    return QC_OK;
}

qc_status forward_impl(const qconv_desc *d, bool dequant, const void *x, const void *w, const int32_t *bias,
                       const int32_t *mult, const int32_t *shift, const float *dq, void *y, void *workspace,
                       size_t ws_bytes, void *stream) {
    Exec ex;
    qc_status s = derive_exec(d, dequant, &ex);
    if (s != QC_OK) return s;
    if (dequant && !is_float_out(d->y_t)) return QC_ERR_INVALID_ARG;
    if (!x || !w || !y) return QC_ERR_INVALID_ARG;
    if (is_packed_out(d->y_t) && (!mult || !shift)) return QC_ERR_INVALID_ARG;
    if (dequant && !dq) return QC_ERR_INVALID_ARG;
    if (!aligned16(x) || !aligned16(w) || !aligned16(y) || (bias && !aligned16(bias)) ||
        (mult && !aligned16(mult)) || (shift && !aligned16(shift)) || (dq && !aligned16(dq)) ||
        (d->w_zero && !aligned16(d->w_zero)) || (workspace && !aligned16(workspace)))
        return QC_ERR_MISALIGNED;
    if (ex.ws_total > 0 && (!workspace || ws_bytes < ex.ws_total)) return QC_ERR_WORKSPACE;
    Plan pl;
    const Choice c = current_choice(d);
    if (!resolve(ex, c, &pl)) {
        if (c.kernel == QC_KERNEL_AUTO || !resolve(ex, Choice(), &pl)) return QC_ERR_UNSUPPORTED;
    }
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    const void *x_e = nullptr, *w_e = nullptr;
    s = run_prologue(ex, x, w, workspace, st, &x_e, &w_e);
    if (s != QC_OK) return s;
    return launch_plan(ex, pl, x_e, w_e, bias, mult, shift, dq, y, workspace, st);
}

// ------------------------------------------------------------------ fused quantization + conv
// qconv2d_forward_quantize: float activations in.  The space-to-depth stem (stride 2, 4c <= 16)
// runs the halo kernel with the quantization fused into its producer / converter warps
// (halo.cuh F32); any other layer quantizes into the workspace, then runs qconv2d_forward.
struct QExec {
    bool fused;
    int esz;                  // input element bytes: 4 (fp32) or 2 (bf16)
    Exec ex;                  // fused: the s2d exec descriptor; else the codes' exec descriptor
    Plan pl;                  // fused: the halo plan with fp32 staging
    qconv_desc dq;            // fallback: the descriptor of the quantized codes
    size_t codes_bytes;       // fallback: quantized activations at the head of the workspace
    size_t ws_total;
};

qc_status derive_qexec(const qconv_desc *d, qc_ftype xt, QExec *qx) {
    if (!d) return QC_ERR_INVALID_ARG;
    if (xt != QC_F32 && xt != QC_BF16) return QC_ERR_INVALID_ARG;
    qx->esz = xt == QC_BF16 ? 2 : 4;
    qconv_desc dv = *d;                      // codes of any 4-bit c live in bytes in the s2d form
    dv.x_t = byte_container(d->x_t);
    Geometry gv;
    qc_status s = validate_desc(&dv, &gv, true);
    if (s != QC_OK) return s;
    if (!is_int_input(d->x_t)) return QC_ERR_INVALID_ARG;
    const bool s2d_ok = d->stride_h == 2 && d->stride_w == 2 && d->dil_h == 1 && d->dil_w == 1 &&
                        4 * d->c <= 16 && d->w_zero == nullptr && d->x_zero == 0 &&
                        (static_cast<int64_t>(d->w) * d->c) % 4 == 0 && static_cast<int64_t>(d->w) * d->c <= 1024 &&
                        is_packed_out(d->y_t);
    qx->fused = false;
    if (s2d_ok && check_overflow(d) == QC_OK) {
        Exec &ex = qx->ex;
        ex.d = d;
        ex.gu = gv;
        ex.e = s2d_of(d, gv);
        if (validate_desc(&ex.e, &ex.g, false) == QC_OK && check_structure(&ex.e, ex.g) == QC_OK) {
            ex.xform = XF_S2D;
            ex.wprep = WP_S2D;
            ex.wprep_needed = !d->w_prepared;
            ex.prep_bytes = static_cast<size_t>(ex.g.w8_bytes);
            ex.zx = ex.zw = false;
            ex.off_w = ex.off_x = ex.off_zx = ex.off_cs = ex.off_x1 = 0;
            ex.prologue = ex.wprep_needed ? 1 : 0;
            ex.ws_total = ex.wprep_needed ? align_up(ex.prep_bytes, 256) : 0;
            // the fused stem runs the channel-major halo when it is eligible (K = 64), unless a
            // plan choice for `d` asks for the pixel-major one
            const uint32_t frow = static_cast<uint32_t>(d->w) * d->c * static_cast<uint32_t>(qx->esz);
            const Choice c = current_choice(d);
            const bool cm_first = c.kernel != QC_KERNEL_HALO;
            if ((cm_first && make_halo_plan(&ex.e, ex.g, &qx->pl, frow, true)) ||
                (c.kernel != QC_KERNEL_HALO_T && make_halo_plan(&ex.e, ex.g, &qx->pl, frow, false))) {
                qx->fused = true;
                qx->ws_total = ex.ws_total;
                return QC_OK;
            }
        }
    }
    // fallback: codes in the workspace, then the ordinary forward
    if (dtype_bits(d->x_t) == 4 && (d->c % 2)) return QC_ERR_UNSUPPORTED;   // no whole-byte code rows
    qx->dq = *d;
    s = derive_exec(&qx->dq, false, &qx->ex);
    if (s != QC_OK) return s;
    qx->codes_bytes = align_up(static_cast<size_t>(qx->ex.gu.x_bytes), 256);
    qx->ws_total = qx->codes_bytes + qx->ex.ws_total;
    return QC_OK;
}

qc_status launch_fused_stem(QExec &qx, const void *x, float in_scale, const void *w8, const int32_t *bias,
                            const int32_t *mult, const int32_t *shift, void *y, cudaStream_t st) {
    const Exec &ex = qx.ex;
    const qconv_desc *d = ex.d;
    const qconv_desc *e = &ex.e;
    Plan &pl = qx.pl;
    qc::ConvParams &p = pl.cp;
    p.acc_lg = 0;
    p.x_sgn4 = 0;
    p.wsum = nullptr;
    p.bias = bias;
    p.mult = mult;
    p.shift = shift;
    p.y = y;
    p.round_tfl = e->rounding == QC_ROUND_TFLITE ? 1 : 0;
    p.q_inv_s = 1.0f / in_scale;
    p.q_z = d->x_zero;
    p.q_qmin = static_cast<int32_t>(dtype_min(d->x_t));
    p.q_qmax = static_cast<int32_t>(dtype_max(d->x_t));
    p.q_flo = static_cast<float>(p.q_qmin - p.q_z);     // exact integer bounds (halo.cuh f32_q)
    p.q_fhi = static_cast<float>(p.q_qmax - p.q_z);
    p.f_w = d->w;
    p.f_c = d->c;
    p.f_pad_h = d->pad_h;
    p.f_pad_w = d->pad_w;
    p.f_rowbytes = d->w * d->c * qx.esz;
    p.bf16 = qx.esz == 2 ? 1 : 0;
    p.fd_pq = qc::make_fastdiv(static_cast<uint32_t>(p.PQ));
    p.fd_q = qc::make_fastdiv(static_cast<uint32_t>(p.Q));
    p.fd_ntn = qc::make_fastdiv(static_cast<uint32_t>(p.n_tiles_n));
    p.fd_tpr = qc::make_fastdiv(1u);
    p.fd_chunks = qc::make_fastdiv(1u);
    p.fd_s = qc::make_fastdiv(static_cast<uint32_t>(std::max(1, p.S)));
    p.fd_tpi = qc::make_fastdiv(static_cast<uint32_t>(std::max(1, p.tiles_per_img)));
    alignas(64) CUtensorMap hm, bm, ym;
    const bool cm = pl.kernel == QC_KERNEL_HALO_T;
    qc_status s = encode_halo_maps(e, ex.g, p, x, w8, y, &hm, &bm, &ym, cm);
    if (s != QC_OK) return s;
    {   // fp32 input rows as raw 8-byte elements: [n][h][k pieces][row/k]; each row piece is one
        // long contiguous TMA row (a 16-byte inner box would cost one request per 16 bytes);
        // rows outside the image are zero-filled (= +0.0f, which quantizes to the zero point)
        const Driver &drv = driver();
        const cuuint64_t rowb = static_cast<cuuint64_t>(d->w) * d->c * qx.esz;
        cuuint64_t k = (rowb + 2047) / 2048;
        while (rowb % (8 * k)) ++k;
        const cuuint64_t piece = rowb / (8 * k);
        cuuint64_t dims[4] = {piece, k, static_cast<cuuint64_t>(d->h), static_cast<cuuint64_t>(d->n)};
        cuuint64_t strides[3] = {piece * 8, rowb, rowb * d->h};
        cuuint32_t box[4] = {static_cast<cuuint32_t>(piece), static_cast<cuuint32_t>(k), 2, 1};   // one row pair
        cuuint32_t es[4] = {1, 1, 1, 1};
        if (piece > 256) return QC_ERR_UNSUPPORTED;
        CUresult r = drv.tiled(&hm, CU_TENSOR_MAP_DATA_TYPE_INT64, 4, const_cast<void *>(x), dims, strides, box, es,
                               CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                               CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        if (r != CUDA_SUCCESS) return cuda_fail(cudaErrorInvalidValue);
    }
    qc::Launch L;
    L.grid = dim3(static_cast<unsigned>(pl.grid));
    L.threads = pl.threads;
    L.smem = pl.smem_bytes;
    L.stream = st;
    static const bool no_pdl = std::getenv("QC_NO_PDL") != nullptr;
    L.pdl = !no_pdl;
    debug_attach(p, st);
    cudaError_t err = qc::launch_halo(L, false, out_kind(e->y_t), hm, bm, ym, p, cm);
    if (err != cudaSuccess) return cuda_fail(err);
    debug_dump(p, st);
    return QC_OK;
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
int qconv_version(void) { return 200; }

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

// Weight preparation of a descriptor whose activations only exist as floats for the fused
// stem: 4-bit codes with an odd c have no packed NHWC form, but the space-to-depth operand holds
// them in bytes, so the weights are prepared as for the byte-container view (same W2).
static qc_status derive_exec_for_weights(const qconv_desc *d, Exec *ex, qconv_desc *tmp) {
    qc_status s = derive_exec(d, true, ex);
    if (s == QC_ERR_INVALID_ARG && d && is_int_input(d->x_t) && dtype_bits(d->x_t) == 4 && (d->c % 2)) {
        *tmp = *d;
        tmp->x_t = byte_container(d->x_t);
        tmp->x_zero = 0;
        s = derive_exec(tmp, true, ex);
        if (s == QC_OK && ex->xform != XF_S2D) return QC_ERR_INVALID_ARG;
    }
    return s;
}

size_t qconv_prepared_weight_bytes(const qconv_desc *d) {
    Exec ex;
    qconv_desc tmp;
    if (derive_exec_for_weights(d, &ex, &tmp) != QC_OK) return 0;
    return ex.prep_bytes;
}

qc_status qconv_prepare_weights(const qconv_desc *d, const void *w, void *w_prep, void *stream) {
    Exec ex;
    qconv_desc tmp;
    qc_status s = derive_exec_for_weights(d, &ex, &tmp);
    if (s != QC_OK) return s;
    if (!w || !w_prep) return QC_ERR_INVALID_ARG;
    if (!aligned16(w) || !aligned16(w_prep)) return QC_ERR_MISALIGNED;
    return prepare_weights_exec(ex, w, w_prep, static_cast<cudaStream_t>(stream));
}

size_t qconv2d_workspace_size(const qconv_desc *d) {
    Exec ex;
    if (derive_exec(d, true, &ex) != QC_OK) return 0;
    return ex.ws_total;
}

qc_status qconv2d_forward(const qconv_desc *d, const void *x, const void *w, const int32_t *bias,
                          const int32_t *multiplier, const int32_t *shift, void *y, void *workspace,
                          size_t ws_bytes, void *stream) {
    return forward_impl(d, false, x, w, bias, multiplier, shift, nullptr, y, workspace, ws_bytes, stream);
}

qc_status qconv2d_forward_dequant(const qconv_desc *d, const void *x, const void *w, const int32_t *bias,
                                  const float *scale, void *y, void *workspace, size_t ws_bytes, void *stream) {
    return forward_impl(d, true, x, w, bias, nullptr, nullptr, scale, y, workspace, ws_bytes, stream);
}

size_t qconv2d_quantize_workspace_size(const qconv_desc *d, qc_ftype xt) {
    QExec qx;
    if (derive_qexec(d, xt, &qx) != QC_OK) return 0;
    return qx.ws_total;
}

qc_status qconv2d_forward_quantize(const qconv_desc *d, const void *x, qc_ftype xt, float in_scale,
                                   const void *w, const int32_t *bias, const int32_t *multiplier,
                                   const int32_t *shift, void *y, void *workspace, size_t ws_bytes,
                                   void *stream) {
    QExec qx;
    qc_status s = derive_qexec(d, xt, &qx);
    if (s != QC_OK) return s;
    if (!x || !w || !y) return QC_ERR_INVALID_ARG;
    if (!(in_scale > 0.0f) || !std::isfinite(in_scale)) return QC_ERR_INVALID_ARG;
    if (qx.ws_total > 0 && (!workspace || ws_bytes < qx.ws_total)) return QC_ERR_WORKSPACE;
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    if (!qx.fused)
        if (!aligned16(x) || (workspace && !aligned16(workspace))) return QC_ERR_MISALIGNED;
    if (qx.fused) {
        if (is_packed_out(d->y_t) && (!multiplier || !shift)) return QC_ERR_INVALID_ARG;
        if (!aligned16(x) || !aligned16(w) || !aligned16(y) || (bias && !aligned16(bias)) ||
            (multiplier && !aligned16(multiplier)) || (shift && !aligned16(shift)))
            return QC_ERR_MISALIGNED;
        const void *w8 = w;
        if (qx.ex.wprep_needed) {
            s = prepare_weights_exec(qx.ex, w, workspace, st);
            if (s != QC_OK) return s;
            w8 = workspace;
        }
        return launch_fused_stem(qx, x, in_scale, w8, bias, multiplier, shift, y, st);
    }
    uint8_t *codes = static_cast<uint8_t *>(workspace);
    s = qconv_quantize_pack(x, xt, static_cast<int64_t>(d->n) * d->h * d->w, d->c, d->c, in_scale, d->x_zero,
                            d->x_t, codes, stream);
    if (s != QC_OK) return s;
    return forward_impl(&qx.dq, false, codes, w, bias, multiplier, shift, nullptr, y, codes + qx.codes_bytes,
                        ws_bytes - qx.codes_bytes, stream);
}

qc_status qconv_debug_plan_quantize(const qconv_desc *d, qc_ftype xt, qconv_plan *out) {
    if (!out) return QC_ERR_INVALID_ARG;
    QExec qx;
    qc_status s = derive_qexec(d, xt, &qx);
    if (s != QC_OK) return s;
    if (qx.fused) {
        fill_plan_out(qx.ex, qx.pl, out);
        out->prologue = qx.ex.prologue;
        return QC_OK;
    }
    s = qconv_debug_plan(&qx.dq, out);
    if (s == QC_OK) out->prologue |= 16;      // + the separate quantize launch
    return s;
}

qc_status qconv_debug_plan(const qconv_desc *d, qconv_plan *out) {
    if (!out) return QC_ERR_INVALID_ARG;
    Exec ex;
    qc_status s = derive_exec(d, true, &ex);
    if (s != QC_OK) return s;
    Plan pl;
    const Choice c = current_choice(d);
    if (!resolve(ex, c, &pl)) {
        if (c.kernel == QC_KERNEL_AUTO || !resolve(ex, Choice(), &pl)) return QC_ERR_UNSUPPORTED;
    }
    fill_plan_out(ex, pl, out);
    return QC_OK;
}

qc_status qconv_plan_set(const qconv_desc *d, const qconv_plan *choice) {
    Exec ex;
    qconv_desc tmp;          // 4-bit odd-C stems: validated on their byte-code view (the fused path)
    qc_status s = derive_exec_for_weights(d, &ex, &tmp);
    if (s != QC_OK) return s;
    const std::string key = desc_key(d);
    std::lock_guard<std::mutex> lk(g_plan_mu);
    if (!choice) {
        g_plans.erase(key);
        return QC_OK;
    }
    Choice c;
    c.kernel = choice->kernel;
    c.bn = choice->bn;
    Plan pl;
    if (c.kernel != QC_KERNEL_AUTO && !resolve(ex, c, &pl)) return QC_ERR_UNSUPPORTED;
    g_plans[key] = c;
    return QC_OK;
}

void qconv_plan_clear(void) {
    std::lock_guard<std::mutex> lk(g_plan_mu);
    g_plans.clear();
}

int32_t qconv_plan_candidates(const qconv_desc *d, qconv_plan *out, int32_t cap) {
    Exec ex;
    if (derive_exec(d, true, &ex) != QC_OK) return 0;
    const std::vector<Choice> cs = candidates(ex);
    for (int32_t i = 0; i < static_cast<int32_t>(cs.size()) && i < cap && out; ++i) {
        Plan pl;
        resolve(ex, cs[i], &pl);
        fill_plan_out(ex, pl, &out[i]);
    }
    return static_cast<int32_t>(cs.size());
}

qc_status qconv_autotune(const qconv_desc *d, const void *x, const void *w, const int32_t *bias,
                         const int32_t *multiplier, const int32_t *shift, void *y, void *workspace,
                         size_t ws_bytes, void *stream, int32_t iters, qconv_plan *best, float *best_us) {
    Exec ex;
    qc_status s = derive_exec(d, false, &ex);
    if (s != QC_OK) return s;
    if (iters < 1) return QC_ERR_INVALID_ARG;
    const std::vector<Choice> cs = candidates(ex);
    if (cs.empty()) return QC_ERR_UNSUPPORTED;
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    cudaEvent_t e0, e1;
    if (cudaEventCreate(&e0) != cudaSuccess || cudaEventCreate(&e1) != cudaSuccess) return cuda_fail(cudaGetLastError());
    float best_t = 0.0f;
    int best_i = -1;
    for (size_t i = 0; i < cs.size(); ++i) {
        g_forced = true;
        g_force = cs[i];
        s = qconv2d_forward(d, x, w, bias, multiplier, shift, y, workspace, ws_bytes, stream);   // warm-up
        if (s == QC_OK) {
            cudaEventRecord(e0, st);
            for (int it = 0; it < iters && s == QC_OK; ++it)
                s = qconv2d_forward(d, x, w, bias, multiplier, shift, y, workspace, ws_bytes, stream);
            cudaEventRecord(e1, st);
        }
        g_forced = false;
        if (s != QC_OK) break;
        cudaError_t err = cudaEventSynchronize(e1);
        if (err != cudaSuccess) { s = cuda_fail(err); break; }
        float ms = 0.0f;
        cudaEventElapsedTime(&ms, e0, e1);
        const float us = 1000.0f * ms / static_cast<float>(iters);
        if (best_i < 0 || us < best_t) { best_t = us; best_i = static_cast<int>(i); }
    }
    g_forced = false;
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    if (s != QC_OK) return s;
    qconv_plan chosen;
    std::memset(&chosen, 0, sizeof(chosen));
    chosen.kernel = cs[best_i].kernel;
    chosen.bn = cs[best_i].bn;
    s = qconv_plan_set(d, &chosen);
    if (s != QC_OK) return s;
    if (best) {
        Plan pl;
        resolve(ex, cs[best_i], &pl);
        fill_plan_out(ex, pl, best);
    }
    if (best_us) *best_us = best_t;
    return QC_OK;
}

// ------------------------------------------------------------------ space-to-depth stem
qc_status qconv_s2d_desc(const qconv_desc *d, qconv_desc *out) {
    if (!d) return QC_ERR_INVALID_ARG;
    // the original activations are float (quantized by qconv_quantize_pack_s2d), so an odd c
    // with a 4-bit code type is fine: validate the byte-container view
    qconv_desc dv = *d;
    dv.x_t = byte_container(d->x_t);
    Geometry g;
    qc_status s = validate_desc(&dv, &g, true);
    if (s != QC_OK) return s;
    if (!is_int_input(d->x_t) || d->x_zero < dtype_min(d->x_t) || d->x_zero > dtype_max(d->x_t))
        return QC_ERR_INVALID_ARG;
    if (!out) return QC_ERR_INVALID_ARG;
    if (d->stride_h != 2 || d->stride_w != 2 || d->dil_h != 1 || d->dil_w != 1) return QC_ERR_UNSUPPORTED;
    if (d->w_zero) return QC_ERR_UNSUPPORTED;
    *out = s2d_of(d, g);
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
    qc_status s = validate_desc(d, &g, true);
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
