// launch.h -- host-side launchers of the conv kernels, one translation unit per kernel
// family (k_*.cu) so the library builds in parallel.  Each launcher picks the template
// instantiation for the runtime (bits, output kind, zero-point) triple.
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>
#include "epilogue.cuh"

namespace qc {

struct Launch {
    dim3 grid;
    int threads = 0;
    uint32_t smem = 0;
    cudaStream_t stream = nullptr;
    bool pdl = true;       // programmatic dependent launch (ptx.cuh griddep_wait)
    int cluster = 1;       // CTAs per cluster (2 for the CTA-pair kernel)
};

cudaError_t launch_fwd(const Launch &L, bool is4, int out, bool zx, const CUtensorMap &xm,
                       const CUtensorMap &wm, const CUtensorMap &ym, const ConvParams &p);
cudaError_t launch_fwd2(const Launch &L, bool is4, int out, const CUtensorMap &xm, const CUtensorMap &wm,
                        const CUtensorMap &ym, const ConvParams &p);
cudaError_t launch_halo(const Launch &L, bool is4, int out, const CUtensorMap &hm, const CUtensorMap &bm,
                        const CUtensorMap &ym, const ConvParams &p, bool cm = false);
cudaError_t launch_trans(const Launch &L, bool is4, int out, bool m64, const CUtensorMap &xm,
                         const CUtensorMap &wm, const CUtensorMap &ym, const ConvParams &p);

// cudaFuncAttributeMaxDynamicSharedMemorySize is a per-device-context attribute: set once per
// (kernel, device), thread-safe (launch_common.cu).
cudaError_t ensure_smem_attr(const void *kern, int bytes);

// One launch of a conv kernel with the Launch attributes.
template <typename Kern>
cudaError_t launch_kernel(const Launch &L, Kern kern, const CUtensorMap &a, const CUtensorMap &b,
                          const CUtensorMap &c, const ConvParams &p) {
    cudaError_t e = ensure_smem_attr(reinterpret_cast<const void *>(kern), 227 * 1024);
    if (e != cudaSuccess) return e;
    cudaLaunchConfig_t cfg;
    memset(&cfg, 0, sizeof(cfg));
    cfg.gridDim = L.grid;
    cfg.blockDim = dim3(static_cast<unsigned>(L.threads));
    cfg.dynamicSmemBytes = L.smem;
    cfg.stream = L.stream;
    cudaLaunchAttribute attr[2];
    int na = 0;
    if (L.pdl) {
        attr[na].id = cudaLaunchAttributeProgrammaticStreamSerialization;
        attr[na].val.programmaticStreamSerializationAllowed = 1;
        ++na;
    }
    if (L.cluster > 1) {
        attr[na].id = cudaLaunchAttributeClusterDimension;
        attr[na].val.clusterDim.x = static_cast<unsigned>(L.cluster);
        attr[na].val.clusterDim.y = 1;
        attr[na].val.clusterDim.z = 1;
        ++na;
    }
    cfg.attrs = na ? attr : nullptr;
    cfg.numAttrs = static_cast<unsigned>(na);
    return cudaLaunchKernelEx(&cfg, kern, a, b, c, p);
}

}  // namespace qc

// Dispatch helper: OUT kind runtime value -> template argument.
#define QC_OUT_SWITCH(out, BODY)                                  \
    switch (out) {                                                \
        case qc::OUT_S32: { constexpr int O = qc::OUT_S32; BODY } \
        case qc::OUT_U8: { constexpr int O = qc::OUT_U8; BODY }   \
        case qc::OUT_S8: { constexpr int O = qc::OUT_S8; BODY }   \
        case qc::OUT_U4: { constexpr int O = qc::OUT_U4; BODY }   \
        case qc::OUT_S4: { constexpr int O = qc::OUT_S4; BODY }   \
        case qc::OUT_F32: { constexpr int O = qc::OUT_F32; BODY } \
        case qc::OUT_BF16: { constexpr int O = qc::OUT_BF16; BODY } \
        default: return cudaErrorInvalidValue;                    \
    }
#define QC_PACKED_OUT_SWITCH(out, BODY)                           \
    switch (out) {                                                \
        case qc::OUT_U8: { constexpr int O = qc::OUT_U8; BODY }   \
        case qc::OUT_S8: { constexpr int O = qc::OUT_S8; BODY }   \
        case qc::OUT_U4: { constexpr int O = qc::OUT_U4; BODY }   \
        case qc::OUT_S4: { constexpr int O = qc::OUT_S4; BODY }   \
        default: return cudaErrorInvalidValue;                    \
    }
