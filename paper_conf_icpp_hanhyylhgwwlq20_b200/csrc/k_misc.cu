// k_misc.cu -- launchers of the CTA-pair (fwd2.cuh), halo (halo.cuh) and channel-major
// (trans.cuh) kernels, and the im2col dispatcher.
#include <cstring>
#include "launch.h"
#include "fwd2.cuh"

namespace qc {

cudaError_t launch_fwd_8(const Launch &L, int out, bool zx, const CUtensorMap &xm, const CUtensorMap &wm,
                         const CUtensorMap &ym, const ConvParams &p);
cudaError_t launch_fwd_4(const Launch &L, int out, bool zx, const CUtensorMap &xm, const CUtensorMap &wm,
                         const CUtensorMap &ym, const ConvParams &p);

cudaError_t launch_fwd(const Launch &L, bool is4, int out, bool zx, const CUtensorMap &xm,
                       const CUtensorMap &wm, const CUtensorMap &ym, const ConvParams &p) {
    return is4 ? launch_fwd_4(L, out, zx, xm, wm, ym, p) : launch_fwd_8(L, out, zx, xm, wm, ym, p);
}

cudaError_t launch_fwd2(const Launch &L, bool is4, int out, const CUtensorMap &xm, const CUtensorMap &wm,
                        const CUtensorMap &ym, const ConvParams &p) {
    if (is4) {
        QC_PACKED_OUT_SWITCH(out, return launch_kernel(L, qconv_fwd2_kernel<true, O>, xm, wm, ym, p);)
    }
    QC_PACKED_OUT_SWITCH(out, return launch_kernel(L, qconv_fwd2_kernel<false, O>, xm, wm, ym, p);)
}

}  // namespace qc
