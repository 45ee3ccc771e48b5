// k_halo.cu -- launcher of the stride-1 halo kernel (halo.cuh).
#include <cstring>
#include "launch.h"
#include "halo.cuh"

namespace qc {

cudaError_t launch_halo(const Launch &L, bool is4, int out, const CUtensorMap &hm, const CUtensorMap &bm,
                        const CUtensorMap &ym, const ConvParams &p, bool cm) {
    if (cm) {                 // channel-major variant (K = 64)
        if (p.f_c > 0) {
            QC_PACKED_OUT_SWITCH(out, return launch_kernel(L, qconv_halo_kernel<false, O, true, true>, hm, bm, ym, p);)
        }
        if (is4) {
            QC_PACKED_OUT_SWITCH(out, return launch_kernel(L, qconv_halo_kernel<true, O, false, true>, hm, bm, ym, p);)
        }
        QC_PACKED_OUT_SWITCH(out, return launch_kernel(L, qconv_halo_kernel<false, O, false, true>, hm, bm, ym, p);)
    }
    if (p.f_c > 0) {          // fused fp32 quantization (space-to-depth stem)
        QC_PACKED_OUT_SWITCH(out, return launch_kernel(L, qconv_halo_kernel<false, O, true>, hm, bm, ym, p);)
    }
    if (is4) {
        QC_PACKED_OUT_SWITCH(out, return launch_kernel(L, qconv_halo_kernel<true, O>, hm, bm, ym, p);)
    }
    QC_PACKED_OUT_SWITCH(out, return launch_kernel(L, qconv_halo_kernel<false, O>, hm, bm, ym, p);)
}

}  // namespace qc
