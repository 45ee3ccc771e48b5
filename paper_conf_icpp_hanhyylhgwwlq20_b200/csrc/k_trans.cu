// k_trans.cu -- launcher of the channel-major 1x1 kernel (trans.cuh).
#include <cstring>
#include "launch.h"
#include "trans.cuh"

namespace qc {

cudaError_t launch_trans(const Launch &L, bool is4, int out, bool m64, const CUtensorMap &xm,
                         const CUtensorMap &wm, const CUtensorMap &ym, const ConvParams &p) {
    if (is4) {
        if (m64) { QC_PACKED_OUT_SWITCH(out, return launch_kernel(L, qconv_t_kernel<true, O, true>, xm, wm, ym, p);) }
        QC_PACKED_OUT_SWITCH(out, return launch_kernel(L, qconv_t_kernel<true, O, false>, xm, wm, ym, p);)
    }
    if (m64) { QC_PACKED_OUT_SWITCH(out, return launch_kernel(L, qconv_t_kernel<false, O, true>, xm, wm, ym, p);) }
    QC_PACKED_OUT_SWITCH(out, return launch_kernel(L, qconv_t_kernel<false, O, false>, xm, wm, ym, p);)
}

}  // namespace qc
