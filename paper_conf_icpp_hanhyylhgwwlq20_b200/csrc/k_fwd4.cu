// k_fwd4.cu -- launcher of the im2col kernel (conv_fwd.cuh) for 4-bit activations.
#include <cstring>
#include "launch.h"
#include "conv_fwd.cuh"

namespace qc {

cudaError_t launch_fwd_4(const Launch &L, int out, bool zx, const CUtensorMap &xm, const CUtensorMap &wm,
                          const CUtensorMap &ym, const ConvParams &p) {
    if (zx) {
        QC_OUT_SWITCH(out, return launch_kernel(L, qconv_fwd_kernel<true, O, true>, xm, wm, ym, p);)
    }
    QC_OUT_SWITCH(out, return launch_kernel(L, qconv_fwd_kernel<true, O, false>, xm, wm, ym, p);)
}

}  // namespace qc
