// launch_common.cu -- per-(kernel, device) shared-memory attribute cache (launch.h).
#include <cstring>
#include <mutex>
#include <set>
#include <utility>

#include "launch.h"

namespace qc {

cudaError_t ensure_smem_attr(const void *kern, int bytes) {
    static std::mutex mu;
    static std::set<std::pair<const void *, int>> done;
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    const std::pair<const void *, int> key(kern, dev);
    {
        std::lock_guard<std::mutex> g(mu);
        if (done.count(key)) return cudaSuccess;
    }
    e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
    if (e != cudaSuccess) return e;
    std::lock_guard<std::mutex> g(mu);
    done.insert(key);
    return cudaSuccess;
}

}  // namespace qc
