// launch_util.cu -- see launch_util.h.
#include "launch_util.h"

#include <map>
#include <mutex>
#include <tuple>

namespace pk {

cudaError_t prepare_kernel(const void* fn, int dev, size_t smem, int threads, KernelDevInfo* out, bool occupancy) {
    static std::mutex mu;
    static std::map<std::tuple<const void*, int, size_t, int>, KernelDevInfo> done;
    std::lock_guard<std::mutex> g(mu);
    const auto key = std::make_tuple(fn, dev, smem, threads);
    auto it = done.find(key);
    if (it != done.end()) {
        *out = it->second;
        return cudaSuccess;
    }
    int cur = -1;
    cudaError_t e = cudaGetDevice(&cur);
    if (e != cudaSuccess) return e;
    if (cur != dev) return cudaErrorInvalidDevice;  // the attribute would land on another device
    if (smem > 48 * 1024) {
        e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
    }
    KernelDevInfo k;
    k.resident = 1;
    if (occupancy) {
        e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&k.resident, fn, threads, smem);
        if (e != cudaSuccess) return e;
    }
    e = cudaDeviceGetAttribute(&k.sms, cudaDevAttrMultiProcessorCount, dev);
    if (e != cudaSuccess) return e;
    if (k.resident < 1) return cudaErrorInvalidConfiguration;  // cannot be resident at all
    done[key] = k;
    *out = k;
    return cudaSuccess;
}

}  // namespace pk
