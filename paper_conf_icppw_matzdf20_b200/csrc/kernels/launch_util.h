// launch_util.h -- per-DEVICE kernel preparation shared by the builtin launchers.
//
// cudaFuncSetAttribute(MaxDynamicSharedMemorySize) and the occupancy it implies are
// properties of (function, device): one process driving several GPUs (the paper's
// single host program) must opt in on every device a partition runs on.
#pragma once

#include <cuda_runtime.h>
#include <stddef.h>

namespace pk {

struct KernelDevInfo {
    int resident = 0;  // CTAs per SM at the given block size / dynamic shared memory
    int sms = 0;       // SM count of the device
};

// On the CURRENT device (the runtime selects the partition's device before calling a
// launcher; `dev` must name it): raise fn's dynamic shared memory limit to `smem`
// (when above the 48 KB default) and compute its residency, once per (fn, dev, smem,
// threads).  Thread-safe.  Returns the first error of the attribute / occupancy calls.
// occupancy = false: only the attribute (cluster kernels, launched one tile per CTA).
cudaError_t prepare_kernel(const void* fn, int dev, size_t smem, int threads, KernelDevInfo* out,
                           bool occupancy = true);

// Persistent grid size: min(work items, resident CTAs x SMs).
inline unsigned persistent_grid(long long items, const KernelDevInfo& k) {
    const long long cap = (long long)(k.resident > 0 ? k.resident : 1) * (k.sms > 0 ? k.sms : 1);
    return (unsigned)(items < cap ? items : cap);
}

}  // namespace pk
