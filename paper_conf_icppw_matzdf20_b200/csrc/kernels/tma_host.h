// tma_host.h -- host-side TMA tensor-map encoding (cuTensorMapEncodeTiled through
// the runtime's driver entry point, so the library does not link libcuda directly).
#pragma once

#include <cuda.h>
#include <cuda_runtime.h>

#include <mutex>

namespace pk {

using EncodeTiledFn = CUresult (*)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                   const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                   CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

inline EncodeTiledFn tma_encode_fn() {
    static EncodeTiledFn fn = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
        void* p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = (EncodeTiledFn)p;
    });
    return fn;
}

// fp32 tensor of `rank` dims (dims[0] innermost), row-major strides, box `box`.
inline bool tma_encode_f32(CUtensorMap* m, const void* base, int rank, const cuuint64_t* dims, const cuuint32_t* box,
                           CUtensorMapSwizzle swz) {
    EncodeTiledFn enc = tma_encode_fn();
    if (!enc) return false;
    cuuint64_t strides[4];
    cuuint64_t s = 4;
    for (int d = 1; d < rank; ++d) {
        s *= dims[d - 1];
        strides[d - 1] = s;
    }
    cuuint32_t estr[5] = {1, 1, 1, 1, 1};
    return enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, (cuuint32_t)rank, const_cast<void*>(base), dims, strides, box, estr,
               CU_TENSOR_MAP_INTERLEAVE_NONE, swz, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

}  // namespace pk
