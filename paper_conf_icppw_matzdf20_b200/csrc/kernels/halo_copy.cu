// halo_copy.cu -- strided halo transfer on the SMs (a4 for tile partitions, NEXT-2).
//
// A tile partition's halo column is `rows` pieces of `len` bytes at a constant
// `pitch`, repeated over `nslab` slabs at a constant `slice` (3-D grids).  The
// copy engine moves such a column one narrow row at a time; here the
// destination's SMs pull it instead: one thread per 4-byte word (or byte),
// grid-stride, the source read through its peer pointer (NVLink/NVSwitch when
// the source lives on another GPU, peer access is enabled for every pair at
// pk_init), the destination written locally.  Launched on the destination's
// stream, so the event DAG of the copy engine path (RAW / WAR) applies unchanged.
#include <cstdint>

#include "runtime/builtins.h"

namespace pk {
namespace {

template <class T>
__global__ void __launch_bounds__(256) k_strided_copy(char* __restrict__ dst, const char* __restrict__ src,
                                                      uint64_t words_per_piece, uint64_t rows, uint64_t pitch,
                                                      uint64_t slice, uint64_t total) {
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < total;
         i += (uint64_t)gridDim.x * blockDim.x) {
        const uint64_t piece = i / words_per_piece, w = i - piece * words_per_piece;
        const uint64_t slab = piece / rows, r = piece - slab * rows;
        const uint64_t off = slab * slice + r * pitch + w * sizeof(T);
        *reinterpret_cast<T*>(dst + off) = *reinterpret_cast<const T*>(src + off);
    }
}

}  // namespace

cudaError_t launch_strided_copy(char* dst, const char* src, uint64_t len, uint64_t pitch, uint64_t rows,
                                uint64_t slice, uint64_t nslab, int sm_count, cudaStream_t stream) {
    const bool words = ((uintptr_t)dst | (uintptr_t)src | len | pitch | slice) % 4 == 0;
    const uint64_t wpp = words ? len / 4 : len;
    const uint64_t total = wpp * rows * nslab;
    if (total == 0) return cudaSuccess;
    const uint64_t want = (total + 255) / 256;
    const unsigned blocks = (unsigned)(want < (uint64_t)sm_count * 4 ? want : (uint64_t)sm_count * 4);
    if (words)
        k_strided_copy<uint32_t><<<blocks, 256, 0, stream>>>(dst, src, wpp, rows, pitch, slice, total);
    else
        k_strided_copy<uint8_t><<<blocks, 256, 0, stream>>>(dst, src, wpp, rows, pitch, slice, total);
    return cudaGetLastError();
}

}  // namespace pk
