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

// Epoch flags of the peer-memory SPMD transport, SM variant (used when the driver
// refuses stream memory operations on a mapped peer address): one thread spins
// with system-scope acquire loads until every flag reaches its target / stores a
// flag with system-scope release after the stream's earlier work.
struct FlagWaitList {
    const unsigned long long* flag[8];
    unsigned long long target[8];
    int n;
};

__global__ void k_flag_wait(FlagWaitList w) {
    for (int i = 0; i < w.n; ++i) {
        unsigned long long v;
        do {
            asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(w.flag[i]) : "memory");
            if (v >= w.target[i]) break;
            __nanosleep(256);
        } while (true);
    }
}

__global__ void k_flag_write(unsigned long long* flag, unsigned long long v) {
    __threadfence_system();
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(flag), "l"(v) : "memory");
}

}  // namespace

cudaError_t launch_flag_wait(const uint64_t* const* flags, const uint64_t* targets, int n, cudaStream_t stream) {
    for (int i0 = 0; i0 < n; i0 += 8) {
        FlagWaitList w{};
        w.n = n - i0 < 8 ? n - i0 : 8;
        for (int i = 0; i < w.n; ++i) {
            w.flag[i] = reinterpret_cast<const unsigned long long*>(flags[i0 + i]);
            w.target[i] = targets[i0 + i];
        }
        k_flag_wait<<<1, 1, 0, stream>>>(w);
    }
    return cudaGetLastError();
}

cudaError_t launch_flag_write(uint64_t* flag, uint64_t v, cudaStream_t stream) {
    k_flag_write<<<1, 1, 0, stream>>>(reinterpret_cast<unsigned long long*>(flag), v);
    return cudaGetLastError();
}

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
