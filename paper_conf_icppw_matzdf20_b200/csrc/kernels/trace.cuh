// trace.cuh -- access recording of the builtin kernels (hard part H5).
//
// The paper requires write maps to be exact and allows read maps to over-approximate
// (P:L568-571); VAST-style tools clone the kernel to mark the memory it touches
// (P:L1231-1236).  In the library built with -DPK_TRACE_ACCESS (libpk_trace.so, see
// build.py) every builtin records, at 4-byte granularity, each global address it
//   reads  -- per plain load, or per TMA copy (the in-bounds part of the box), i.e.
//             what the kernel FETCHES, including halo over-fetch it never uses;
//   writes -- per store (partition stores and halo-push stores).
// into one read and one write bitmap per registered instance.  pk_trace_* in pk_api.h
// resets and fetches them; tests/test_gpu_trace.py compares them with pk_enumerate.
// In the product build the macros compile to nothing.
#pragma once

#include <stdint.h>

namespace pk {
namespace trace {

constexpr int kMaxInst = 256;

struct Table {
    int32_t n;
    int32_t pad;
    unsigned long long stray;            // accesses outside every registered instance
    uint64_t base[kMaxInst];             // instance [base, base + bytes)
    uint64_t bytes[kMaxInst];
    uint32_t* bits[kMaxInst][2];         // [i][0] fetched words, [i][1] written words
};

}  // namespace trace
}  // namespace pk

#ifdef PK_TRACE_ACCESS
extern __device__ pk::trace::Table g_pk_trace;  // defined in runtime.cu (relocatable device code)

namespace pk {
namespace trace {
__device__ inline void mark(const void* p, uint64_t nbytes, int kind) {
    if (nbytes == 0) return;
    const uint64_t a = (uint64_t)(uintptr_t)p;
    const int n = g_pk_trace.n;
    for (int i = 0; i < n; ++i) {
        const uint64_t b = g_pk_trace.base[i];
        if (a < b || a >= b + g_pk_trace.bytes[i]) continue;
        if (a + nbytes > b + g_pk_trace.bytes[i]) atomicAdd(&g_pk_trace.stray, 1ull);  // runs off the end
        uint32_t* bits = g_pk_trace.bits[i][kind];
        uint64_t w = (a - b) / 4, we = (a - b + nbytes + 3) / 4;
        const uint64_t lim = g_pk_trace.bytes[i] / 4;
        if (we > lim) we = lim;
        while (w < we) {  // one atomicOr per 32-word bitmap word
            const uint64_t word = w >> 5;
            const uint64_t hi = (word + 1) << 5 < we ? (word + 1) << 5 : we;
            const uint32_t lo_bit = (uint32_t)(w & 31), nb = (uint32_t)(hi - w);
            const uint32_t m = nb == 32 ? 0xffffffffu : (((1u << nb) - 1u) << lo_bit);
            atomicOr(&bits[word], m);
            w = hi;
        }
        return;
    }
    atomicAdd(&g_pk_trace.stray, 1ull);
}
// rows of a 2-D / 3-D box [x0, x0+nx) x [y0, y0+ny) of plane z of a (D, H, W) fp32 array,
// clipped to the array (what a tensor TMA with zero fill actually reads)
__device__ inline void mark_box(const float* base, int64_t H, int64_t W, int64_t x0, int64_t nx, int64_t y0,
                                int64_t ny, int64_t z) {
    const int64_t xa = x0 < 0 ? 0 : x0, xb = x0 + nx > W ? W : x0 + nx;
    if (xb <= xa) return;
    for (int64_t y = y0 < 0 ? 0 : y0; y < y0 + ny && y < H; ++y) mark(base + (z * H + y) * W + xa, (xb - xa) * 4, 0);
}
}  // namespace trace
}  // namespace pk
#define PK_TRACE_R(p, n) ::pk::trace::mark((p), (uint64_t)(n), 0)
#define PK_TRACE_W(p, n) ::pk::trace::mark((p), (uint64_t)(n), 1)
#define PK_TRACE_BOX(base, H, W, x0, nx, y0, ny, z) ::pk::trace::mark_box((base), (H), (W), (x0), (nx), (y0), (ny), (z))
#else
#define PK_TRACE_R(p, n) ((void)0)
#define PK_TRACE_W(p, n) ((void)0)
#define PK_TRACE_BOX(base, H, W, x0, nx, y0, ny, z) ((void)0)
#endif
