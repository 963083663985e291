// common.cuh -- small device helpers shared by the sm_100a kernels.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include "pk_api.h"
#include "trace.cuh"

namespace pk {
namespace dev {

// Streaming read-only 16-byte load: the stencils read every input byte once, so
// keep it out of L1 (L2 still catches the neighbour-block halo re-reads).
__device__ __forceinline__ float4 ld_stream4(const float* p) {
    float4 r;
    asm("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
                 : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w)
                 : "l"(p));
    return r;
}
__device__ __forceinline__ float ld_nc(const float* p) {
    float r;
    asm("ld.global.nc.f32 %0, [%1];" : "=f"(r) : "l"(p));
    return r;
}
__device__ __forceinline__ float4 ld_l1(const float* p) {  // expect an L1 hit (re-read by a neighbour warp)
    float4 r;
    asm("ld.global.nc.v4.f32 {%0,%1,%2,%3}, [%4];"
                 : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w)
                 : "l"(p));
    return r;
}
__device__ __forceinline__ void st4(float* p, float4 v) {
    asm volatile("st.global.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(p), "f"(v.x), "f"(v.y), "f"(v.z), "f"(v.w)
                 : "memory");
}

}  // namespace dev
}  // namespace pk

#include "../runtime/builtins.h"

namespace pk {
namespace dev {
// Halo push (PK_MODE_PUSH): the value just stored at byte offset `off` of the output
// instance also goes to every destination instance whose push range covers it
// (4-byte granularity ranges; `n` is uniform, usually 0 or 2).
// (static indices only: a runtime-indexed by-value struct would be copied to local
// memory.  Kernels instantiate a PUSH=false variant without any of this.)
// The rows [r0, r1) of a row-major array (row = `pitch` bytes: a grid row, or a plane of
// a 3-D grid) whose bytes a push range may cover: the hull [*a, *b) of the intersecting
// rows (empty: *a == *b).  Computed once per tile; a store outside it skips push4's
// per-range checks, which on every store cost as much as the stencil update itself.
__device__ __forceinline__ void push_rows(const PushList& pl, int64_t r0, int64_t r1, uint64_t pitch, int64_t* a,
                                          int64_t* b) {
    int64_t lo = r1, hi = r0;
    for (int i = 0; i < kMaxPush; ++i) {
        if (i >= pl.n) break;
        if (pl.hi[i] <= pl.lo[i]) continue;
        const int64_t ra = (int64_t)(pl.lo[i] / pitch), rb = (int64_t)((pl.hi[i] - 1) / pitch) + 1;
        const int64_t x = ra > r0 ? ra : r0, y = rb < r1 ? rb : r1;
        if (x < y) {
            lo = x < lo ? x : lo;
            hi = y > hi ? y : hi;
        }
    }
    *a = lo < hi ? lo : r0;
    *b = lo < hi ? hi : r0;
}
__device__ __forceinline__ bool in_rows(int64_t r, int64_t a, int64_t b) { return (uint64_t)(r - a) < (uint64_t)(b - a); }

__device__ __forceinline__ void push4(const PushList& pl, uint64_t off, const float4& v) {
#pragma unroll
    for (int i = 0; i < kMaxPush; ++i)
        if (i < pl.n && off >= pl.lo[i] && off < pl.hi[i]) {
            *reinterpret_cast<float4*>(pl.dst[i] + off) = v;
            PK_TRACE_W((const void*)(pl.dst[i] + off), 16);
        }
}
__device__ __forceinline__ void push1(const PushList& pl, uint64_t off, float v) {
#pragma unroll
    for (int i = 0; i < kMaxPush; ++i)
        if (i < pl.n && off >= pl.lo[i] && off < pl.hi[i]) {
            *reinterpret_cast<float*>(pl.dst[i] + off) = v;
            PK_TRACE_W((const void*)(pl.dst[i] + off), 4);
        }
}
}  // namespace dev
}  // namespace pk
