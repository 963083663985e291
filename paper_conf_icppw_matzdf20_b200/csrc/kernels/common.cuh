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
