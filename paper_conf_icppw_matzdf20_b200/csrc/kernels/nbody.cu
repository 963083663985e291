// nbody.cu -- all-pairs gravitational N-body step, partitioned over body blocks.
//
// PAPER.md P:L986-993 (§9.1 "direct gravitational N-Body simulation ...
// computation per thread grows [with] the problem size, while the data
// requirements per thread grow only linearly").  Reading Q16:
//   a_i = sum_j m_j d_ij (|d_ij|^2 + eps^2)^(-3/2),  d_ij = p_j - p_i,
//   v' = v + a dt,  x' = x + v' dt  (kick-drift Euler), G = 1.
// Positions are float4 (x, y, z, m) and ping-pong between launches; velocities
// are updated in place (each thread reads and writes only its own bodies).
//
// FP32-ALU / issue bound.  Sources are staged in shared memory 256 at a time,
// pre-duplicated as (x,x,y,y) (z,z,m,m) so that two LDS.128 broadcasts yield
// packed pairs; each thread owns 4 bodies as two f32x2 pairs and evaluates the
// interaction with Blackwell's packed FADD2/FFMA2/FMUL2 (one instruction per two
// bodies) + 2 MUFU.RSQ -- about 7 issued instructions per interaction instead of
// 13+.  Accumulation is two-level (partial sums over 1024-source chunks added
// into the total), keeping the FP32 error of a 1M-term sum near 1e-6 (Q16).
#include <cuda_runtime.h>
#include <stdint.h>

#include <mutex>
#include <unordered_map>
#include <utility>

#include "../runtime/builtins.h"
#include "launch_util.h"
#include "trace.cuh"

namespace pk {
namespace {

constexpr float kEps2 = 1e-4f;
constexpr float kDt = 1e-3f;
constexpr int kTile = 256;   // sources per shared-memory tile
constexpr int kChunk = 1024; // sources per partial sum
constexpr int kBodies = 4;   // bodies per thread = 2 packed pairs

typedef unsigned long long u64;

__device__ __forceinline__ u64 pk2(float a, float b) {
    u64 r;
    asm("mov.b64 %0, {%1,%2};" : "=l"(r) : "f"(a), "f"(b));
    return r;
}
__device__ __forceinline__ void up2(u64 v, float& a, float& b) { asm("mov.b64 {%0,%1}, %2;" : "=f"(a), "=f"(b) : "l"(v)); }
__device__ __forceinline__ u64 sub2(u64 a, u64 b) {
    u64 r;
    asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
    return r;
}
__device__ __forceinline__ u64 add2(u64 a, u64 b) {
    u64 r;
    asm("add.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
    return r;
}
__device__ __forceinline__ u64 mul2(u64 a, u64 b) {
    u64 r;
    asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
    return r;
}
__device__ __forceinline__ u64 fma2(u64 a, u64 b, u64 c) {
    u64 r;
    asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(r) : "l"(a), "l"(b), "l"(c));
    return r;
}
// r2 >= eps^2 = 1e-4 is never denormal, so the flush-to-zero MUFU.RSQ is exact
// enough and skips rsqrtf's denormal scaling (2 FMUL per call).
__device__ __forceinline__ u64 rsqrt2(u64 v) {
    // one asm block so that ptxas can keep both MUFU results in the register pair
    // (separate unpack / MUFU / pack statements cost ~3 MOVs per interaction)
    u64 r;
    asm("{\n\t.reg .f32 a, b;\n\t"
        "mov.b64 {a, b}, %1;\n\t"
        "rsqrt.approx.ftz.f32 a, a;\n\t"
        "rsqrt.approx.ftz.f32 b, b;\n\t"
        "mov.b64 %0, {a, b};\n\t}"
        : "=l"(r)
        : "l"(v));
    return r;
}

// Source split (fixed, independent of P and of the physical grid): the
// ceil(N / 1024) source chunks are cut into kSplit contiguous parts; part s of
// body i is accumulated chunk by chunk into partial[s][i]; the finalize kernel
// adds the kSplit partials in order s = 0..kSplit-1.  The persistent grid walks
// (logical block, part) items, so ~kSplit x more, smaller work items than blocks
// keep every SM busy to the end (no 2.3-wave tail).
#ifndef PK_NBODY_SPLIT
#define PK_NBODY_SPLIT 16
#endif
constexpr int kSplit = PK_NBODY_SPLIT;  // 16: 16384 items over 444 CTAs (measured 8/16/32: 2386/2396/2397)

__device__ __forceinline__ void part_chunks(int64_t N, int s, int64_t& c_begin, int64_t& c_end) {
    const int64_t nch = (N + kChunk - 1) / kChunk;
    c_begin = (nch * s) / kSplit * kChunk;
    c_end = (nch * (s + 1)) / kSplit * kChunk;
    if (c_end > N) c_end = N;
}

// Logical block = bdx threads owning bodies [b*4*bdx, (b+1)*4*bdx): thread t holds
// bodies base + t + u*bdx (u = 0..3).  The packed f32x2 lanes carry two SOURCES
// (even / odd within the tile) against a scalar body coordinate, which FADD2 /
// FFMA2 take as a free broadcast operand; each body accumulates two interleaved
// partial sums (even and odd sources) that are added at the end -- a fixed,
// position-only order.
// 2 CTAs/SM (125 registers, no spill) and the source loop unrolled 32-fold give the
// scheduler independent chains to cover the MUFU and FFMA2 latencies.  Measured
// (CTAs/SM, unroll) on C5: (3, 4) 2408, (2, 4) 2491, (2, 8) 2557, (2, 16) 2605,
// (2, 32) 2620, (2, 64) 2293, (1, 16) 2604 G interactions/s.
#ifndef PK_NBODY_MINB
#define PK_NBODY_MINB 2
#endif
#ifndef PK_NBODY_UNROLL
#define PK_NBODY_UNROLL 32
#endif
#define PK_PRAGMA(x) _Pragma(#x)
#define PK_UNROLL(n) PK_PRAGMA(unroll n)
__global__ void __launch_bounds__(256, PK_NBODY_MINB) k_nbody_partial(const float4* __restrict__ pin, float4* __restrict__ partial,
                                                       int64_t N, pk_partition part) {
    __shared__ float4 sh[kTile];  // kTile / 2 source pairs: (x0,x1,y0,y1), (z0,z1,m0,m1)
    const int64_t nb = part.max[0] - part.min[0];
    const int64_t nitems = nb * kSplit;
    const u64 zero = pk2(0.f, 0.f), eps = pk2(kEps2, kEps2);
    for (int64_t it = blockIdx.x; it < nitems; it += gridDim.x) {
        const int64_t bx = part.min[0] + it % nb;  // Eq. 8
        const int s_part = (int)(it / nb);
        const int64_t base = bx * (int64_t)kBodies * blockDim.x;
        u64 px[kBodies], py[kBodies], pz[kBodies], ax[kBodies], ay[kBodies], az[kBodies];
#pragma unroll
        for (int u = 0; u < kBodies; ++u) {
            const int64_t i = base + threadIdx.x + u * (int64_t)blockDim.x;
            const float4 p = i < N ? pin[i] : make_float4(0.f, 0.f, 0.f, 0.f);
            if (i < N) PK_TRACE_R(pin + i, 16);
            px[u] = pk2(p.x, p.x);  // broadcast pairs: ptxas uses the scalar .F32 operand form
            py[u] = pk2(p.y, p.y);
            pz[u] = pk2(p.z, p.z);
            ax[u] = ay[u] = az[u] = zero;
        }
        int64_t cb, ce;
        part_chunks(N, s_part, cb, ce);
        for (int64_t c0 = cb; c0 < ce; c0 += kChunk) {
            u64 sx[kBodies], sy[kBodies], sz[kBodies];
#pragma unroll
            for (int u = 0; u < kBodies; ++u) sx[u] = sy[u] = sz[u] = zero;
            const int64_t c1 = c0 + kChunk < N ? c0 + kChunk : N;
            for (int64_t t0 = c0; t0 < c1; t0 += kTile) {
                __syncthreads();
                for (int s = threadIdx.x; s < kTile / 2; s += blockDim.x) {
                    const int64_t j = t0 + 2 * s;
                    const float4 q0 = j < c1 ? pin[j] : make_float4(0.f, 0.f, 0.f, 0.f);  // m = 0 pads add 0
                    const float4 q1 = j + 1 < c1 ? pin[j + 1] : make_float4(0.f, 0.f, 0.f, 0.f);
                    if (j < c1) PK_TRACE_R(pin + j, 16);
                    if (j + 1 < c1) PK_TRACE_R(pin + j + 1, 16);
                    sh[2 * s] = make_float4(q0.x, q1.x, q0.y, q1.y);
                    sh[2 * s + 1] = make_float4(q0.z, q1.z, q0.w, q1.w);
                }
                __syncthreads();
                PK_UNROLL(PK_NBODY_UNROLL)
                for (int s = 0; s < kTile / 2; ++s) {
                    const float4 A = sh[2 * s], B = sh[2 * s + 1];
                    const u64 qx = pk2(A.x, A.y), qy = pk2(A.z, A.w), qz = pk2(B.x, B.y), qm = pk2(B.z, B.w);
#pragma unroll
                    for (int u = 0; u < kBodies; ++u) {
                        const u64 dx = sub2(qx, px[u]), dy = sub2(qy, py[u]), dz = sub2(qz, pz[u]);
                        const u64 r2 = fma2(dx, dx, fma2(dy, dy, fma2(dz, dz, eps)));
                        const u64 inv = rsqrt2(r2);
                        const u64 sc = mul2(qm, mul2(mul2(inv, inv), inv));
                        sx[u] = fma2(dx, sc, sx[u]);
                        sy[u] = fma2(dy, sc, sy[u]);
                        sz[u] = fma2(dz, sc, sz[u]);
                    }
                }
            }
#pragma unroll
            for (int u = 0; u < kBodies; ++u) {
                ax[u] = add2(ax[u], sx[u]);
                ay[u] = add2(ay[u], sy[u]);
                az[u] = add2(az[u], sz[u]);
            }
        }
#pragma unroll
        for (int u = 0; u < kBodies; ++u) {
            const int64_t i = base + threadIdx.x + u * (int64_t)blockDim.x;
            if (i >= N) continue;
            float a0, a1, b0, b1, c0_, c1_;
            up2(ax[u], a0, a1);
            up2(ay[u], b0, b1);
            up2(az[u], c0_, c1_);
            partial[(int64_t)s_part * N + i] = make_float4(a0 + a1, b0 + b1, c0_ + c1_, 0.f);
        }
        __syncthreads();  // the next item reuses the shared-memory tile
    }
}

// a_i = sum of the kSplit partials in order; kick-drift (reading Q16).
__global__ void __launch_bounds__(256) k_nbody_final(const float4* __restrict__ pin, float4* __restrict__ vel,
                                                     float4* __restrict__ pout, const float4* __restrict__ partial,
                                                     int64_t N, int64_t i0, int64_t i1) {
    const int64_t i = i0 + blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i >= i1) return;
    float4 a = partial[i];
#pragma unroll
    for (int s = 1; s < kSplit; ++s) {
        const float4 q = partial[(int64_t)s * N + i];
        a.x += q.x;
        a.y += q.y;
        a.z += q.z;
    }
    const float4 p = pin[i];
    float4 v = vel[i];
    PK_TRACE_R(pin + i, 16);
    PK_TRACE_R(vel + i, 16);
    v.x = fmaf(a.x, kDt, v.x);
    v.y = fmaf(a.y, kDt, v.y);
    v.z = fmaf(a.z, kDt, v.z);
    vel[i] = v;
    pout[i] = make_float4(fmaf(v.x, kDt, p.x), fmaf(v.y, kDt, p.y), fmaf(v.z, kDt, p.z), p.w);
    PK_TRACE_W(vel + i, 16);
    PK_TRACE_W(pout + i, 16);
}

int describe_nbody(pk_ctx c, pk_kernel k) {
    // scalars: 0 = N.  Buffers are [N] float4 bodies.  Block b owns bodies
    // [b*4*bdx, (b+1)*4*bdx) n [0, N); it reads every body of pos_in.
    pk_affine_access all{};
    all.ndim = 1;
    all.dim[0] = DimMap(-1, E(0), S(0), E(0), 0);
    if (int r = pk_declare_affine_access(c, k, 0, PK_READ, &all)) return r;
    pk_affine_access own{};
    own.ndim = 1;
    own.dim[0] = DimMap(0, BD(0, kBodies), BD(0, kBodies), E(0), PK_DIM_GUARD, E(0), S(0));
    if (int r = pk_declare_affine_access(c, k, 1, PK_MAY_WRITE, &own)) return r;
    return pk_declare_affine_access(c, k, 2, PK_WRITE, &own);
}

cudaError_t launch_nbody(const LaunchInfo& li) {
    if (li.nscalars < 1) return cudaErrorInvalidValue;
    int64_t N = li.scalars[0];
    if (li.block.x > kTile || li.block.x < 1 || li.block.y != 1 || li.block.z != 1) return cudaErrorInvalidValue;
    if (N < 1) return cudaSuccess;
    // the kSplit partial accelerations: context-owned scratch of this partition (grow-only,
    // never freed under a memoised graph that may replay into it)
    cudaError_t e = cudaSuccess;
    float4* partial = (float4*)context_scratch(li, 0, (size_t)kSplit * (size_t)N * sizeof(float4), &e);
    if (!partial) return e;
    KernelDevInfo kd;
    if ((e = prepare_kernel((const void*)k_nbody_partial, li.device, 0, (int)li.block.x, &kd)) != cudaSuccess) return e;
    const int64_t items = (int64_t)li.grid.x * kSplit;
    dim3 grid(persistent_grid(items, kd));
    void* argv[] = {(void*)&li.inst[0], &partial, &N, (void*)&li.part};
    e = cudaLaunchKernel((const void*)k_nbody_partial, grid, li.block, argv, 0, li.stream);
    if (e != cudaSuccess) return e;
    const int64_t per_block = (int64_t)kBodies * li.block.x;
    int64_t i0 = (int64_t)li.part.min[0] * per_block, i1 = (int64_t)li.part.max[0] * per_block;
    if (i1 > N) i1 = N;
    if (i1 <= i0) return cudaSuccess;
    void* argf[] = {(void*)&li.inst[0], (void*)&li.inst[1], (void*)&li.inst[2], &partial, &N, &i0, &i1};
    return cudaLaunchKernel((const void*)k_nbody_final, dim3((unsigned)((i1 - i0 + 255) / 256)), dim3(256), argf, 0,
                            li.stream);
}

}  // namespace

const Builtin kBuiltinNbody = {"nbody", (const void*)k_nbody_partial, 4,
                               {PK_ARG_BUFFER, PK_ARG_BUFFER, PK_ARG_BUFFER, PK_ARG_SCALAR}, 0,
                               describe_nbody, launch_nbody};

}  // namespace pk
