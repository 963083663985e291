// nbody.cu -- all-pairs gravitational N-body step, partitioned over body blocks.
//
// PAPER.md P:L986-993 (§9.1 "direct gravitational N-Body simulation ...
// computation per thread grows [with] the problem size, while the data
// requirements per thread grow only linearly").  Reading Q16:
//   a_i = sum_j m_j d_ij (|d_ij|^2 + eps^2)^(-3/2),  d_ij = p_j - p_i,
//   v' = v + a dt,  x' = x + v' dt  (kick-drift Euler), G = 1.
// Positions are float4 (x, y, z, m) and ping-pong between launches; velocities
// are updated in place (each thread reads and writes only its own body).
//
// FP32-ALU bound (12 FP32-pipe ops + 1 MUFU per interaction): sources are staged
// in shared memory 256 at a time and broadcast to the warp; each thread keeps
// two bodies to double the FMA chains per shared-memory read.  Accumulation is
// two-level (partial sums over 1024-source chunks, then added into the total),
// which keeps the FP32 error of a 1M-term sum near 1e-6 (reading Q16).
#include <cuda_runtime.h>

#include "../runtime/builtins.h"

namespace pk {
namespace {

constexpr float kEps2 = 1e-4f;
constexpr float kDt = 1e-3f;
constexpr int kTile = 256;   // sources per shared-memory tile
constexpr int kChunk = 1024; // sources per partial sum
constexpr int kBodies = 2;   // bodies per thread

// Block = kThreads threads; block b owns bodies [b*kBodies*bdx, (b+1)*kBodies*bdx):
// thread t holds bodies base + t and base + t + bdx.
__global__ void __launch_bounds__(256) k_nbody(const float4* __restrict__ pin, float4* __restrict__ vel,
                                               float4* __restrict__ pout, int64_t N, pk_partition part) {
    __shared__ float4 sh[kTile];
    const int64_t bx = part.min[0] + blockIdx.x;  // Eq. 8
    const int64_t base = bx * (int64_t)kBodies * blockDim.x;
    float4 pi[kBodies];
    float ax[kBodies], ay[kBodies], az[kBodies];
#pragma unroll
    for (int u = 0; u < kBodies; ++u) {
        const int64_t i = base + threadIdx.x + u * (int64_t)blockDim.x;
        pi[u] = i < N ? pin[i] : make_float4(0.f, 0.f, 0.f, 0.f);
        ax[u] = ay[u] = az[u] = 0.f;
    }
    for (int64_t c0 = 0; c0 < N; c0 += kChunk) {
        float px[kBodies], py[kBodies], pz[kBodies];
#pragma unroll
        for (int u = 0; u < kBodies; ++u) px[u] = py[u] = pz[u] = 0.f;
        const int64_t c1 = c0 + kChunk < N ? c0 + kChunk : N;
        for (int64_t t0 = c0; t0 < c1; t0 += kTile) {
            __syncthreads();
            for (int s = threadIdx.x; s < kTile; s += blockDim.x) {
                const int64_t j = t0 + s;
                sh[s] = j < c1 ? pin[j] : make_float4(0.f, 0.f, 0.f, 0.f);  // m = 0 pads contribute 0
            }
            __syncthreads();
#pragma unroll 8
            for (int s = 0; s < kTile; ++s) {
                const float4 q = sh[s];
#pragma unroll
                for (int u = 0; u < kBodies; ++u) {
                    const float dx = q.x - pi[u].x, dy = q.y - pi[u].y, dz = q.z - pi[u].z;
                    const float r2 = fmaf(dx, dx, fmaf(dy, dy, fmaf(dz, dz, kEps2)));
                    const float inv = rsqrtf(r2);
                    const float sc = q.w * (inv * inv * inv);
                    px[u] = fmaf(dx, sc, px[u]);
                    py[u] = fmaf(dy, sc, py[u]);
                    pz[u] = fmaf(dz, sc, pz[u]);
                }
            }
        }
#pragma unroll
        for (int u = 0; u < kBodies; ++u) {
            ax[u] += px[u];
            ay[u] += py[u];
            az[u] += pz[u];
        }
    }
#pragma unroll
    for (int u = 0; u < kBodies; ++u) {
        const int64_t i = base + threadIdx.x + u * (int64_t)blockDim.x;
        if (i >= N) continue;
        float4 v = vel[i];
        v.x = fmaf(ax[u], kDt, v.x);
        v.y = fmaf(ay[u], kDt, v.y);
        v.z = fmaf(az[u], kDt, v.z);
        vel[i] = v;
        pout[i] = make_float4(fmaf(v.x, kDt, pi[u].x), fmaf(v.y, kDt, pi[u].y), fmaf(v.z, kDt, pi[u].z), pi[u].w);
    }
}

int describe_nbody(pk_ctx c, pk_kernel k) {
    // scalars: 0 = N.  Buffers are [N] float4 bodies.  Block b owns bodies
    // [b*2*bdx, (b+1)*2*bdx) n [0, N); it reads every body of pos_in.
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
    if (li.block.x > kTile || li.block.y != 1 || li.block.z != 1) return cudaErrorInvalidValue;
    void* argv[] = {(void*)&li.inst[0], (void*)&li.inst[1], (void*)&li.inst[2], &N, (void*)&li.part};
    return cudaLaunchKernel(li.fn, li.grid, li.block, argv, 0, li.stream);
}

}  // namespace

const Builtin kBuiltinNbody = {"nbody", (const void*)k_nbody, 4,
                               {PK_ARG_BUFFER, PK_ARG_BUFFER, PK_ARG_BUFFER, PK_ARG_SCALAR}, 0,
                               describe_nbody, launch_nbody};

}  // namespace pk
