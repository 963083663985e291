// jacobi_tb.cu -- C1 Jacobi, temporally blocked: K sweeps per launch (SURVEY §8(f)
// NEXT-3 applied to the overhead-bound case the paper highlights: C1's
// microsecond sweeps are bound by launch latency and one halo exchange per sweep).
//
// Semantics: one launch = K consecutive sweeps of reading Q15's C1 (Dirichlet):
//   out[i][j] = 0.25 * (((in[i-1][j] + in[i+1][j]) + in[i][j-1]) + in[i][j+1])
// on interior cells; boundary cells keep their value (both buffers carry it).  An
// interior output cell depends on the cells within K of it, so a partition's read set
// is its box dilated by K (clamped to the grid; the square's corners are a read
// over-approximation of the dependency diamond) and its write set its own
// interior cells.
//
// Design: ghost-zone tiling in shared memory.  Logical block = 32 x 32 cells; a CTA of
// 512 threads loads the (32 + 2K)^2 window once (guarded to the grid; 1 MB grids stay in
// L2), runs K sweeps between two shared buffers -- sweep k computes the window shrunk by
// k, so the owned tile is exact after K -- and stores its interior cells.  Every cell of
// every sweep is the same expression on the same inputs as in jacobi2d, so the result is
// bit-identical to K jacobi2d launches and P-way launches are bit-identical to 1-way.
// Consecutive launches use programmatic dependent launch like jacobi2d.
#include <cuda_runtime.h>

#include "../runtime/builtins.h"
#include "launch_util.h"
#include "trace.cuh"
#include "common.cuh"

namespace pk {
namespace {

constexpr int kT = 32;          // owned tile (rows and columns)
constexpr int kMaxK = 16;       // sweeps per launch
constexpr int kThreads = 512;   // 32 columns x 16 rows of threads

// One CTA per logical block; KS = K is a template parameter so that the window side, the
// loop trip counts and the shared-memory offsets are compile-time constants (the loops
// unroll and the cells a thread handles in one sweep are independent instructions).
template <int KS, bool PUSH>
__global__ void __launch_bounds__(kThreads) k_jacobi2d_tb(const float* __restrict__ in, float* __restrict__ out,
                                                          int64_t H, int64_t W, int64_t K, pk_partition part,
                                                          PushList push) {
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    asm volatile("griddepcontrol.wait;" ::: "memory");
    constexpr int S = kT + 2 * KS;                 // window side
    extern __shared__ float sm[];
    const int64_t bx = part.min[0] + blockIdx.x, by = part.min[1] + blockIdx.y;  // Eq. 8
    const int64_t r0 = by * kT, c0 = bx * kT;
    if (r0 >= H || c0 >= W) return;                                                // block-uniform
    float* a = sm;
    float* b = sm + S * S;
    const int Hi = (int)H, Wi = (int)W, R0 = (int)r0 - KS, C0 = (int)c0 - KS;
    const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5;
#pragma unroll
    for (int i0 = 0; i0 < S; i0 += 16) {
        const int i = i0 + ty, r = R0 + i;
#pragma unroll
        for (int j0 = 0; j0 < S; j0 += 32) {
            const int j = j0 + tx, c = C0 + j;
            if (i < S && j < S) {
                float v = 0.f;
                if (r >= 0 && r < Hi && c >= 0 && c < Wi) {
                    v = in[(int64_t)r * W + c];
                    PK_TRACE_R(in + (int64_t)r * W + c, 4);
                }
                a[i * S + j] = v;
            }
        }
    }
    __syncthreads();
#ifndef PK_JTB_SUNROLL
#define PK_JTB_SUNROLL 1
#endif
#if PK_JTB_SUNROLL
#pragma unroll
#else
#pragma unroll 1
#endif
    for (int s = 1; s <= KS; ++s) {   // sweep s covers the window shrunk by s
#pragma unroll
        for (int i0 = s; i0 < S - s; i0 += 16) {
            const int i = i0 + ty, r = R0 + i;
            const bool rint = i < S - s && r >= 1 && r <= Hi - 2;
#pragma unroll
            for (int j0 = s; j0 < S - s; j0 += 32) {
                const int j = j0 + tx, c = C0 + j;
                if (i < S - s && j < S - s) {
                    const float* p = a + i * S + j;
                    float v = *p;   // boundary cells (and cells outside the grid, never read) keep their value
                    if (rint && c >= 1 && c <= Wi - 2)
                        v = __fmul_rn(0.25f, __fadd_rn(__fadd_rn(__fadd_rn(p[-S], p[S]), p[-1]), p[1]));
                    b[i * S + j] = v;
                }
            }
        }
        __syncthreads();
        float* t = a;
        a = b;
        b = t;
    }
#pragma unroll
    for (int i0 = 0; i0 < kT; i0 += 16) {
        const int i = i0 + ty, r = (int)r0 + i, c = (int)c0 + tx;
        if (r < 1 || r > Hi - 2 || c < 1 || c > Wi - 2) continue;
        float* o = out + (int64_t)r * W + c;
        const float v = a[(KS + i) * S + KS + tx];
        *o = v;
        PK_TRACE_W(o, 4);
        // fused halo push (PK_MODE_PUSH): only the rows a push range may cover (the K edge rows
        // of a partition) take the per-range check
        if (PUSH) {
            int64_t pa = 0, pb = 0;
            dev::push_rows(push, r0, r0 + kT, (uint64_t)W * 4u, &pa, &pb);
            if (dev::in_rows(r, pa, pb)) dev::push1(push, (uint64_t)((int64_t)r * W + c) * 4u, v);
        }
    }
}

template <int KS, bool P>
const void* tb_fn() { return (const void*)k_jacobi2d_tb<KS, P>; }
template <bool P>
const void* tb_fn_k(int64_t k) {
    switch (k) {
        case 1: return tb_fn<1, P>();   case 2: return tb_fn<2, P>();   case 3: return tb_fn<3, P>();
        case 4: return tb_fn<4, P>();   case 5: return tb_fn<5, P>();   case 6: return tb_fn<6, P>();
        case 7: return tb_fn<7, P>();   case 8: return tb_fn<8, P>();   case 9: return tb_fn<9, P>();
        case 10: return tb_fn<10, P>(); case 11: return tb_fn<11, P>(); case 12: return tb_fn<12, P>();
        case 13: return tb_fn<13, P>(); case 14: return tb_fn<14, P>(); case 15: return tb_fn<15, P>();
        case 16: return tb_fn<16, P>(); default: return nullptr;
    }
}

int describe_jacobi2d_tb(pk_ctx c, pk_kernel k) {
    // scalars: 0 = H, 1 = W, 2 = K.  Logical block (bx, by) = rows [32 by, +32) x columns
    // [32 bx, +32).  Reads the box dilated by K, clamped to the grid (positions
    // [32 b, 32 b + 32 + 2K) with the guard shifted by 2K, offset -K, clamped); writes its
    // interior cells (rows and columns in [1, n - 1)).
    const uint32_t f = PK_DIM_GUARD | PK_DIM_CLAMP;
    pk_affine_access a{};
    a.ndim = 2;
    a.dim[0] = DimMap(1, E(kT), S(2, 2, kT), S(2, -1), f, E(0), S(0, 1, 0));
    a.dim[0].guard_hi.c_scalar[2] = 2;   // H + 2K
    a.dim[1] = DimMap(0, E(kT), S(2, 2, kT), S(2, -1), f, E(0), S(1, 1, 0));
    a.dim[1].guard_hi.c_scalar[2] = 2;   // W + 2K
    if (int r = pk_declare_affine_access(c, k, 0, PK_READ, &a)) return r;
    pk_affine_access w{};
    w.ndim = 2;
    w.dim[0] = DimMap(1, E(kT), E(kT), E(0), PK_DIM_GUARD, E(1), S(0, 1, -1));
    w.dim[1] = DimMap(0, E(kT), E(kT), E(0), PK_DIM_GUARD, E(1), S(1, 1, -1));
    return pk_declare_affine_access(c, k, 1, PK_WRITE, &w);
}

cudaError_t launch_jacobi2d_tb(const LaunchInfo& li) {
    if (li.nscalars < 3) return cudaErrorInvalidValue;
    int64_t H = li.scalars[0], W = li.scalars[1], K = li.scalars[2];
    if (K < 1 || K > kMaxK || H < 1 || W < 1 || H >= (int64_t)1 << 30 || W >= (int64_t)1 << 30)
        return cudaErrorInvalidValue;
    const bool push = li.push && li.push->n > 0;
    const void* fn = push ? tb_fn_k<true>(K) : tb_fn_k<false>(K);
    PushList pl{};
    if (li.push) pl = *li.push;
    const size_t smem = (size_t)2 * (kT + 2 * K) * (kT + 2 * K) * sizeof(float);
    KernelDevInfo kd;
    if (cudaError_t e = prepare_kernel(fn, li.device, smem, kThreads, &kd)) return e;
    void* argv[] = {(void*)&li.inst[0], (void*)&li.inst[1], &H, &W, &K, (void*)&li.part, &pl};
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = li.grid;
    cfg.blockDim = dim3(kThreads);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = li.stream;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    return cudaLaunchKernelExC(&cfg, fn, argv);
}

}  // namespace

const Builtin kBuiltinJacobi2dTb = {
    "jacobi2d_tb", (const void*)k_jacobi2d_tb<1, false>, 5,
    {PK_ARG_BUFFER, PK_ARG_BUFFER, PK_ARG_SCALAR, PK_ARG_SCALAR, PK_ARG_SCALAR}, -1,
    describe_jacobi2d_tb, launch_jacobi2d_tb, /*push_arg=*/1};

}  // namespace pk
