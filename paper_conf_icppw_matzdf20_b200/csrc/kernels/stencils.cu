// stencils.cu -- sm_100a partitioned stencil kernels + their access descriptors.
//
// Every kernel takes a pk_partition as its last argument and runs only the
// thread blocks of [min, max) of the ORIGINAL grid: blockIdx' = min + blockIdx
// (Eq. 8); the full grid comes from part.grid (Eq. 9, reading
// Q10); the launch grid is max - min (Eq. 10).  Because every output element's
// arithmetic depends only on its global position, a P-way launch is
// bit-identical to the 1-way launch.
//
// All three are HBM-streaming kernels (no dense contraction, so no tensor
// cores): one 16-byte vector per thread per row/plane, loads issued one
// row/plane ahead of the arithmetic, horizontal neighbours exchanged with warp
// shuffles, vertical (and z) neighbours kept in a register window so that each
// input byte is fetched from HBM about once.  Formulas: DESIGN.md §3 (Q14, Q15).
#include <cuda_runtime.h>

#include <cstdlib>

#include "../runtime/builtins.h"
#include "common.cuh"

namespace pk {
namespace {

using dev::ld_l1;
using dev::ld_nc;
using dev::ld_stream4;
using dev::st4;

// ============================================================ C1 jacobi2d
// One thread per cell: i = by*bdy + ty, j = bx*bdx + tx; Dirichlet interior
//   out[i][j] = 0.25 * (((in[i-1][j] + in[i+1][j]) + in[i][j-1]) + in[i][j+1])
template <bool PUSH>
__global__ void __launch_bounds__(256) k_jacobi2d(const float* __restrict__ in, float* __restrict__ out,
                                                  int64_t H, int64_t W, pk_partition part, PushList push) {
    // programmatic dependent launch (launch_jacobi2d): let the next sweep's grid be scheduled
    // now, and wait here until the previous sweep's grid has completed and its stores are
    // visible -- before any load or store, so ping-pong RAW and WAR both stay ordered
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    asm volatile("griddepcontrol.wait;" ::: "memory");
    const int64_t bx = part.min[0] + blockIdx.x, by = part.min[1] + blockIdx.y;  // Eq. 8
    const int64_t i = by * blockDim.y + threadIdx.y, j = bx * blockDim.x + threadIdx.x;
    if (i < 1 || i > H - 2 || j < 1 || j > W - 2) return;
    const float n = in[(i - 1) * W + j], s = in[(i + 1) * W + j];
    const float w = in[i * W + j - 1], e = in[i * W + j + 1];
    PK_TRACE_R(in + (i - 1) * W + j, 4);
    PK_TRACE_R(in + (i + 1) * W + j, 4);
    PK_TRACE_R(in + i * W + j - 1, 4);
    PK_TRACE_R(in + i * W + j + 1, 4);
    const float v = __fmul_rn(0.25f, __fadd_rn(__fadd_rn(__fadd_rn(n, s), w), e));
    out[i * W + j] = v;
    PK_TRACE_W(out + i * W + j, 4);
    if (PUSH) dev::push1(push, (uint64_t)(i * W + j) * 4u, v);  // fused halo push
}

int describe_jacobi2d(pk_ctx c, pk_kernel k) {
    // scalars: 0 = H, 1 = W.  Threads on rows [1, H-1) x cols [1, W-1) (guard).
    const int32_t off[4][2] = {{-1, 0}, {1, 0}, {0, -1}, {0, 1}};
    for (int t = 0; t < 5; ++t) {
        pk_affine_access a{};
        a.ndim = 2;
        int di = t < 4 ? off[t][0] : 0, dj = t < 4 ? off[t][1] : 0;
        a.dim[0] = DimMap(1, BD(1), BD(1), E(di), PK_DIM_GUARD, E(1), S(0, 1, -1));
        a.dim[1] = DimMap(0, BD(0), BD(0), E(dj), PK_DIM_GUARD, E(1), S(1, 1, -1));
        int r = pk_declare_affine_access(c, k, t < 4 ? 0 : 1, t < 4 ? PK_READ : PK_WRITE, &a);
        if (r) return r;
    }
    return PK_OK;
}

cudaError_t launch_jacobi2d(const LaunchInfo& li) {
    if (li.nscalars < 2) return cudaErrorInvalidValue;
    int64_t H = li.scalars[0], W = li.scalars[1];
    PushList pl{};
    if (li.push) pl = *li.push;
    void* argv[] = {(void*)&li.inst[0], (void*)&li.inst[1], &H, &W, (void*)&li.part, &pl};
    const void* fn = (li.push && li.push->n > 0) ? (const void*)k_jacobi2d<true> : (const void*)k_jacobi2d<false>;
    // C1 sweeps are microsecond kernels: with programmatic stream serialisation the next
    // sweep's launch overlaps this one (only a kernel directly after a kernel in the same
    // stream is affected; copies and event waits keep their full dependencies)
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = li.grid;
    cfg.blockDim = li.block;
    cfg.dynamicSmemBytes = 0;
    cfg.stream = li.stream;
    cfg.attrs = at;
    static const bool no_pdl = getenv("PK_NO_PDL") != nullptr;   // A/B switch (scripts/r02/gpu_39.sh)
    cfg.numAttrs = no_pdl ? 0 : 1;
    return cudaLaunchKernelExC(&cfg, fn, argv);
}

// ============================================================ C2 hotspot2d
// Rodinia-form hotspot, constants frozen at the N = 1024 values (reading Q14).
constexpr float kCap = 4096.0f / 3000.0f;  // step / Cap
constexpr float kRx1 = 0.1f, kRy1 = 0.1f;
constexpr float kRz1 = 1.0f / 20480.0f;
constexpr float kAmb = 80.0f;

struct Row4 {
    float4 c;   // columns j0 .. j0+3
    float w, e; // column j0-1 (lane 0 only) and j0+4 (lane 31 only), clamped
};

// we = the row will be a centre row (its W/E halo columns are used); halo rows above and
// below the block are only read straight up / down (no diagonal reads, as declared)
__device__ __forceinline__ Row4 load_row(const float* __restrict__ t, int64_t r, int64_t W, int64_t jl,
                                         int64_t jw, int64_t je, int lane, bool we) {
    Row4 x;
    const float* row = t + r * W;
    x.c = ld_stream4(row + jl);
    x.w = we && lane == 0 ? ld_nc(row + jw) : 0.f;
    x.e = we && lane == 31 ? ld_nc(row + je) : 0.f;
    PK_TRACE_R(row + jl, 16);
    if (we && lane == 0) PK_TRACE_R(row + jw, 4);
    if (we && lane == 31) PK_TRACE_R(row + je, 4);
    return x;
}

__device__ __forceinline__ float hs(float c, float n, float s, float e, float w, float p) {
    return c + kCap * (p + (s + n - 2.0f * c) * kRy1 + (e + w - 2.0f * c) * kRx1 + (kAmb - c) * kRz1);
}

// Block = bdx threads (multiple of 32); thread owns 4 columns j0 = bx*4*bdx + 4*tx
// and marches the TY rows [by*TY, by*TY + TY) of its column strip.
__global__ void __launch_bounds__(128) k_hotspot2d(const float* __restrict__ tin, const float* __restrict__ pw,
                                                   float* __restrict__ tout, int64_t H, int64_t W, int64_t TY,
                                                   pk_partition part) {
    const int64_t bx = part.min[0] + blockIdx.x, by = part.min[1] + blockIdx.y;  // Eq. 8
    const int lane = threadIdx.x & 31;
    const int64_t j0 = bx * (4 * (int64_t)blockDim.x) + 4 * (int64_t)threadIdx.x;
    const int64_t wfirst = j0 - 4 * lane;
    if (wfirst >= W) return;                                    // whole warp outside: warp-uniform
    const int64_t r0 = by * TY;
    if (r0 >= H) return;                                        // block-uniform
    const int64_t r1 = min(r0 + TY, H);
    const bool active = j0 < W;
    const int64_t jl = active ? j0 : W - 4;                     // shuffle partner still loads in-bounds
    const int64_t jw = jl > 0 ? jl - 1 : 0, je = jl + 4 < W ? jl + 4 : W - 1;
    const bool west_edge = jl == 0, east_edge = jl + 4 >= W;

    Row4 N = load_row(tin, r0 > 0 ? r0 - 1 : 0, W, jl, jw, je, lane, false);
    Row4 C = load_row(tin, r0, W, jl, jw, je, lane, true);
    Row4 S = load_row(tin, r0 + 1 < H ? r0 + 1 : H - 1, W, jl, jw, je, lane, r0 + 1 < r1);
    float4 P = ld_stream4(pw + r0 * W + jl);
    PK_TRACE_R(pw + r0 * W + jl, 16);
    for (int64_t r = r0; r < r1; ++r) {
        // prefetch the row after next and the next power row
        Row4 S2 = S;
        float4 P2 = P;
        if (r + 1 < r1) {
            S2 = load_row(tin, r + 2 < H ? r + 2 : H - 1, W, jl, jw, je, lane, r + 2 < r1);
            P2 = ld_stream4(pw + (r + 1) * W + jl);
            PK_TRACE_R(pw + (r + 1) * W + jl, 16);
        }
        float wv = __shfl_up_sync(0xffffffffu, C.c.w, 1);
        float ev = __shfl_down_sync(0xffffffffu, C.c.x, 1);
        if (lane == 0) wv = C.w;
        if (lane == 31) ev = C.e;
        if (west_edge) wv = C.c.x;
        if (east_edge) ev = C.c.w;
        float4 o;
        o.x = hs(C.c.x, N.c.x, S.c.x, C.c.y, wv, P.x);
        o.y = hs(C.c.y, N.c.y, S.c.y, C.c.z, C.c.x, P.y);
        o.z = hs(C.c.z, N.c.z, S.c.z, C.c.w, C.c.y, P.z);
        o.w = hs(C.c.w, N.c.w, S.c.w, ev, C.c.z, P.w);
        if (active) {
            st4(tout + r * W + j0, o);
            PK_TRACE_W(tout + r * W + j0, 16);
        }
        N = C;
        C = S;
        S = S2;
        P = P2;
    }
}

int describe_hotspot2d(pk_ctx c, pk_kernel k) {
    // scalars: 0 = H, 1 = W, 2 = TY (rows per block).  Block (bx, by) owns rows
    // [by*TY, by*TY+TY) and columns [bx*4*bdx, bx*4*bdx + 4*bdx), guarded to the grid.
    const int32_t off[5][2] = {{0, 0}, {-1, 0}, {1, 0}, {0, -1}, {0, 1}};
    const uint32_t f = PK_DIM_GUARD | PK_DIM_CLAMP;
    for (int t = 0; t < 5; ++t) {
        pk_affine_access a{};
        a.ndim = 2;
        a.dim[0] = DimMap(1, S(2), S(2), E(off[t][0]), f, E(0), S(0));
        a.dim[1] = DimMap(0, BD(0, 4), BD(0, 4), E(off[t][1]), f, E(0), S(1));
        if (int r = pk_declare_affine_access(c, k, 0, PK_READ, &a)) return r;
        if (t == 0) {
            if (int r = pk_declare_affine_access(c, k, 1, PK_READ, &a)) return r;
            if (int r = pk_declare_affine_access(c, k, 2, PK_WRITE, &a)) return r;
        }
    }
    return PK_OK;
}

cudaError_t launch_hotspot2d(const LaunchInfo& li) {
    if (li.nscalars < 3) return cudaErrorInvalidValue;
    int64_t H = li.scalars[0], W = li.scalars[1], TY = li.scalars[2];
    if (W % 4 || W < 4 || TY < 1 || li.block.x % 32 || li.block.y != 1 || li.block.z != 1)
        return cudaErrorInvalidValue;
    void* argv[] = {(void*)&li.inst[0], (void*)&li.inst[1], (void*)&li.inst[2], &H, &W, &TY, (void*)&li.part};
    return cudaLaunchKernel(li.fn, li.grid, li.block, argv, 0, li.stream);
}

// ============================================================ C3 heat3d
constexpr float kAlpha = 0.125f;  // reading Q15

struct Pl4 {
    float4 c;
    float w, e;
};

__device__ __forceinline__ Pl4 load_pl(const float* __restrict__ u, int64_t off, int64_t jl, int64_t jw, int64_t je,
                                       int lane) {
    Pl4 x;
    x.c = ld_stream4(u + off + jl);
    x.w = lane == 0 ? ld_nc(u + off + jw) : 0.f;
    x.e = lane == 31 ? ld_nc(u + off + je) : 0.f;
    PK_TRACE_R(u + off + jl, 16);
    if (lane == 0) PK_TRACE_R(u + off + jw, 4);
    if (lane == 31) PK_TRACE_R(u + off + je, 4);
    return x;
}

// Block = (32, bdy <= kHeatMaxBdy): warp ty owns row i = by*bdy + ty, 128 columns
// j0 = bx*128 + 4*tx, and marches the ZC planes [bz*ZC, bz*ZC + ZC).  The z
// neighbours live in a per-thread register window; the y neighbours are the
// adjacent warps' centre rows, exchanged through a double-buffered shared-memory
// plane (one barrier per plane keeps the CTA's warps in lock-step, so every input
// row is fetched from HBM once); only the two CTA-boundary halo rows are loaded
// extra (by warps 0 and bdy-1), one plane ahead.
constexpr int kHeatMaxBdy = 32;

__global__ void __launch_bounds__(1024) k_heat3d(const float* __restrict__ uin, float* __restrict__ uout,
                                                int64_t D, int64_t H, int64_t W, int64_t ZC, pk_partition part) {
    __shared__ float4 ysh[2][kHeatMaxBdy + 2][32];
    const int64_t bx = part.min[0] + blockIdx.x, by = part.min[1] + blockIdx.y, bz = part.min[2] + blockIdx.z;
    const int lane = threadIdx.x;  // blockDim.x == 32
    const int ty = threadIdx.y, bdy = blockDim.y;
    const int64_t i = by * bdy + ty;
    const int64_t j0 = bx * 128 + 4 * (int64_t)lane;
    const int64_t k0 = bz * ZC;
    if (bx * 128 >= W || by * bdy >= H || k0 >= D) return;     // block-uniform
    const int64_t k1 = min(k0 + ZC, D);
    const bool active = j0 < W && i < H;
    const int64_t il = i < H ? i : H - 1;                       // rows past H mirror the last row
    const int64_t jl = j0 < W ? j0 : W - 4;
    const int64_t jw = jl > 0 ? jl - 1 : 0, je = jl + 4 < W ? jl + 4 : W - 1;
    const bool west_edge = jl == 0, east_edge = jl + 4 >= W;
    const int64_t HW = H * W;
    const int64_t rowc = il * W;
    // CTA-boundary halo rows (clamped): warp 0 fetches row i0-1, warp bdy-1 row i0+bdy
    const bool halo_lo = ty == 0, halo_hi = ty == bdy - 1;
    const int64_t i0 = by * bdy;
    const int64_t rowh = halo_lo ? (i0 > 0 ? i0 - 1 : 0) * W : (i0 + bdy < H ? i0 + bdy : H - 1) * W;

    Pl4 Zm = load_pl(uin, (k0 > 0 ? k0 - 1 : 0) * HW + rowc, jl, jw, je, lane);
    Pl4 Zc = load_pl(uin, k0 * HW + rowc, jl, jw, je, lane);
    Pl4 Zp = load_pl(uin, (k0 + 1 < D ? k0 + 1 : D - 1) * HW + rowc, jl, jw, je, lane);
    float4 Hr = make_float4(0.f, 0.f, 0.f, 0.f);
    if (halo_lo || halo_hi) {
        Hr = ld_stream4(uin + k0 * HW + rowh + jl);
        PK_TRACE_R(uin + k0 * HW + rowh + jl, 16);
    }
    int buf = 0;
    for (int64_t k = k0; k < k1; ++k) {
        Pl4 Zn = Zp;
        float4 Hn = Hr;
        if (k + 1 < k1) {
            Zn = load_pl(uin, (k + 2 < D ? k + 2 : D - 1) * HW + rowc, jl, jw, je, lane);
            if (halo_lo || halo_hi) {
                Hn = ld_stream4(uin + (k + 1) * HW + rowh + jl);
                PK_TRACE_R(uin + (k + 1) * HW + rowh + jl, 16);
            }
        }
        ysh[buf][ty + 1][lane] = Zc.c;
        if (halo_lo) ysh[buf][0][lane] = Hr;
        if (halo_hi) ysh[buf][bdy + 1][lane] = Hr;
        __syncthreads();
        const float4 Ym = ysh[buf][ty][lane];
        const float4 Yp = ysh[buf][ty + 2][lane];
        buf ^= 1;
        float wv = __shfl_up_sync(0xffffffffu, Zc.c.w, 1);
        float ev = __shfl_down_sync(0xffffffffu, Zc.c.x, 1);
        if (lane == 0) wv = Zc.w;
        if (lane == 31) ev = Zc.e;
        if (west_edge) wv = Zc.c.x;
        if (east_edge) ev = Zc.c.w;
        float4 o;
        const float4 c = Zc.c;
        o.x = c.x + kAlpha * ((Zm.c.x + Zp.c.x + Ym.x + Yp.x + wv + c.y) - 6.0f * c.x);
        o.y = c.y + kAlpha * ((Zm.c.y + Zp.c.y + Ym.y + Yp.y + c.x + c.z) - 6.0f * c.y);
        o.z = c.z + kAlpha * ((Zm.c.z + Zp.c.z + Ym.z + Yp.z + c.y + c.w) - 6.0f * c.z);
        o.w = c.w + kAlpha * ((Zm.c.w + Zp.c.w + Ym.w + Yp.w + c.z + ev) - 6.0f * c.w);
        if (active) {
            st4(uout + k * HW + rowc + j0, o);
            PK_TRACE_W(uout + k * HW + rowc + j0, 16);
        }
        Zm = Zc;
        Zc = Zp;
        Zp = Zn;
        Hr = Hn;
    }
}

int describe_heat3d(pk_ctx c, pk_kernel k) {
    // scalars: 0 = D, 1 = H, 2 = W, 3 = ZC.  Block (bx, by, bz) owns planes
    // [bz*ZC, +ZC), rows [by*bdy, +bdy), columns [bx*4*bdx, +4*bdx), guarded.
    const int32_t off[7][3] = {{0, 0, 0}, {-1, 0, 0}, {1, 0, 0}, {0, -1, 0}, {0, 1, 0}, {0, 0, -1}, {0, 0, 1}};
    const uint32_t f = PK_DIM_GUARD | PK_DIM_CLAMP;
    for (int t = 0; t < 7; ++t) {
        pk_affine_access a{};
        a.ndim = 3;
        a.dim[0] = DimMap(2, S(3), S(3), E(off[t][0]), f, E(0), S(0));
        a.dim[1] = DimMap(1, BD(1), BD(1), E(off[t][1]), f, E(0), S(1));
        a.dim[2] = DimMap(0, BD(0, 4), BD(0, 4), E(off[t][2]), f, E(0), S(2));
        if (int r = pk_declare_affine_access(c, k, 0, PK_READ, &a)) return r;
        if (t == 0)
            if (int r = pk_declare_affine_access(c, k, 1, PK_WRITE, &a)) return r;
    }
    return PK_OK;
}

cudaError_t launch_heat3d(const LaunchInfo& li) {
    if (li.nscalars < 4) return cudaErrorInvalidValue;
    int64_t D = li.scalars[0], H = li.scalars[1], W = li.scalars[2], ZC = li.scalars[3];
    if (W % 4 || W < 4 || ZC < 1 || li.block.x != 32 || li.block.y < 2 || li.block.y > kHeatMaxBdy ||
        li.block.z != 1)
        return cudaErrorInvalidValue;
    void* argv[] = {(void*)&li.inst[0], (void*)&li.inst[1], &D, &H, &W, &ZC, (void*)&li.part};
    return cudaLaunchKernel(li.fn, li.grid, li.block, argv, 0, li.stream);
}

}  // namespace

const Builtin kBuiltinJacobi2d = {
    "jacobi2d", (const void*)k_jacobi2d<false>, 4,
    {PK_ARG_BUFFER, PK_ARG_BUFFER, PK_ARG_SCALAR, PK_ARG_SCALAR}, -1, describe_jacobi2d, launch_jacobi2d,
    /*push_arg=*/1};
const Builtin kBuiltinHotspot2d = {
    "hotspot2d_regs", (const void*)k_hotspot2d, 6,
    {PK_ARG_BUFFER, PK_ARG_BUFFER, PK_ARG_BUFFER, PK_ARG_SCALAR, PK_ARG_SCALAR, PK_ARG_SCALAR}, -1,
    describe_hotspot2d, launch_hotspot2d};
const Builtin kBuiltinHeat3d = {
    "heat3d_regs", (const void*)k_heat3d, 6,
    {PK_ARG_BUFFER, PK_ARG_BUFFER, PK_ARG_SCALAR, PK_ARG_SCALAR, PK_ARG_SCALAR, PK_ARG_SCALAR}, -1,
    describe_heat3d, launch_heat3d};

}  // namespace pk
