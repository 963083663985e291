// heat_tma.cu -- C3 3-D 7-point heat stencil on sm_100a with a TMA plane ring.
//
// Same semantics, formula (reading Q15: u' = u + alpha((zm+zp+ym+yp+xm+xp) - 6u),
// replicate-clamped, alpha = 1/8) and logical block contract as heat3d_regs in
// stencils.cu: block (bx, by, bz) = 128 columns x bdy rows x ZC planes.
//
// Memory side: a ring of NS shared-memory planes, each holding the block's
// bdy + 2 rows (one halo row above and below, clamped) x (128 + 2 x 4) columns.
// Warp 0 streams whole row segments of plane z + NS - 2 with cp.async.bulk (TMA
// engine, one copy per row issued by the warp's lanes, one mbarrier per slot)
// while every warp computes plane z from slots z-1, z, z+1: all seven neighbours
// come from shared memory (x neighbours by warp shuffle + the column halo).  One
// barrier per plane releases the oldest slot.  Bytes in flight per CTA ~ (NS-3)
// planes, independent of registers.  Each input byte is fetched from HBM once,
// plus the two CTA-boundary halo rows (2/bdy) and two halo planes (2/ZC).
#include <cuda_runtime.h>

#include "../runtime/builtins.h"
#include "ptx.cuh"

namespace pk {
namespace {

constexpr float kAlpha = 0.125f;
constexpr int kMaxBdy = 32;
constexpr int kHalo = 4;
constexpr int kRowF = 128 + 2 * kHalo;  // floats per smem row (544 B, 16-B multiple)
constexpr int kNS = 6;                  // ring depth (planes)

__host__ __device__ constexpr size_t slot_floats(int bdy) { return (size_t)(bdy + 2) * kRowF; }
__host__ __device__ constexpr size_t smem_bytes(int bdy) { return kNS * slot_floats(bdy) * 4 + kNS * 8; }

__global__ void __launch_bounds__(1024) k_heat3d_tma(const float* __restrict__ uin, float* __restrict__ uout,
                                                    int64_t D, int64_t H, int64_t W, int64_t ZC,
                                                    pk_partition part) {
    extern __shared__ __align__(128) unsigned char smem[];
    const int bdy = blockDim.y;
    float* ring = reinterpret_cast<float*>(smem);
    uint64_t* full = reinterpret_cast<uint64_t*>(smem + kNS * slot_floats(bdy) * 4);
    const int lane = threadIdx.x, ty = threadIdx.y, warp = ty;
    const int64_t bx = part.min[0] + blockIdx.x, by = part.min[1] + blockIdx.y, bz = part.min[2] + blockIdx.z;
    const int64_t c0 = bx * 128, i0 = by * bdy, k0 = bz * ZC;
    if (c0 >= W || i0 >= H || k0 >= D) return;  // block-uniform
    const int64_t k1 = min(k0 + ZC, D);
    const int nz = (int)(k1 - k0);             // planes computed
    const int nq = nz + 2;                     // planes streamed: k0-1 .. k1 (clamped)
    const int64_t HW = H * W;
    // column segment [c0 - 4, c0 + 132) clipped to [0, W)
    const int64_t tlo = max(c0 - kHalo, (int64_t)0), thi = min(c0 + 128 + kHalo, W);
    const uint32_t rbytes = (uint32_t)(thi - tlo) * 4u;
    const int toff = (int)(tlo - (c0 - kHalo));
    const int nrows = bdy + 2;

    if (warp == 0 && lane == 0) {
        for (int s = 0; s < kNS; ++s) ptx::mbar_init(&full[s], 1);
        ptx::fence_mbar_init();
    }
    __syncthreads();

    // stream plane sequence index q (plane k0 - 1 + q, clamped) into slot q % kNS
    auto issue = [&](int q) {
        const int s = q % kNS;
        int64_t p = k0 - 1 + q;
        p = p < 0 ? 0 : (p >= D ? D - 1 : p);
        float* slot = ring + (size_t)s * slot_floats(bdy);
        if (lane == 0) ptx::mbar_arrive_expect_tx(&full[s], rbytes * (uint32_t)nrows);
        __syncwarp();
        for (int r = lane; r < nrows; r += 32) {
            int64_t row = i0 - 1 + r;
            row = row < 0 ? 0 : (row >= H ? H - 1 : row);
            ptx::bulk_g2s(slot + (size_t)r * kRowF + toff, uin + p * HW + row * W + tlo, rbytes, &full[s]);
        }
    };
    // fill every slot; after plane q is computed (barrier), slot (q - 1) % kNS is
    // refilled with sequence q - 1 + kNS, so sequences are issued in order
    if (warp == 0)
        for (int q = 0; q < kNS && q < nq; ++q) issue(q);

    const int64_t i = i0 + ty, j0 = c0 + 4 * lane;
    const bool active = i < H && j0 < W;
    const bool west_edge = j0 == 0, east_edge = j0 + 4 >= W;
    const int cx = kHalo + 4 * lane;
    ptx::mbar_wait(&full[0], 0);
    ptx::mbar_wait(&full[1 % kNS], (1 / kNS) & 1);
    for (int q = 1; q <= nz; ++q) {
        ptx::mbar_wait(&full[(q + 1) % kNS], ((q + 1) / kNS) & 1);
        const float* sm = ring + (size_t)((q - 1) % kNS) * slot_floats(bdy);
        const float* sc = ring + (size_t)(q % kNS) * slot_floats(bdy);
        const float* sp = ring + (size_t)((q + 1) % kNS) * slot_floats(bdy);
        const float4 c = *reinterpret_cast<const float4*>(sc + (ty + 1) * kRowF + cx);
        const float4 zm = *reinterpret_cast<const float4*>(sm + (ty + 1) * kRowF + cx);
        const float4 zp = *reinterpret_cast<const float4*>(sp + (ty + 1) * kRowF + cx);
        const float4 ym = *reinterpret_cast<const float4*>(sc + ty * kRowF + cx);
        const float4 yp = *reinterpret_cast<const float4*>(sc + (ty + 2) * kRowF + cx);
        float wv = __shfl_up_sync(0xffffffffu, c.w, 1);
        float ev = __shfl_down_sync(0xffffffffu, c.x, 1);
        if (lane == 0) wv = sc[(ty + 1) * kRowF + cx - 1];
        if (lane == 31) ev = sc[(ty + 1) * kRowF + cx + 4];
        if (west_edge) wv = c.x;
        if (east_edge) ev = c.w;
        if (active) {
            float4 o;
            o.x = c.x + kAlpha * ((zm.x + zp.x + ym.x + yp.x + wv + c.y) - 6.0f * c.x);
            o.y = c.y + kAlpha * ((zm.y + zp.y + ym.y + yp.y + c.x + c.z) - 6.0f * c.y);
            o.z = c.z + kAlpha * ((zm.z + zp.z + ym.z + yp.z + c.y + c.w) - 6.0f * c.z);
            o.w = c.w + kAlpha * ((zm.w + zp.w + ym.w + yp.w + c.z + ev) - 6.0f * c.w);
            *reinterpret_cast<float4*>(uout + (k0 + q - 1) * HW + i * W + j0) = o;
        }
        __syncthreads();  // everyone is done with slot (q - 1): refill it NS planes ahead
        const int qn = q - 1 + kNS;
        if (warp == 0 && qn < nq) issue(qn);
    }
}

int describe_heat3d_tma(pk_ctx c, pk_kernel k) {
    // identical contract to heat3d_regs (stencils.cu): scalars 0 = D, 1 = H, 2 = W, 3 = ZC
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

cudaError_t launch_heat3d_tma(const LaunchInfo& li) {
    if (li.nscalars < 4) return cudaErrorInvalidValue;
    int64_t D = li.scalars[0], H = li.scalars[1], W = li.scalars[2], ZC = li.scalars[3];
    if (W % 4 || W < 4 || ZC < 1 || li.block.x != 32 || li.block.y < 1 || li.block.y > kMaxBdy || li.block.z != 1)
        return cudaErrorInvalidValue;
    const size_t smem = smem_bytes(li.block.y);
    static bool attr = false;
    if (!attr) {
        cudaError_t e = cudaFuncSetAttribute(k_heat3d_tma, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                             (int)smem_bytes(kMaxBdy));
        if (e != cudaSuccess) return e;
        attr = true;
    }
    void* argv[] = {(void*)&li.inst[0], (void*)&li.inst[1], &D, &H, &W, &ZC, (void*)&li.part};
    return cudaLaunchKernel((const void*)k_heat3d_tma, li.grid, li.block, argv, smem, li.stream);
}

}  // namespace

const Builtin kBuiltinHeat3dTma = {
    "heat3d", (const void*)k_heat3d_tma, 6,
    {PK_ARG_BUFFER, PK_ARG_BUFFER, PK_ARG_SCALAR, PK_ARG_SCALAR, PK_ARG_SCALAR, PK_ARG_SCALAR}, -1,
    describe_heat3d_tma, launch_heat3d_tma};

}  // namespace pk
