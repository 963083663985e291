// hotspot_tma.cu -- C2 Hotspot on sm_100a: persistent CTAs, TMA bulk-copy row ring.
//
// Same semantics, formula and logical block contract as hotspot2d_regs in
// stencils.cu (reading Q14; block (bx, by) = columns [512 bx, 512 bx + 512) x rows
// [TY by, TY by + TY)), but the memory side is Blackwell-native:
//   * one producer thread per CTA streams each row segment (temp with a 4-float
//     halo on both sides, and power) with cp.async.bulk through the TMA engine
//     into an NS-stage shared-memory ring guarded by mbarriers (full: tx bytes;
//     empty: 4 consumer-warp arrivals) -- the bytes in flight no longer depend on
//     registers or occupancy;
//   * 4 consumer warps (128 threads x 4 columns) compute row r from ring stages
//     r-1, r, r+1; horizontal neighbours come from warp shuffles + the halo;
//   * the grid is persistent (min(tiles, SMs x resident CTAs)) and walks the
//     partition's logical blocks [min, max) (Eq. 8-10) in row-major tile order;
//     odd tile rows march upwards so that both tiles sharing a boundary touch the
//     halo rows at the same time (the second read hits L2).
// Because every output element's arithmetic is position-only, P-way results
// are bit-identical to 1-way.
#include <cuda_runtime.h>

#include "../runtime/builtins.h"
#include "launch_util.h"
#include "common.cuh"
#include "ptx.cuh"

namespace pk {
namespace {

constexpr float kCap = 4096.0f / 3000.0f;
constexpr float kRx1 = 0.1f, kRy1 = 0.1f;
constexpr float kRz1 = 1.0f / 20480.0f;
constexpr float kAmb = 80.0f;

constexpr int kTC = 512;                    // columns per tile (128 threads x 4)
constexpr int kHalo = 4;                    // halo floats each side (keeps 16-B alignment)
constexpr int kTRow = kTC + 2 * kHalo;      // temp floats per stage
constexpr int kStageFloats = kTRow + kTC;   // temp + power
constexpr int kStageBytes = kStageFloats * 4;
constexpr int kNS = 8;                      // ring depth
constexpr int kConsumers = 128;
constexpr int kThreads = kConsumers + 32;   // + producer warp
constexpr size_t kSmem = (size_t)kNS * kStageBytes + 2 * kNS * sizeof(uint64_t);

__device__ __forceinline__ float hs(float c, float n, float s, float e, float w, float p) {
    return c + kCap * (p + (s + n - 2.0f * c) * kRy1 + (e + w - 2.0f * c) * kRx1 + (kAmb - c) * kRz1);
}

template <bool PUSH>
__global__ void __launch_bounds__(kThreads) k_hotspot2d_tma(const float* __restrict__ tin,
                                                            const float* __restrict__ pw,
                                                            float* __restrict__ tout, int64_t H, int64_t W,
                                                            int64_t TY, pk_partition part, PushList push) {
    extern __shared__ __align__(128) unsigned char smem[];
    float* ring = reinterpret_cast<float*>(smem);
    uint64_t* full = reinterpret_cast<uint64_t*>(smem + (size_t)kNS * kStageBytes);
    uint64_t* empty = full + kNS;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int s = 0; s < kNS; ++s) {
            ptx::mbar_init(&full[s], 1);
            ptx::mbar_init(&empty[s], kConsumers / 32);
        }
        ptx::fence_mbar_init();
    }
    __syncthreads();
    const int64_t gx = part.max[0] - part.min[0], gy = part.max[1] - part.min[1];
    const int64_t ntiles = gx * gy;

    if (warp == kConsumers / 32) {  // ---------------- producer
        if (lane != 0) return;
        uint32_t g = 0;
        for (int64_t T = blockIdx.x; T < ntiles; T += gridDim.x) {
            const int64_t bx = part.min[0] + T % gx, by = part.min[1] + T / gx;  // Eq. 8
            const int64_t c0 = bx * kTC, r0 = by * TY, rend = min(r0 + TY, H), nr = rend - r0;
            const bool down = (by & 1) == 0;
            const int64_t tlo = max(c0 - kHalo, (int64_t)0), thi = min(c0 + kTC + kHalo, W);
            const uint32_t tbytes = (uint32_t)(thi - tlo) * 4u;
            const int64_t toff = tlo - (c0 - kHalo);
            const uint32_t pbytes = (uint32_t)(min(c0 + kTC, W) - c0) * 4u;
            for (int64_t t = 0; t < nr + 2; ++t, ++g) {
                const uint32_t s = g % kNS, par = (g / kNS) & 1u;
                ptx::mbar_wait(&empty[s], par ^ 1u);
                int64_t row = down ? r0 - 1 + t : rend - t;
                row = row < 0 ? 0 : (row >= H ? H - 1 : row);
                const bool need_p = t >= 1 && t <= nr;
                float* st = ring + (size_t)s * kStageFloats;
                ptx::mbar_arrive_expect_tx(&full[s], tbytes + (need_p ? pbytes : 0u));
                ptx::bulk_g2s(st + toff, tin + row * W + tlo, tbytes, &full[s]);
                PK_TRACE_R(tin + row * W + tlo, tbytes);
                if (need_p) {
                    ptx::bulk_g2s(st + kTRow, pw + row * W + c0, pbytes, &full[s]);
                    PK_TRACE_R(pw + row * W + c0, pbytes);
                }
            }
        }
        return;
    }

    // ---------------- consumers: thread owns columns c0 + 4*tc .. +3
    const int tc = threadIdx.x;
    uint32_t g = 0;
    for (int64_t T = blockIdx.x; T < ntiles; T += gridDim.x) {
        const int64_t bx = part.min[0] + T % gx, by = part.min[1] + T / gx;
        const int64_t c0 = bx * kTC, r0 = by * TY, rend = min(r0 + TY, H), nr = rend - r0;
        const bool down = (by & 1) == 0;
        const int64_t j0 = c0 + 4 * tc;
        const bool active = j0 < W;
        const bool west_edge = j0 == 0, east_edge = j0 + 4 >= W;
        int64_t pa = 0, pb = 0;  // rows of this tile a push range may cover
        if (PUSH) dev::push_rows(push, r0, rend, (uint64_t)W * 4u, &pa, &pb);
        ptx::mbar_wait(&full[g % kNS], (g / kNS) & 1u);
        ptx::mbar_wait(&full[(g + 1) % kNS], ((g + 1) / kNS) & 1u);
        for (int64_t t = 1; t <= nr; ++t) {
            const uint32_t gp = g + (uint32_t)t - 1, gc = gp + 1, gn = gp + 2;
            ptx::mbar_wait(&full[gn % kNS], (gn / kNS) & 1u);
            const float* sp = ring + (size_t)(gp % kNS) * kStageFloats;
            const float* sc = ring + (size_t)(gc % kNS) * kStageFloats;
            const float* sn = ring + (size_t)(gn % kNS) * kStageFloats;
            const float4 c = *reinterpret_cast<const float4*>(sc + kHalo + 4 * tc);
            const float4 a = *reinterpret_cast<const float4*>(sp + kHalo + 4 * tc);
            const float4 b = *reinterpret_cast<const float4*>(sn + kHalo + 4 * tc);
            const float4 p = *reinterpret_cast<const float4*>(sc + kTRow + 4 * tc);
            float wv = __shfl_up_sync(0xffffffffu, c.w, 1);
            float ev = __shfl_down_sync(0xffffffffu, c.x, 1);
            if (lane == 0) wv = sc[kHalo + 4 * tc - 1];
            if (lane == 31) ev = sc[kHalo + 4 * tc + 4];
            if (west_edge) wv = c.x;
            if (east_edge) ev = c.w;
            if (active) {
                float4 o;
                o.x = hs(c.x, a.x, b.x, c.y, wv, p.x);
                o.y = hs(c.y, a.y, b.y, c.z, c.x, p.y);
                o.z = hs(c.z, a.z, b.z, c.w, c.y, p.z);
                o.w = hs(c.w, a.w, b.w, ev, c.z, p.w);
                const int64_t row = down ? r0 - 1 + t : rend - t;
                *reinterpret_cast<float4*>(tout + row * W + j0) = o;
                PK_TRACE_W(tout + row * W + j0, 16);
                if (PUSH && dev::in_rows(row, pa, pb))
                    dev::push4(push, (uint64_t)(row * W + j0) * 4u, o);  // fused halo push
            }
            __syncwarp();
            if (lane == 0) ptx::mbar_arrive(&empty[gp % kNS]);
        }
        __syncwarp();
        if (lane == 0) {
            ptx::mbar_arrive(&empty[(g + nr) % kNS]);
            ptx::mbar_arrive(&empty[(g + nr + 1) % kNS]);
        }
        g += (uint32_t)nr + 2;
    }
}

int describe_hotspot2d_tma(pk_ctx c, pk_kernel k) {
    // scalars: 0 = H, 1 = W, 2 = TY.  Logical block (bx, by) = rows [by*TY, +TY) x
    // columns [512 bx, 512 bx + 512), guarded to the grid; clamped 5-point reads.
    const int32_t off[5][2] = {{0, 0}, {-1, 0}, {1, 0}, {0, -1}, {0, 1}};
    const uint32_t f = PK_DIM_GUARD | PK_DIM_CLAMP;
    for (int t = 0; t < 5; ++t) {
        pk_affine_access a{};
        a.ndim = 2;
        a.dim[0] = DimMap(1, S(2), S(2), E(off[t][0]), f, E(0), S(0));
        a.dim[1] = DimMap(0, E(kTC), E(kTC), E(off[t][1]), f, E(0), S(1));
        if (int r = pk_declare_affine_access(c, k, 0, PK_READ, &a)) return r;
        if (t == 0) {
            if (int r = pk_declare_affine_access(c, k, 1, PK_READ, &a)) return r;
            if (int r = pk_declare_affine_access(c, k, 2, PK_WRITE, &a)) return r;
        }
    }
    return PK_OK;
}

template <bool PUSH>
cudaError_t launch_tma(const LaunchInfo& li, int64_t H, int64_t W, int64_t TY) {
    KernelDevInfo kd;
    cudaError_t e = prepare_kernel((const void*)k_hotspot2d_tma<PUSH>, li.device, kSmem, kThreads, &kd);
    if (e != cudaSuccess) return e;
    const int64_t ntiles = (int64_t)li.grid.x * li.grid.y;
    if (ntiles == 0) return cudaSuccess;
    dim3 grid(persistent_grid(ntiles, kd));
    PushList pl{};
    if (li.push) pl = *li.push;
    void* argv[] = {(void*)&li.inst[0], (void*)&li.inst[1], (void*)&li.inst[2], &H, &W, &TY, (void*)&li.part, &pl};
    return cudaLaunchKernel((const void*)k_hotspot2d_tma<PUSH>, grid, dim3(kThreads), argv, kSmem, li.stream);
}

cudaError_t launch_hotspot2d_tma(const LaunchInfo& li) {
    if (li.nscalars < 3) return cudaErrorInvalidValue;
    int64_t H = li.scalars[0], W = li.scalars[1], TY = li.scalars[2];
    // logical block = 128 threads x 4 columns (the launcher adds the producer warp)
    if (W % 4 || W < 4 || TY < 1 || li.block.x != kConsumers || li.block.y != 1 || li.block.z != 1)
        return cudaErrorInvalidValue;
    if (li.push && li.push->n > 0) return launch_tma<true>(li, H, W, TY);
    return launch_tma<false>(li, H, W, TY);
}


}  // namespace

const Builtin kBuiltinHotspot2dTma = {
    "hotspot2d", (const void*)k_hotspot2d_tma<false>, 6,
    {PK_ARG_BUFFER, PK_ARG_BUFFER, PK_ARG_BUFFER, PK_ARG_SCALAR, PK_ARG_SCALAR, PK_ARG_SCALAR}, -1,
    describe_hotspot2d_tma, launch_hotspot2d_tma, /*push_arg=*/2};

}  // namespace pk
