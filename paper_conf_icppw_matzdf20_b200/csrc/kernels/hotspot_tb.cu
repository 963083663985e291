// hotspot_tb.cu -- C2 Hotspot, temporally blocked: TWO time steps per launch
// (the Rodinia benchmark the paper runs is itself
// pyramid-blocked).
//
// Semantics: one launch = two consecutive Hotspot sweeps (reading Q14), i.e.
// temp_out = F(F(temp_in)); every output cell depends on the 5x5 clamped square
// of temp_in and the 3x3 clamped square of power around it, so a partition's read
// set is its rows/columns plus a halo of 2 (1 for power), its write set its own
// cells.  Halo cells of the intermediate sweep are recomputed redundantly by the
// two tiles that need them (identical inputs, identical operation order), so a
// P-way launch is bit-identical to the 1-way launch and HBM traffic
// per lattice update halves (6 B/LU instead of 12 B/LU).
//
// Design = hotspot_tma.cu's TMA bulk ring (persistent CTAs, producer thread,
// mbarrier full/empty, alternating march direction) plus a 4-row shared-memory
// ring for the intermediate sweep: at input row q the 4 consumer warps compute
// sweep-1 row q-1 (columns c0-1 .. c0+512, edge lanes add the two halo columns),
// sync on a named barrier, then compute sweep-2 row q-2 and store it.
#include <cuda_runtime.h>

#include "../runtime/builtins.h"
#include "ptx.cuh"

namespace pk {
namespace {

constexpr float kCap = 4096.0f / 3000.0f;
constexpr float kRx1 = 0.1f, kRy1 = 0.1f;
constexpr float kRz1 = 1.0f / 20480.0f;
constexpr float kAmb = 80.0f;

constexpr int kTC = 512;                  // columns per tile (128 threads x 4)
constexpr int kHalo = 4;                  // halo floats each side (16-B alignment; 2 are used)
constexpr int kRowF = kTC + 2 * kHalo;    // 520 floats per row segment
constexpr int kStageFloats = 2 * kRowF;   // temp row + power row
constexpr int kStageBytes = kStageFloats * 4;
constexpr int kNS = 8;                    // input ring depth
constexpr int kS1 = 4;                    // sweep-1 row ring
constexpr int kConsumers = 128;
constexpr int kThreads = kConsumers + 32;
constexpr size_t kSmem = (size_t)kNS * kStageBytes + (size_t)kS1 * kRowF * 4 + 2 * kNS * sizeof(uint64_t);

__device__ __forceinline__ float hs(float c, float n, float s, float e, float w, float p) {
    return c + kCap * (p + (s + n - 2.0f * c) * kRy1 + (e + w - 2.0f * c) * kRx1 + (kAmb - c) * kRz1);
}

__device__ __forceinline__ void consumer_bar() { asm volatile("bar.sync 1, 128;" ::: "memory"); }

__global__ void __launch_bounds__(kThreads) k_hotspot2d_tb2(const float* __restrict__ tin,
                                                            const float* __restrict__ pw,
                                                            float* __restrict__ tout, int64_t H, int64_t W,
                                                            int64_t TY, pk_partition part) {
    extern __shared__ __align__(128) unsigned char smem[];
    float* ring = reinterpret_cast<float*>(smem);
    float* s1 = ring + (size_t)kNS * kStageFloats;  // [kS1][kRowF]
    uint64_t* full = reinterpret_cast<uint64_t*>(s1 + (size_t)kS1 * kRowF);
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

    if (warp == kConsumers / 32) {  // ---------------- producer: input rows r0-2 .. r1+1
        if (lane != 0) return;
        uint32_t g = 0;
        for (int64_t T = blockIdx.x; T < ntiles; T += gridDim.x) {
            const int64_t bx = part.min[0] + T % gx, by = part.min[1] + T / gx;  // Eq. 8
            const int64_t c0 = bx * kTC, r0 = by * TY, rend = min(r0 + TY, H), nr = rend - r0;
            const bool down = (by & 1) == 0;
            const int64_t tlo = max(c0 - kHalo, (int64_t)0), thi = min(c0 + kTC + kHalo, W);
            const uint32_t bytes = (uint32_t)(thi - tlo) * 4u;
            const int64_t toff = tlo - (c0 - kHalo);
            for (int64_t t = 0; t < nr + 4; ++t, ++g) {
                const uint32_t s = g % kNS, par = (g / kNS) & 1u;
                ptx::mbar_wait(&empty[s], par ^ 1u);
                int64_t row = down ? r0 - 2 + t : rend + 1 - t;
                row = row < 0 ? 0 : (row >= H ? H - 1 : row);
                float* st = ring + (size_t)s * kStageFloats;
                ptx::mbar_arrive_expect_tx(&full[s], 2u * bytes);
                ptx::bulk_g2s(st + toff, tin + row * W + tlo, bytes, &full[s]);
                ptx::bulk_g2s(st + kRowF + toff, pw + row * W + tlo, bytes, &full[s]);
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
        const int64_t dir = down ? 1 : -1;
        const int64_t rstart = down ? r0 - 2 : rend + 1;  // input row of sequence index 0
        const int64_t j0 = c0 + 4 * tc;
        const bool active = j0 < W;
        const int cx = kHalo + 4 * tc;  // smem column of j0
        // clamped smem columns of the west/east neighbours of j0 and j0+3
        const int cw = j0 == 0 ? cx : cx - 1;
        const int ce = j0 + 4 >= W ? cx + 3 : cx + 4;
        ptx::mbar_wait(&full[g % kNS], (g / kNS) & 1u);
        ptx::mbar_wait(&full[(g + 1) % kNS], ((g + 1) / kNS) & 1u);
        static_assert((kNS & (kNS - 1)) == 0 && (kS1 & (kS1 - 1)) == 0, "rings are powers of two");
        const int nt = (int)nr + 4;
        int row1 = (int)(rstart + dir);              // sweep-1 row of iteration t = 2
        float* outp = tout + (rstart + 2 * dir) * W + j0;  // sweep-2 row of iteration t = 4
        const int64_t dW = dir * W;
        for (int t = 2; t < nt; ++t, row1 += (int)dir) {
            // input rows (sequence) t-2, t-1, t are in the ring; compute sweep-1 of
            // the row at sequence t-1 (rows r0-1 .. rend in march order), then sweep-2
            // of the row at sequence t-2 (rows r0 .. rend-1).
            const uint32_t gq = g + (uint32_t)t;
            ptx::mbar_wait(&full[gq & (kNS - 1)], (gq / kNS) & 1u);
            const float* sa = ring + ((gq - 2) & (kNS - 1)) * kStageFloats;  // seq t-2
            const float* sb = ring + ((gq - 1) & (kNS - 1)) * kStageFloats;  // seq t-1
            const float* sc = ring + (gq & (kNS - 1)) * kStageFloats;        // seq t
            const bool need1 = row1 >= 0 && row1 < H;      // rows outside the grid are never read
            float* s1row = s1 + ((t - 1) & (kS1 - 1)) * kRowF;
            if (need1) {
                // sweep 1 on columns j0..j0+3 (N/S = rows t-2 / t, order-independent)
                const float4 c = *reinterpret_cast<const float4*>(sb + cx);
                const float4 a = *reinterpret_cast<const float4*>(sa + cx);
                const float4 b = *reinterpret_cast<const float4*>(sc + cx);
                const float4 p = *reinterpret_cast<const float4*>(sb + kRowF + cx);
                float wv = __shfl_up_sync(0xffffffffu, c.w, 1);
                float ev = __shfl_down_sync(0xffffffffu, c.x, 1);
                if (lane == 0) wv = sb[cw];
                if (lane == 31 || j0 + 4 >= W) ev = sb[ce];
                if (j0 == 0) wv = c.x;
                float4 o;
                o.x = hs(c.x, a.x, b.x, c.y, wv, p.x);
                o.y = hs(c.y, a.y, b.y, c.z, c.x, p.y);
                o.z = hs(c.z, a.z, b.z, c.w, c.y, p.z);
                o.w = hs(c.w, a.w, b.w, ev, c.z, p.w);
                *reinterpret_cast<float4*>(s1row + cx) = o;
                // the two sweep-1 halo columns c0-1 and c0+512 (if inside the grid)
                if (tc == 0 && c0 > 0) {
                    const int k = kHalo - 1;  // column c0-1: neighbours c0-2 (clamped) and c0
                    const int kw = c0 - 2 >= 0 ? k - 1 : k;
                    s1row[k] = hs(sb[k], sa[k], sc[k], sb[k + 1], sb[kw], sb[kRowF + k]);
                }
                if (tc == kConsumers - 1 && c0 + kTC < W) {
                    const int k = kHalo + kTC;  // column c0+512
                    const int ke = c0 + kTC + 1 < W ? k + 1 : k;
                    s1row[k] = hs(sb[k], sa[k], sc[k], sb[ke], sb[k - 1], sb[kRowF + k]);
                }
            }
            consumer_bar();
            const bool need2 = t >= 4;  // sweep-2 rows: sequence 2 .. nr+1
            if (need2) {  // uniform: every lane joins the shuffles
                // sweep-1 rows t-3, t-2, t-1 (clamped to the grid: the row outside the grid
                // mirrors row2 = row1 - dir itself)
                const int row2 = row1 - (int)dir;
                const float* m0 = s1 + ((t - 2) & (kS1 - 1)) * kRowF;
                const int rn = row2 - (int)dir, rs = row1;
                const float* mn = (rn < 0 || rn >= H) ? m0 : s1 + ((t - 3) & (kS1 - 1)) * kRowF;
                const float* ms = (rs < 0 || rs >= H) ? m0 : s1 + ((t - 1) & (kS1 - 1)) * kRowF;
                const float4 c = *reinterpret_cast<const float4*>(m0 + cx);
                const float4 a = *reinterpret_cast<const float4*>(mn + cx);
                const float4 b = *reinterpret_cast<const float4*>(ms + cx);
                const float4 p = *reinterpret_cast<const float4*>(sa + kRowF + cx);  // power of row2 (seq t-2)
                float wv = __shfl_up_sync(0xffffffffu, c.w, 1);
                float ev = __shfl_down_sync(0xffffffffu, c.x, 1);
                if (lane == 0) wv = m0[cw];
                if (lane == 31 || j0 + 4 >= W) ev = m0[ce];
                if (j0 == 0) wv = c.x;
                float4 o;
                o.x = hs(c.x, a.x, b.x, c.y, wv, p.x);
                o.y = hs(c.y, a.y, b.y, c.z, c.x, p.y);
                o.z = hs(c.z, a.z, b.z, c.w, c.y, p.z);
                o.w = hs(c.w, a.w, b.w, ev, c.z, p.w);
                if (active) *reinterpret_cast<float4*>(outp) = o;
                outp += dW;
            }
            __syncwarp();
            if (lane == 0) ptx::mbar_arrive(&empty[(gq - 2) & (kNS - 1)]);  // seq t-2 fully used
        }
        __syncwarp();
        if (lane == 0) {
            ptx::mbar_arrive(&empty[(g + nr + 2) % kNS]);
            ptx::mbar_arrive(&empty[(g + nr + 3) % kNS]);
        }
        g += (uint32_t)nr + 4;
        consumer_bar();  // the sweep-1 ring is reused by the next tile
    }
}

int describe_hotspot2d_tb2(pk_ctx c, pk_kernel k) {
    // scalars: 0 = H, 1 = W, 2 = TY.  Logical block (bx, by) = rows [by*TY, +TY) x
    // columns [512 bx, +512), guarded.  Reads the clamped 5x5 square of temp and the
    // clamped 3x3 square of power around every cell (corners included: a read
    // over-approximation); writes its own cells.
    const uint32_t f = PK_DIM_GUARD | PK_DIM_CLAMP;
    for (int di = -2; di <= 2; ++di)
        for (int dj = -2; dj <= 2; ++dj) {
            pk_affine_access a{};
            a.ndim = 2;
            a.dim[0] = DimMap(1, S(2), S(2), E(di), f, E(0), S(0));
            a.dim[1] = DimMap(0, E(kTC), E(kTC), E(dj), f, E(0), S(1));
            if (int r = pk_declare_affine_access(c, k, 0, PK_READ, &a)) return r;
            if (di >= -1 && di <= 1 && dj >= -1 && dj <= 1)
                if (int r = pk_declare_affine_access(c, k, 1, PK_READ, &a)) return r;
            if (di == 0 && dj == 0)
                if (int r = pk_declare_affine_access(c, k, 2, PK_WRITE, &a)) return r;
        }
    return PK_OK;
}

cudaError_t launch_hotspot2d_tb2(const LaunchInfo& li) {
    if (li.nscalars < 3) return cudaErrorInvalidValue;
    int64_t H = li.scalars[0], W = li.scalars[1], TY = li.scalars[2];
    if (W % 4 || W < 4 || TY < 1 || li.block.x != kConsumers || li.block.y != 1 || li.block.z != 1)
        return cudaErrorInvalidValue;
    static int resident[64] = {0};
    static int sms[64] = {0};
    const int d = li.device;
    if (d < 0 || d >= 64) return cudaErrorInvalidDevice;
    if (!resident[d]) {
        cudaError_t e = cudaFuncSetAttribute(k_hotspot2d_tb2, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSmem);
        if (e != cudaSuccess) return e;
        int nb = 0;
        e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_hotspot2d_tb2, kThreads, kSmem);
        if (e != cudaSuccess) return e;
        e = cudaDeviceGetAttribute(&sms[d], cudaDevAttrMultiProcessorCount, d);
        if (e != cudaSuccess) return e;
        resident[d] = nb > 0 ? nb : 1;
    }
    const int64_t ntiles = (int64_t)li.grid.x * li.grid.y;
    if (ntiles == 0) return cudaSuccess;
    const int64_t cap = (int64_t)resident[d] * sms[d];
    dim3 grid((unsigned)(ntiles < cap ? ntiles : cap));
    void* argv[] = {(void*)&li.inst[0], (void*)&li.inst[1], (void*)&li.inst[2], &H, &W, &TY, (void*)&li.part};
    return cudaLaunchKernel((const void*)k_hotspot2d_tb2, grid, dim3(kThreads), argv, kSmem, li.stream);
}

}  // namespace

const Builtin kBuiltinHotspot2dTb2 = {
    "hotspot2d_tb2", (const void*)k_hotspot2d_tb2, 6,
    {PK_ARG_BUFFER, PK_ARG_BUFFER, PK_ARG_BUFFER, PK_ARG_SCALAR, PK_ARG_SCALAR, PK_ARG_SCALAR}, -1,
    describe_hotspot2d_tb2, launch_hotspot2d_tb2};

}  // namespace pk
