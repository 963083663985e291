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
// mbarrier full/empty, alternating march direction); the consumers keep both
// sweeps in registers: a thread owns 4 columns for the whole tile and carries
// 3-row windows of the input and of sweep 1, so per input row q it loads one new
// input row (+ power), computes sweep-1 row q-1 and sweep-2 row q-2 and stores
// it.  W/E neighbours come from warp shuffles; the warp's edge lanes also compute
// sweep 1 on the column just outside the warp (redundantly, bit-identically), so
// the 4 consumer warps never synchronise with each other -- only with the ring.
// (v1 staged sweep 1 through a shared-memory row ring with a named barrier per
// row: 521 M issued instructions per launch at C2, issue-bound at 76 % of HBM.)
#include <cuda_runtime.h>

#include "../runtime/builtins.h"
#include "launch_util.h"
#include "trace.cuh"
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
constexpr int kConsumers = 128;
constexpr int kThreads = kConsumers + 32;
constexpr size_t kSmem = (size_t)kNS * kStageBytes + 2 * kNS * sizeof(uint64_t);

__device__ __forceinline__ float hs(float c, float n, float s, float e, float w, float p) {
    return c + kCap * (p + (s + n - 2.0f * c) * kRy1 + (e + w - 2.0f * c) * kRx1 + (kAmb - c) * kRz1);
}

__global__ void __launch_bounds__(kThreads) k_hotspot2d_tb2(const float* __restrict__ tin,
                                                            const float* __restrict__ pw,
                                                            float* __restrict__ tout, int64_t H, int64_t W,
                                                            int64_t TY, pk_partition part) {
    extern __shared__ __align__(128) unsigned char smem[];
    float* ring = reinterpret_cast<float*>(smem);
    uint64_t* full = reinterpret_cast<uint64_t*>(ring + (size_t)kNS * kStageFloats);
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
                PK_TRACE_R(tin + row * W + tlo, bytes);
                PK_TRACE_R(pw + row * W + tlo, bytes);
            }
        }
        return;
    }

    // ---------------- consumers: thread owns columns j0 = c0 + 4*tc .. j0+3 for every row.
    // Everything a thread needs vertically stays in registers (3-row windows of the
    // input and of sweep 1); horizontal neighbours come from warp shuffles.  Each warp
    // is independent: its two edge lanes also compute sweep 1 at the column just
    // outside the warp (lane 0: w0-1, lane 31: w0+128) -- the warp's own halo,
    // recomputed redundantly with identical inputs and operation order -- so no
    // barrier among consumers is needed and warps drift freely through the ring.
    const int tc = threadIdx.x;
    const bool left = lane == 0;          // edge lane: extra column w0-1 (left) or w0+128 (right)
    uint32_t g = 0;
    for (int64_t T = blockIdx.x; T < ntiles; T += gridDim.x) {
        const int64_t bx = part.min[0] + T % gx, by = part.min[1] + T / gx;
        const int64_t c0 = bx * kTC, r0 = by * TY, rend = min(r0 + TY, H), nr = rend - r0;
        const bool down = (by & 1) == 0;
        const int dir = down ? 1 : -1;
        const int64_t j0 = c0 + 4 * tc;
        const bool active = j0 < W;
        const int cx = kHalo + 4 * tc;  // smem column of j0
        const bool wclamp = j0 == 0;            // west neighbour of j0 is j0 itself (grid border)
        const bool eclamp = j0 + 4 >= W;        // east neighbour of j0+3 is j0+3 itself
        // extra column of the edge lanes (other lanes evaluate a harmless copy of their own)
        const int64_t xe = left ? j0 - 1 : j0 + 4;
        const bool xneed = (lane == 0 || lane == 31) && xe >= 0 && xe < W;
        const int xc = xneed ? (left ? cx - 1 : cx + 4) : cx;          // smem column of xe
        const int xf = xneed ? (left ? cx - 2 : (xe + 1 < W ? cx + 5 : cx + 4)) : cx;  // far neighbour
        // W/E neighbours the edge lanes take from the extra column instead of a shuffle
        const bool use_xw = lane == 0 && xneed, use_xe = lane == 31 && xneed;
        const float* st = ring + (size_t)(g & (kNS - 1)) * kStageFloats;
        ptx::mbar_wait(&full[g & (kNS - 1)], (g / kNS) & 1u);
        const float4 in0 = *reinterpret_cast<const float4*>(st + cx);
        const float x0 = st[xc];
        st = ring + (size_t)((g + 1) & (kNS - 1)) * kStageFloats;
        ptx::mbar_wait(&full[(g + 1) & (kNS - 1)], ((g + 1) / kNS) & 1u);
        float4 inA = in0, inB = *reinterpret_cast<const float4*>(st + cx);  // input rows seq t-2, t-1
        float xA = x0, xB = st[xc];
        float4 s1A = make_float4(0.f, 0.f, 0.f, 0.f), s1B = s1A;         // sweep-1 rows seq t-3, t-2
        float eB = 0.f;                                                  // extra column, sweep 1, seq t-2
        float4 pA = s1A;                                                  // power, seq t-2
        const int nt = (int)nr + 4;
        int row1 = (int)((down ? r0 - 2 : rend + 1) + dir);  // grid row of sweep-1 seq t-1 (t = 2)
        const int Hi = (int)H;
        float* outp = tout + ((down ? r0 - 2 : rend + 1) + 2 * dir) * W + j0;  // sweep-2 row, t = 4
        const int64_t dW = dir * W;
        for (int t = 2; t < nt; ++t, row1 += dir) {
            const uint32_t gq = g + (uint32_t)t;
            ptx::mbar_wait(&full[gq & (kNS - 1)], (gq / kNS) & 1u);
            const float* sc = ring + (size_t)(gq & (kNS - 1)) * kStageFloats;        // seq t
            const float* sb = ring + (size_t)((gq - 1) & (kNS - 1)) * kStageFloats;  // seq t-1
            const float4 inC = *reinterpret_cast<const float4*>(sc + cx);
            const float4 pB = *reinterpret_cast<const float4*>(sb + kRowF + cx);     // power, seq t-1
            const float xC = sc[xc], xfar = sb[xf], xp = sb[kRowF + xc];
            // ---- sweep 1 at seq t-1 (own 4 columns + the edge lane's extra column)
            float wv = __shfl_up_sync(0xffffffffu, inB.w, 1);
            float ev = __shfl_down_sync(0xffffffffu, inB.x, 1);
            if (use_xw) wv = xB;
            if (use_xe) ev = xB;
            if (wclamp) wv = inB.x;
            if (eclamp) ev = inB.w;
            float4 s1C;
            s1C.x = hs(inB.x, inA.x, inC.x, inB.y, wv, pB.x);
            s1C.y = hs(inB.y, inA.y, inC.y, inB.z, inB.x, pB.y);
            s1C.z = hs(inB.z, inA.z, inC.z, inB.w, inB.y, pB.z);
            s1C.w = hs(inB.w, inA.w, inC.w, ev, inB.z, pB.w);
            // extra column xe: its near neighbour is the lane's own j0 (left) / j0+3 (right)
            const float eC = left ? hs(xB, xA, xC, inB.x, xfar, xp) : hs(xB, xA, xC, xfar, inB.w, xp);
            // ---- sweep 2 at seq t-2 (rows r0 .. rend-1), from the sweep-1 window
            if (t >= 4) {
                const int row2 = row1 - dir;
                const bool nin = (unsigned)(row2 - dir) < (unsigned)Hi, sin_ = (unsigned)row1 < (unsigned)Hi;
                const float4 n4 = nin ? s1A : s1B, s4 = sin_ ? s1C : s1B;
                float w2 = __shfl_up_sync(0xffffffffu, s1B.w, 1);
                float e2 = __shfl_down_sync(0xffffffffu, s1B.x, 1);
                if (use_xw) w2 = eB;
                if (use_xe) e2 = eB;
                if (wclamp) w2 = s1B.x;
                if (eclamp) e2 = s1B.w;
                float4 o;
                o.x = hs(s1B.x, n4.x, s4.x, s1B.y, w2, pA.x);
                o.y = hs(s1B.y, n4.y, s4.y, s1B.z, s1B.x, pA.y);
                o.z = hs(s1B.z, n4.z, s4.z, s1B.w, s1B.y, pA.z);
                o.w = hs(s1B.w, n4.w, s4.w, e2, s1B.z, pA.w);
                if (active) {
                    *reinterpret_cast<float4*>(outp) = o;
                    PK_TRACE_W(outp, 16);
                }
                outp += dW;
            }
            // ---- rotate the register windows; stage seq t-2 is no longer read by this warp
            inA = inB; inB = inC; xA = xB; xB = xC;
            s1A = s1B; s1B = s1C; eB = eC; pA = pB;
            __syncwarp();
            if (lane == 0) ptx::mbar_arrive(&empty[(gq - 2) & (kNS - 1)]);
        }
        __syncwarp();
        if (lane == 0) {
            ptx::mbar_arrive(&empty[(g + nr + 2) & (kNS - 1)]);
            ptx::mbar_arrive(&empty[(g + nr + 3) & (kNS - 1)]);
        }
        g += (uint32_t)nr + 4;
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
    KernelDevInfo kd;
    cudaError_t e = prepare_kernel((const void*)k_hotspot2d_tb2, li.device, kSmem, kThreads, &kd);
    if (e != cudaSuccess) return e;
    const int64_t ntiles = (int64_t)li.grid.x * li.grid.y;
    if (ntiles == 0) return cudaSuccess;
    dim3 grid(persistent_grid(ntiles, kd));
    void* argv[] = {(void*)&li.inst[0], (void*)&li.inst[1], (void*)&li.inst[2], &H, &W, &TY, (void*)&li.part};
    return cudaLaunchKernel((const void*)k_hotspot2d_tb2, grid, dim3(kThreads), argv, kSmem, li.stream);
}

}  // namespace

const Builtin kBuiltinHotspot2dTb2 = {
    "hotspot2d_tb2", (const void*)k_hotspot2d_tb2, 6,
    {PK_ARG_BUFFER, PK_ARG_BUFFER, PK_ARG_BUFFER, PK_ARG_SCALAR, PK_ARG_SCALAR, PK_ARG_SCALAR}, -1,
    describe_hotspot2d_tb2, launch_hotspot2d_tb2};

}  // namespace pk
