// hotspot_tbk.cu -- C2 Hotspot, temporally blocked to depth K (2..8): K time steps
// per launch ("halo width h per launch": the Rodinia
// benchmark the paper runs is itself pyramid-blocked).
//
// Semantics: one launch = K consecutive Hotspot sweeps (reading Q14, replicate-
// clamped borders applied at every sweep).  An output cell depends on the clamped
// (2K+1)^2 square of temp_in and the (2K-1)^2 square of power around it, so a
// partition's read set is its box dilated by K (K-1 for power) and its write set
// its own cells.  HBM traffic is 12 B per cell per launch = 12/K B per lattice
// update (K = 4: 3 B/LU, a quarter of the one-sweep kernel).
//
// Design (B200): persistent CTAs walking the partition's logical blocks (Eq. 8),
// one producer thread streaming row segments (temp + power, 488 floats each) with
// cp.async.bulk into an mbarrier ring, 4 consumer warps.  A consumer lane owns 4
// adjacent columns for the whole tile and keeps, per sweep level, a 3-row window
// in registers (slot = row sequence mod 3, so the 3-fold unrolled loop needs no
// register moves): per input row it loads one new temp row, computes level k at
// row sequence t-k for k = 1..K (power from the ring) and stores level K.  W/E neighbours are warp shuffles.
// Warps overlap: a warp covers 128 columns, but its HL = ceil(K/4) outermost lanes
// on each side are halo lanes (a lane holds 4 columns; the shuffle wrap corrupts
// one more column per sweep), so only lanes HL..31-HL store: 120 owned columns per
// warp and 480 per tile for K <= 4, 112 and 448 for K = 5..8.  Consumers
// therefore never synchronise with each other, only with the ring.  Halo rows and
// columns are recomputed redundantly from identical inputs in identical operation
// order, so P-way launches are bit-identical to 1-way.
//
// Arithmetic per cell and sweep (6 FP32 ops, fixed order):
//   T' = c*A + (((n + s) + e) + w)*B + (p*kCap + D)
// with A = 1 - kCap(2 Ry1 + 2 Rx1 + Rz1), B = kCap Ry1 (Rx1 == Ry1), D = kCap Rz1 amb:
// the Rodinia update of reading Q14 with its constant terms folded.  (Measured and
// rejected: the order s*B + ((n + e) + w)*B + ..., which leaves only the last FMA
// on the level chain -- equal speed at K = 4 within noise, more registers.)
//
// Depth: K = 2..8 are instantiated; K = 4 is the bench default.  K > 4 needs two
// halo lanes per side and ~170 registers (2 CTAs/SM): measured on C2 at 96
// sweeps, K = 4 / 6 / 8: 1977 / 1432 / 1270 GLUP/s -- beyond K = 4 the kernel is
// bound by the K-level dependency chain per row at 8 consumer warps per SM, not by
// HBM (0.44 / 0.29 of the measured HBM roof), so deeper blocking does not pay here.
#include <cuda_runtime.h>

#include "../runtime/builtins.h"
#include "launch_util.h"
#include "common.cuh"
#include "ptx.cuh"

namespace pk {
namespace {

constexpr double kCapD = 4096.0 / 3000.0;
constexpr double kR1D = 0.1;  // Rx1 == Ry1
constexpr double kRz1D = 1.0 / 20480.0;
constexpr double kAmbD = 80.0;
constexpr float kA = (float)(1.0 - kCapD * (4.0 * kR1D + kRz1D));
constexpr float kB = (float)(kCapD * kR1D);
constexpr float kCap = (float)kCapD;
constexpr float kD = (float)(kCapD * kRz1D * kAmbD);

// per-depth geometry: HL halo lanes per side, owned columns per warp / tile, row
// segment [c0 - 4 HL, c0 + TC + 4 HL) of temp (then power) per ring stage
template <int K>
struct Geo {
    static constexpr int HL = (K + 3) / 4;
    static constexpr int Own = (32 - 2 * HL) * 4;
    static constexpr int TC = 4 * Own;
    static constexpr int RowF = TC + 8 * HL;
    static constexpr int StageFloats = 2 * RowF;
    static constexpr int StageBytes = StageFloats * 4;
};
#ifndef PK_TBK_NS
#define PK_TBK_NS 16
#endif
constexpr int kNS = PK_TBK_NS;            // ring depth (power of two)
static_assert((kNS & (kNS - 1)) == 0 && kNS >= 16, "ring holds K+1 <= 9 rows plus prefetch");
constexpr int kConsumers = 128;
constexpr int kThreads = kConsumers + 32;
template <int K>
constexpr size_t smem_bytes() { return (size_t)kNS * Geo<K>::StageBytes + 2 * kNS * sizeof(uint64_t); }

__device__ __forceinline__ float upd(float c, float n, float s, float e, float w, float p) {
    return fmaf(c, kA, fmaf(((n + s) + e) + w, kB, fmaf(p, kCap, kD)));
}

// one level: row `c` with N/S rows, W/E from neighbouring lanes (clamped at the
// grid's first/last column when the tile touches them: COLEDGE)
template <bool COLEDGE>
__device__ __forceinline__ float4 level(const float4& c, const float4& n, const float4& s, const float4& p,
                                        bool wclamp, bool eclamp) {
    float wv = __shfl_up_sync(0xffffffffu, c.w, 1);
    float ev = __shfl_down_sync(0xffffffffu, c.x, 1);
    if (COLEDGE) {
        if (wclamp) wv = c.x;
        if (eclamp) ev = c.w;
    }
    float4 o;
    o.x = upd(c.x, n.x, s.x, c.y, wv, p.x);
    o.y = upd(c.y, n.y, s.y, c.z, c.x, p.y);
    o.z = upd(c.z, n.z, s.z, c.w, c.y, p.z);
    o.w = upd(c.w, n.w, s.w, ev, c.z, p.w);
    return o;
}

// Register windows are indexed by row sequence mod 3; the loop is unrolled 3-fold
// from t = 2, so every window slot is a compile-time register.  Power rows are read
// from the ring per level.  Measured alternatives (C2, K = 4): a K-row power window
// in registers (4-fold unroll) needs 168 registers -> 2 CTAs/SM, 1764 GLUP/s; a
// skewed level schedule (level k at row t-2k+1, independent levels) 1476 GLUP/s;
// this variant at 128 registers, 3 CTAs/SM and a 16-stage ring: 1940 GLUP/s.
template <int K, bool EDGE, bool COLEDGE>
__device__ __forceinline__ void consume_tile(const float* ring, uint64_t* full, uint64_t* empty, float* tout,
                                             int64_t W, int H, int64_t c0, int64_t r0, int64_t rend, bool down,
                                             uint32_t g, int lane, int warp) {
    using G = Geo<K>;
    constexpr int kW3 = 3;
    const int scol = G::Own * warp + 4 * lane;
    const int64_t col0 = c0 - 4 * G::HL + scol;
    const bool store = lane >= G::HL && lane <= 31 - G::HL && col0 < W;
    const bool wclamp = col0 == 0, eclamp = col0 + 4 >= W;
    const int nr = (int)(rend - r0), nt = nr + 2 * K;
    const int dir = down ? 1 : -1;
    const int base = (int)(down ? r0 - K : rend - 1 + K);
    float4 in[kW3];
    float4 L[K > 1 ? K - 1 : 1][kW3];
    auto stage = [&](int seq) { return ring + (size_t)((g + (uint32_t)seq) & (kNS - 1)) * G::StageFloats; };
    ptx::mbar_wait(&full[g & (kNS - 1)], (g / kNS) & 1u);
    in[0] = *reinterpret_cast<const float4*>(stage(0) + scol);
    ptx::mbar_wait(&full[(g + 1) & (kNS - 1)], ((g + 1) / kNS) & 1u);
    in[1] = *reinterpret_cast<const float4*>(stage(1) + scol);
    float* outp = tout + (int64_t)(base + dir * K) * W + col0;
    const int64_t dW = dir * W;
    for (int t0 = 2; t0 < nt; t0 += kW3) {
#pragma unroll
        for (int u = 0; u < kW3; ++u) {
            const int t = t0 + u;
            if (t >= nt) break;
            const uint32_t gq = g + (uint32_t)t;
            ptx::mbar_wait(&full[gq & (kNS - 1)], (gq / kNS) & 1u);
            in[(2 + u) % kW3] = *reinterpret_cast<const float4*>(stage(t) + scol);
#pragma unroll
            for (int k = 1; k <= K; ++k) {
                const int sc = (2 + u - k + kW3 * K) % kW3;
                const int sn = (2 + u - k - 1 + kW3 * K) % kW3;
                const int ss = (2 + u - k + 1 + kW3 * K) % kW3;
                const float4* prev = k == 1 ? in : L[k - 2 < 0 ? 0 : k - 2];
                const float4 p = *reinterpret_cast<const float4*>(stage(t - k) + G::RowF + scol);
                float4 n4 = prev[sn], s4 = prev[ss];
                if (EDGE && k > 1) {
                    const int R = base + dir * (t - k);
                    if ((unsigned)(R - dir) >= (unsigned)H) n4 = prev[sc];
                    if ((unsigned)(R + dir) >= (unsigned)H) s4 = prev[sc];
                }
                const float4 o = level<COLEDGE>(prev[sc], n4, s4, p, wclamp, eclamp);
                if (k < K) {
                    L[k - 1][sc] = o;
                } else if (t >= 2 * K) {
                    if (store) {
                        *reinterpret_cast<float4*>(outp) = o;
                        PK_TRACE_W(outp, 16);
                    }
                    outp += dW;
                }
            }
            __syncwarp();
            if (t >= K && lane == 0) ptx::mbar_arrive(&empty[(gq - K) & (kNS - 1)]);  // seq t-K done
        }
    }
    __syncwarp();
    if (lane == 0)
        for (int sq = nt - K; sq < nt; ++sq) ptx::mbar_arrive(&empty[(g + (uint32_t)sq) & (kNS - 1)]);
}
#ifndef PK_TBK_MINB
#define PK_TBK_MINB 3
#endif
#ifndef PK_TBK8_MINB
#define PK_TBK8_MINB 2
#endif
template <int K, bool PUSH>
__global__ void __launch_bounds__(kThreads, K <= 4 ? PK_TBK_MINB : PK_TBK8_MINB) k_hotspot2d_tbk(const float* __restrict__ tin,
                                                            const float* __restrict__ pw,
                                                            float* __restrict__ tout, int64_t H, int64_t W,
                                                            int64_t TY, pk_partition part, PushList push) {
    using G = Geo<K>;
    extern __shared__ __align__(128) unsigned char smem[];
    float* ring = reinterpret_cast<float*>(smem);
    uint64_t* full = reinterpret_cast<uint64_t*>(ring + (size_t)kNS * G::StageFloats);
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

    if (warp == kConsumers / 32) {  // ---------------- producer: input rows r0-K .. rend+K-1
        if (lane != 0) return;
        uint32_t g = 0;
        for (int64_t T = blockIdx.x; T < ntiles; T += gridDim.x) {
            const int64_t bx = part.min[0] + T % gx, by = part.min[1] + T / gx;  // Eq. 8
            const int64_t c0 = bx * G::TC, r0 = by * TY, rend = min(r0 + TY, H), nr = rend - r0;
            const bool down = (by & 1) == 0;
            const int64_t tlo = max(c0 - 4 * G::HL, (int64_t)0), thi = min(c0 + G::TC + 4 * G::HL, W);
            const uint32_t bytes = (uint32_t)(thi - tlo) * 4u;
            const int64_t toff = tlo - (c0 - 4 * G::HL);
            for (int64_t t = 0; t < nr + 2 * K; ++t, ++g) {
                const uint32_t s = g % kNS, par = (g / kNS) & 1u;
                ptx::mbar_wait(&empty[s], par ^ 1u);
                int64_t row = down ? r0 - K + t : rend - 1 + K - t;
                row = row < 0 ? 0 : (row >= H ? H - 1 : row);
                float* st = ring + (size_t)s * G::StageFloats;
                ptx::mbar_arrive_expect_tx(&full[s], 2u * bytes);
                ptx::bulk_g2s(st + toff, tin + row * W + tlo, bytes, &full[s]);
                ptx::bulk_g2s(st + G::RowF + toff, pw + row * W + tlo, bytes, &full[s]);
                PK_TRACE_R(tin + row * W + tlo, bytes);
                PK_TRACE_R(pw + row * W + tlo, bytes);
            }
        }
        return;
    }

    uint32_t g = 0;
    for (int64_t T = blockIdx.x; T < ntiles; T += gridDim.x) {
        const int64_t bx = part.min[0] + T % gx, by = part.min[1] + T / gx;
        const int64_t c0 = bx * G::TC, r0 = by * TY, rend = min(r0 + TY, H);
        const bool down = (by & 1) == 0;
        // tiles whose (dilated) rows reach the grid's first/last row need the clamp selects
        const bool redge = r0 < K + 1 || rend + K + 1 > H;
        const bool cedge = c0 == 0 || c0 + G::TC + 4 * G::HL >= W;
        if (redge || cedge)
            consume_tile<K, true, true>(ring, full, empty, tout, W, (int)H, c0, r0, rend, down, g, lane, warp);
        else
            consume_tile<K, false, false>(ring, full, empty, tout, W, (int)H, c0, r0, rend, down, g, lane, warp);
        if (PUSH) {
            // fused halo push: the tile's rows a push range may cover (usually the K rows at a
            // partition edge, else none) are re-read from this thread's own stores and forwarded.
            // A store branch inside the level loop cost ~19 % per launch even when never taken.
            int64_t pa = 0, pb = 0;
            dev::push_rows(push, r0, rend, (uint64_t)W * 4u, &pa, &pb);
            const int64_t col0 = c0 - 4 * G::HL + G::Own * warp + 4 * lane;
            if (pb > pa && lane >= G::HL && lane <= 31 - G::HL && col0 < W)
                for (int64_t R = pa; R < pb; ++R) {
                    const float* rp = tout + R * W + col0;
                    dev::push4(push, (uint64_t)(rp - tout) * 4u, *reinterpret_cast<const float4*>(rp));
                }
        }
        g += (uint32_t)(rend - r0) + 2 * K;
    }
}

int describe_hotspot2d_tbk(pk_ctx c, pk_kernel k) {
    // scalars: 0 = H, 1 = W, 2 = TY, 3 = K, 4 = TC (owned columns per logical block:
    // 480 for K <= 4, 448 for K = 5..8, checked by the launcher).  Logical block
    // (bx, by) = rows [by*TY, +TY) x columns [TC bx, +TC), guarded.  Reads the clamped (2K+1)^2 square of temp
    // (the dilated box: one tap, exact union of the shifted boxes; corners included,
    // a read over-approximation) and the (2K-1)^2 square of power; writes
    // its own cells.  Positions are taken in [b*scale, b*scale + extent + 2K) with the
    // guard shifted by the same 2K, then offset by -K and clamped.
    const uint32_t f = PK_DIM_GUARD | PK_DIM_CLAMP;
    pk_affine_access a{};
    a.ndim = 2;
    // temp: rows [by*TY - K, by*TY + TY + K) ∩ guard, cols likewise, clamped
    a.dim[0] = DimMap(1, S(2), S(2, 1), S(3, -1), f, E(0), S(0));
    a.dim[0].extent.c_scalar[3] = 2;   // TY + 2K
    a.dim[0].guard_hi.c_scalar[3] = 2; // H + 2K
    a.dim[1] = DimMap(0, S(4), S(4), S(3, -1), f, E(0), S(1));
    a.dim[1].extent.c_scalar[3] = 2;
    a.dim[1].guard_hi.c_scalar[3] = 2;
    if (int r = pk_declare_affine_access(c, k, 0, PK_READ, &a)) return r;
    // power: dilated by K-1
    pk_affine_access b = a;
    for (int d = 0; d < 2; ++d) {
        b.dim[d].extent.c0 -= 2;          // + 2K - 2
        b.dim[d].guard_hi.c0 -= 2;
        b.dim[d].offset.c0 += 1;          // -(K-1)
    }
    if (int r = pk_declare_affine_access(c, k, 1, PK_READ, &b)) return r;
    pk_affine_access w{};
    w.ndim = 2;
    w.dim[0] = DimMap(1, S(2), S(2), E(0), f, E(0), S(0));
    w.dim[1] = DimMap(0, S(4), S(4), E(0), f, E(0), S(1));
    return pk_declare_affine_access(c, k, 2, PK_WRITE, &w);
}

template <int K, bool PUSH>
cudaError_t launch_k(const LaunchInfo& li, int64_t H, int64_t W, int64_t TY) {
    constexpr size_t kSmem = smem_bytes<K>();
    KernelDevInfo kd;
    cudaError_t e = prepare_kernel((const void*)k_hotspot2d_tbk<K, PUSH>, li.device, kSmem, kThreads, &kd);
    if (e != cudaSuccess) return e;
    const int64_t ntiles = (int64_t)li.grid.x * li.grid.y;
    if (ntiles == 0) return cudaSuccess;
    dim3 grid(persistent_grid(ntiles, kd));
    PushList pl{};
    if (li.push) pl = *li.push;
    void* argv[] = {(void*)&li.inst[0], (void*)&li.inst[1], (void*)&li.inst[2], &H, &W, &TY, (void*)&li.part, &pl};
    return cudaLaunchKernel((const void*)k_hotspot2d_tbk<K, PUSH>, grid, dim3(kThreads), argv, kSmem, li.stream);
}

cudaError_t launch_hotspot2d_tbk(const LaunchInfo& li) {
    if (li.nscalars < 5) return cudaErrorInvalidValue;
    const int64_t H = li.scalars[0], W = li.scalars[1], TY = li.scalars[2], K = li.scalars[3], TC = li.scalars[4];
    if (W % 4 || W < 4 || TY < 1 || H < 1 || H > (1ll << 30) || li.block.x != kConsumers || li.block.y != 1 ||
        li.block.z != 1 || TC != (K <= 4 ? Geo<4>::TC : Geo<8>::TC))
        return cudaErrorInvalidValue;
    const bool push = li.push && li.push->n > 0;
    switch (K) {
        case 2: return push ? launch_k<2, true>(li, H, W, TY) : launch_k<2, false>(li, H, W, TY);
        case 3: return push ? launch_k<3, true>(li, H, W, TY) : launch_k<3, false>(li, H, W, TY);
        case 4: return push ? launch_k<4, true>(li, H, W, TY) : launch_k<4, false>(li, H, W, TY);
        case 5: return push ? launch_k<5, true>(li, H, W, TY) : launch_k<5, false>(li, H, W, TY);
        case 6: return push ? launch_k<6, true>(li, H, W, TY) : launch_k<6, false>(li, H, W, TY);
        case 7: return push ? launch_k<7, true>(li, H, W, TY) : launch_k<7, false>(li, H, W, TY);
        case 8: return push ? launch_k<8, true>(li, H, W, TY) : launch_k<8, false>(li, H, W, TY);
        default: return cudaErrorInvalidValue;
    }
}

}  // namespace

const Builtin kBuiltinHotspot2dTbk = {
    "hotspot2d_tbk", (const void*)k_hotspot2d_tbk<4, false>, 6,
    {PK_ARG_BUFFER, PK_ARG_BUFFER, PK_ARG_BUFFER, PK_ARG_SCALAR, PK_ARG_SCALAR, PK_ARG_SCALAR}, -1,
    describe_hotspot2d_tbk, launch_hotspot2d_tbk, /*push_arg=*/2};

}  // namespace pk
