// heat_tb.cu -- C3 3-D 7-point heat stencil, temporally blocked: TWO time steps
// per launch (the 3-D counterpart of hotspot2d_tbk).
//
// Semantics: one launch = two consecutive sweeps of reading Q15
//   u' = u + alpha((zm + zp + ym + yp + xm + xp) - 6u),  alpha = 1/8,
// replicate-clamped at every sweep.  An output cell depends on the clamped
// 5x5x5 cube of u_in around it, so a partition's read set is its box dilated by 2
// and its write set its own cells: 8 B per cell per launch = 4 B per lattice
// update (half the one-sweep kernel's 8 B/LU).
//
// Design (B200): logical block = 120 columns x 16 rows x ZC planes.  A producer
// warp streams one 3-D tensor-TMA box per plane -- 128 columns [c0-4, c0+124) x
// 20 rows [y0-2, y0+18) x 1 plane, out-of-grid columns/rows zero-filled, the plane
// index clamped -- into a 6-slot mbarrier ring, 3 CTAs/SM.  4 consumer warps march z; warp w
// owns rows y0+4w .. +3, a lane owns 4 columns.  Per input plane q a warp computes
// sweep 1 of plane q-1 on its 4 rows (warp 0 also the block's halo row above, warp 3
// the one below; inputs from shared memory) into a register window of 3 planes x 4
// rows, hands its top and bottom sweep-1 rows to its neighbours through shared memory
// (one named barrier among the consumer warps per plane), and computes sweep 2 of
// plane q-2 on its own 4 rows, which it stores.  x neighbours are warp shuffles;
// lanes 0 and 31 are halo lanes whose outer column is wrong after each sweep (shuffle
// wrap), so lanes 1..30 store: 120 owned columns.  Halo rows, columns and planes of
// sweep 1 are recomputed by the blocks that need them from identical inputs in
// identical order, so P-way launches are bit-identical to 1-way.
#include <cuda.h>
#include <cuda_runtime.h>

#include <mutex>
#include <unordered_map>

#include "../runtime/builtins.h"
#include "launch_util.h"
#include "trace.cuh"
#include "common.cuh"
#include "ptx.cuh"
#include "tma_host.h"

namespace pk {
namespace {

constexpr float kAlpha = 0.125f;
constexpr int kCols = 128;                // columns per warp window (box width)
constexpr int kOwnC = 120;                // owned columns per block (lanes 1..30)
constexpr int kRW = 4;                    // owned rows per consumer warp
constexpr int kNW = 4;                    // consumer warps (3 CTAs/SM; measured 6 warps x 2 CTAs: -4 %)
constexpr int kRows = kRW * kNW;          // owned rows per block (16)
constexpr int kBoxRows = kRows + 4;       // rows y0-2 .. y0+kRows+1
#ifndef PK_HEATTB_NS
#define PK_HEATTB_NS 6
#endif
constexpr int kNS = PK_HEATTB_NS;         // plane ring depth (3 CTAs x 6 x 10 KB per SM; 7 slots: -2 %)
constexpr int kSlot = kBoxRows * kCols;   // floats per plane slot (14 KB)
// sweep-1 rows shared between warps: per plane, each warp's top and bottom own row plus the
// block's two halo rows (10 rows), double-buffered by plane parity
constexpr int kXRows = 2 * kNW + 2;
constexpr size_t kXBytes = (size_t)2 * kXRows * kCols * 4;
constexpr size_t kSmem = (size_t)kNS * kSlot * 4 + kXBytes + 2 * kNS * 8 + 128;
#ifndef PK_HEATTB_PNS
#define PK_HEATTB_PNS 256
#endif

__device__ __forceinline__ void tma_3d(void* dst, const CUtensorMap* map, int32_t x, int32_t y, int32_t z,
                                       uint64_t* bar) {
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], "
        "[%5];" ::"r"(ptx::smem_u32(dst)),
        "l"(map), "r"(x), "r"(y), "r"(z), "r"(ptx::smem_u32(bar))
        : "memory");
}

// u + alpha((zm + zp + ym + yp + w + e) - 6u), same operation order for every cell
__device__ __forceinline__ float upd(float c, float zm, float zp, float ym, float yp, float w, float e) {
    return c + kAlpha * ((zm + zp + ym + yp + w + e) - 6.0f * c);
}

__device__ __forceinline__ float4 sweep(const float4& c, const float4& zm, const float4& zp, const float4& ym,
                                        const float4& yp, bool wclamp, bool eclamp) {
#ifdef PK_HEATTB_DIAG   // diagnostic only (power / rate of the data stream without the arithmetic)
    return c;
#endif
    float wv = __shfl_up_sync(0xffffffffu, c.w, 1);
    float ev = __shfl_down_sync(0xffffffffu, c.x, 1);
    if (wclamp) wv = c.x;
    if (eclamp) ev = c.w;
    float4 o;
    o.x = upd(c.x, zm.x, zp.x, ym.x, yp.x, wv, c.y);
    o.y = upd(c.y, zm.y, zp.y, ym.y, yp.y, c.x, c.z);
    o.z = upd(c.z, zm.z, zp.z, ym.z, yp.z, c.y, c.w);
    o.w = upd(c.w, zm.w, zp.w, ym.w, yp.w, c.z, ev);
    return o;
}

template <bool PUSH, bool EDGE>
__device__ __forceinline__ void consume(const float* ring, float* xbuf, uint64_t* full, uint64_t* empty,
                                        float* __restrict__ uout, int64_t D, int64_t H, int64_t W, int64_t c0,
                                        int64_t y0, int64_t k0, int nq, int lane, int warp, const PushList& push);

// 3 CTAs/SM = 128 registers per thread.  __maxnreg__(136) (15 warps x 17 allocation units)
// removed most spills but measured slower (1238-1264 vs 1331-1349 GLUP/s, scripts/gpu_run100.sh)
#ifndef PK_HEATTB_MAXNREG
#define PK_HEATTB_MAXNREG 128
#endif
template <bool PUSH>
__global__ void __maxnreg__(PK_HEATTB_MAXNREG)
    k_heat3d_tb2(const __grid_constant__ CUtensorMap tm_u, float* __restrict__ uout, int64_t D, int64_t H, int64_t W,
                 int64_t ZC, pk_partition part, PushList push, const float* uin_trace) {
    extern __shared__ __align__(1024) unsigned char smem_raw[];
    // 128-B aligned ring; pointer arithmetic on the shared array (not a uintptr_t round
    // trip) keeps the shared address space visible, so the loads below are LDS, not LD
    float* ring = reinterpret_cast<float*>(smem_raw + ((128u - ((uint32_t)(uintptr_t)smem_raw & 127u)) & 127u));
    float* xbuf = ring + (size_t)kNS * kSlot;   // exchange rows (kXBytes)
    uint64_t* full = reinterpret_cast<uint64_t*>(reinterpret_cast<unsigned char*>(xbuf) + kXBytes);
    uint64_t* empty = full + kNS;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int64_t bx = part.min[0] + blockIdx.x, by = part.min[1] + blockIdx.y, bz = part.min[2] + blockIdx.z;
    const int64_t c0 = bx * kOwnC, y0 = by * kRows, k0 = bz * ZC;  // Eq. 8
    if (c0 >= W || y0 >= H || k0 >= D) return;                      // block-uniform
    const int64_t k1 = min(k0 + ZC, D);
    const int nz = (int)(k1 - k0);
    const int nq = nz + 4;                                           // planes k0-2 .. k1+1 (clamped)
    if (threadIdx.x == 0) {
        for (int s = 0; s < kNS; ++s) {
            ptx::mbar_init(&full[s], 1);
            ptx::mbar_init(&empty[s], kNW);
        }
        ptx::fence_mbar_init();
        asm volatile("prefetch.tensormap [%0];" ::"l"(&tm_u) : "memory");
    }
    __syncthreads();

    if (warp == kNW) {  // ---------------- producer: one TMA box per plane
        if (lane != 0) return;
        constexpr uint32_t bytes = (uint32_t)kSlot * 4u;
        for (int q = 0; q < nq; ++q) {
            const int s = q % kNS;
            // polls with a 256-ns back-off: 3 producers per SM spinning took issue slots from the
            // 12 consumer warps (1261-1267 spinning vs 1296-1311 GLUP/s); Hotspot's ring of 4-KB
            // rows needs prompt refills instead (back-off there: 1810 vs 1900)
            ptx::mbar_wait_backoff(&empty[s], ((q / kNS) & 1u) ^ 1u, PK_HEATTB_PNS);
            int64_t p = k0 - 2 + q;
            p = p < 0 ? 0 : (p >= D ? D - 1 : p);
            ptx::mbar_arrive_expect_tx(&full[s], bytes);
            tma_3d(ring + (size_t)s * kSlot, &tm_u, (int32_t)(c0 - 4), (int32_t)(y0 - 2), (int32_t)p, &full[s]);
            PK_TRACE_BOX(uin_trace, H, W, c0 - 4, kCols, y0 - 2, kBoxRows, p);
        }
        return;
    }

    // ---------------- consumers: blocks touching the grid's first/last row or plane apply
    // the replicate clamp of the intermediate sweep; interior blocks skip the selects
#ifdef PK_HEATTB_ALLEDGE   // diagnostic: every block through the clamping consumer
    const bool edge = true;
#else
    const bool edge = y0 < 2 || y0 + kRows + 2 > H || k0 < 2 || k0 + ZC + 2 > D;
#endif
    if (edge)
        consume<PUSH, true>(ring, xbuf, full, empty, uout, D, H, W, c0, y0, k0, nq, lane, warp, push);
    else
        consume<PUSH, false>(ring, xbuf, full, empty, uout, D, H, W, c0, y0, k0, nq, lane, warp, push);
}

// Consumers.  Round 1 had every warp recompute sweep 1 on one halo row above and below its
// own rows (24 sweep-1 rows per block and plane, a 3 x 6-row register window, spills at the
// 128-register cap); here a warp computes its own 4 rows (warp 0 / 3 also the block's halo
// row above / below: 18 rows) and takes the sweep-1 rows next to its own from its
// neighbours through shared memory: 6 % fewer instructions, no spills, throughput equal
// within noise (power-capped, scripts/r02/gpu_29.sh, gpu_30.sh).  Compact exchange rows:
// 2w + 1 / 2w + 2 = warp w's top / bottom own row, 0 / 9 = the block's halo rows, so warp
// w's row above is 2w and its row below 2w + 3.  One named barrier among the consumer warps
// per plane, after sweep 1 and before the exchange writes, orders (a) the writes of plane
// q-1 after every read of the same buffer (plane q-3) in the previous iteration and (b) the
// reads of plane q-2 after their writes in the previous iteration.  Each value is computed by
// the same expression on the same inputs as in the recomputing version, so the results are
// bit-identical to it.
template <bool PUSH, bool EDGE>
__device__ __forceinline__ void consume(const float* ring, float* xbuf, uint64_t* full, uint64_t* empty,
                                        float* __restrict__ uout, int64_t D, int64_t H, int64_t W, int64_t c0,
                                        int64_t y0, int64_t k0, int nq, int lane, int warp, const PushList& push) {
    const int cx = 4 * lane;
    const int64_t col0 = c0 - 4 + cx;
    const bool wclamp = col0 == 0, eclamp = col0 + 4 >= W;
    const bool store_col = lane >= 1 && lane <= 30 && col0 < W;
    const int Hi = (int)H, Di = (int)D;
    const int gr1 = (int)y0 + kRW * warp - 1;         // grid row of sweep-1 row j = 0 (the row above)
    const int br1 = kRW * warp + 1;                   // its box row
    const int64_t HW = H * W;
    const int64_t rowcol = (int64_t)(gr1 + 1) * W + col0;
    const bool top = warp == 0, bot = warp == kNW - 1;
    float4 L1[3][kRW];                                // own rows j = 1..4 at index j - 1
    int64_t pa = 0, pb = 0;                           // planes of this block a push range may cover
    if (PUSH) dev::push_rows(push, k0, k0 + nq - 4, (uint64_t)HW * 4u, &pa, &pb);
    ptx::mbar_wait(&full[0], 0);
    ptx::mbar_wait(&full[1], 0);
    for (int q0 = 2; q0 < nq; q0 += 3) {
#pragma unroll
        for (int u = 0; u < 3; ++u) {
            const int q = q0 + u;
            if (q >= nq) break;
            ptx::mbar_wait(&full[q % kNS], (uint32_t)((q / kNS) & 1));
            const float* sm = ring + (size_t)((q - 2) % kNS) * kSlot;
            const float* sc = ring + (size_t)((q - 1) % kNS) * kSlot;
            const float* sp = ring + (size_t)(q % kNS) * kSlot;
            const int s1 = (2 + u - 1 + 3) % 3;
            float4 h0 = make_float4(0.f, 0.f, 0.f, 0.f), h5 = h0;
            float4 up, cc;
            if (top) {   // block halo row above (j = 0)
                up = *reinterpret_cast<const float4*>(sc + (br1 - 1) * kCols + cx);
                cc = *reinterpret_cast<const float4*>(sc + br1 * kCols + cx);
                const float4 dn = *reinterpret_cast<const float4*>(sc + (br1 + 1) * kCols + cx);
                const float4 zm = *reinterpret_cast<const float4*>(sm + br1 * kCols + cx);
                const float4 zp = *reinterpret_cast<const float4*>(sp + br1 * kCols + cx);
                const float4 ym = (EDGE && gr1 == 0) ? cc : up;
                const float4 yp = (EDGE && gr1 == Hi - 1) ? cc : dn;
                h0 = sweep(cc, zm, zp, ym, yp, wclamp, eclamp);
                up = cc;
                cc = dn;
            } else {
                up = *reinterpret_cast<const float4*>(sc + br1 * kCols + cx);
                cc = *reinterpret_cast<const float4*>(sc + (br1 + 1) * kCols + cx);
            }
#pragma unroll
            for (int j = 1; j <= kRW; ++j) {
                const int br = br1 + j;
                const int gr = gr1 + j;
                const float4 dn = *reinterpret_cast<const float4*>(sc + (br + 1) * kCols + cx);
                const float4 zm = *reinterpret_cast<const float4*>(sm + br * kCols + cx);
                const float4 zp = *reinterpret_cast<const float4*>(sp + br * kCols + cx);
                const float4 ym = (EDGE && gr == 0) ? cc : up;
                const float4 yp = (EDGE && gr == Hi - 1) ? cc : dn;
                L1[s1][j - 1] = sweep(cc, zm, zp, ym, yp, wclamp, eclamp);
                up = cc;
                cc = dn;
            }
            if (bot) {   // block halo row below (j = 5)
                const int br = br1 + kRW + 1, gr = gr1 + kRW + 1;
                const float4 dn = *reinterpret_cast<const float4*>(sc + (br + 1) * kCols + cx);
                const float4 zm = *reinterpret_cast<const float4*>(sm + br * kCols + cx);
                const float4 zp = *reinterpret_cast<const float4*>(sp + br * kCols + cx);
                const float4 ym = (EDGE && gr == 0) ? cc : up;
                const float4 yp = (EDGE && gr == Hi - 1) ? cc : dn;
                h5 = sweep(cc, zm, zp, ym, yp, wclamp, eclamp);
            }
            // plane seq q-2 is no longer read from the ring by this warp
            __syncwarp();
            if (lane == 0) ptx::mbar_arrive(&empty[(q - 2) % kNS]);
            asm volatile("bar.sync 1, %0;" ::"n"(kNW * 32) : "memory");
            float* xw = xbuf + (size_t)((q - 1) & 1) * kXRows * kCols + cx;   // plane seq q-1
            *reinterpret_cast<float4*>(xw + (2 * warp + 1) * kCols) = L1[s1][0];
            *reinterpret_cast<float4*>(xw + (2 * warp + 2) * kCols) = L1[s1][kRW - 1];
            if (top) *reinterpret_cast<float4*>(xw) = h0;
            if (bot) *reinterpret_cast<float4*>(xw + (kXRows - 1) * kCols) = h5;
            if (q >= 4) {   // sweep 2 on plane seq q-2 = grid plane k0 + q - 4
                const int s0 = (2 + u - 2 + 3) % 3, sM = (2 + u - 3 + 3) % 3;
                const float* xr = xbuf + (size_t)((q - 2) & 1) * kXRows * kCols + cx;   // plane seq q-2
                const float4 above = *reinterpret_cast<const float4*>(xr + (2 * warp) * kCols);
                const float4 below = *reinterpret_cast<const float4*>(xr + (2 * warp + 3) * kCols);
                const int pz = (int)k0 + q - 4;
                const bool zlo = EDGE && pz == 0, zhi = EDGE && pz == Di - 1;

                float* outp = uout + (int64_t)pz * HW + rowcol;
#pragma unroll
                for (int j = 1; j <= kRW; ++j) {
                    const int gr = gr1 + j;
                    const float4 c = L1[s0][j - 1];
                    const float4 zm = zlo ? c : L1[sM][j - 1];
                    const float4 zp = zhi ? c : L1[s1][j - 1];
                    const float4 ym = (EDGE && gr == 0) ? c : (j == 1 ? above : L1[s0][j - 2]);
                    const float4 yp = (EDGE && gr == Hi - 1) ? c : (j == kRW ? below : L1[s0][j]);
                    const float4 o = sweep(c, zm, zp, ym, yp, wclamp, eclamp);
                    if (store_col && (!EDGE || gr < Hi)) {
                        *reinterpret_cast<float4*>(outp) = o;
                        PK_TRACE_W(outp, 16);
                    }
                    outp += W;
                }
                // PUSH: on the (few) planes a push range may cover, re-read the rows this thread
                // just stored (its own writes) and forward them -- outside the row loop, so the
                // update loop carries no store branch
                if (PUSH && dev::in_rows(pz, pa, pb)) {
                    const float* rp = uout + (int64_t)pz * HW + rowcol;
#pragma unroll
                    for (int j = 1; j <= kRW; ++j, rp += W) {
                        const int gr = gr1 + j;
                        if (store_col && (!EDGE || gr < Hi))
                            dev::push4(push, (uint64_t)(rp - uout) * 4u, *reinterpret_cast<const float4*>(rp));
                    }
                }
            }
        }
    }
    __syncwarp();
    if (lane == 0) {
        ptx::mbar_arrive(&empty[(nq - 2) % kNS]);
        ptx::mbar_arrive(&empty[(nq - 1) % kNS]);
    }
}

int describe_heat3d_tb2(pk_ctx c, pk_kernel k) {
    // scalars: 0 = D, 1 = H, 2 = W, 3 = ZC.  Logical block (bx, by, bz) = columns
    // [120 bx, +120) x rows [16 by, +16) x planes [ZC bz, +ZC), guarded.  Reads the
    // clamped 5x5x5 cube around every cell (the box dilated by 2 in every dimension:
    // one tap, positions [b*scale, b*scale + extent + 4) with the guard shifted by 4,
    // offset -2, clamped; corners included -- a read over-approximation);
    // writes its own cells.
    const uint32_t f = PK_DIM_GUARD | PK_DIM_CLAMP;
    pk_affine_access a{};
    a.ndim = 3;
    a.dim[0] = DimMap(2, S(3), S(3, 1, 4), E(-2), f, E(0), S(0, 1, 4));
    a.dim[1] = DimMap(1, E(kRows), E(kRows + 4), E(-2), f, E(0), S(1, 1, 4));
    a.dim[2] = DimMap(0, E(kOwnC), E(kOwnC + 4), E(-2), f, E(0), S(2, 1, 4));
    if (int r = pk_declare_affine_access(c, k, 0, PK_READ, &a)) return r;
    pk_affine_access w{};
    w.ndim = 3;
    w.dim[0] = DimMap(2, S(3), S(3), E(0), f, E(0), S(0));
    w.dim[1] = DimMap(1, E(kRows), E(kRows), E(0), f, E(0), S(1));
    w.dim[2] = DimMap(0, E(kOwnC), E(kOwnC), E(0), f, E(0), S(2));
    return pk_declare_affine_access(c, k, 1, PK_WRITE, &w);
}

cudaError_t launch_heat3d_tb2(const LaunchInfo& li) {
    if (li.nscalars < 4) return cudaErrorInvalidValue;
    int64_t D = li.scalars[0], H = li.scalars[1], W = li.scalars[2], ZC = li.scalars[3];
    if (W % 4 || W < 4 || ZC < 1 || H < 1 || D < 1) return cudaErrorInvalidValue;
    if (H >= (int64_t)1 << 30 || D >= (int64_t)1 << 30) return cudaErrorInvalidValue;   // 32-bit row/plane indices
    const bool push = li.push && li.push->n > 0;
    const void* fn = push ? (const void*)k_heat3d_tb2<true> : (const void*)k_heat3d_tb2<false>;
    KernelDevInfo kd;   // per device: the opt-in above 48 KB is a (function, device) attribute
    if (cudaError_t e = prepare_kernel(fn, li.device, kSmem, (kNW + 1) * 32, &kd)) return e;
    // tensor map of this instance: dims (W, H, D), box (128, 20, 1), OOB zero fill
    static std::mutex mu;
    static std::unordered_map<const void*, std::pair<uint64_t, CUtensorMap>> cache;
    CUtensorMap tm;
    {
        std::lock_guard<std::mutex> g(mu);
        const uint64_t key = ((uint64_t)W * 1315423911ull) ^ ((uint64_t)H << 20) ^ ((uint64_t)D << 40);
        auto it = cache.find(li.inst[0]);
        if (it != cache.end() && it->second.first == key) {
            tm = it->second.second;
        } else {
            cuuint64_t dims[3] = {(cuuint64_t)W, (cuuint64_t)H, (cuuint64_t)D};
            cuuint32_t box[3] = {(cuuint32_t)kCols, (cuuint32_t)kBoxRows, 1};
            if (!tma_encode_f32(&tm, li.inst[0], 3, dims, box, CU_TENSOR_MAP_SWIZZLE_NONE))
                return cudaErrorInvalidValue;
            cache[li.inst[0]] = {key, tm};
        }
    }
    PushList pl{};
    if (li.push) pl = *li.push;
    void* argv[] = {&tm, (void*)&li.inst[1], &D, &H, &W, &ZC, (void*)&li.part, &pl, (void*)&li.inst[0]};
    return cudaLaunchKernel(fn, li.grid, dim3((kNW + 1) * 32), argv, kSmem, li.stream);
}

}  // namespace

const Builtin kBuiltinHeat3dTb2 = {
    "heat3d_tb2", (const void*)k_heat3d_tb2<false>, 6,
    {PK_ARG_BUFFER, PK_ARG_BUFFER, PK_ARG_SCALAR, PK_ARG_SCALAR, PK_ARG_SCALAR, PK_ARG_SCALAR}, -1,
    describe_heat3d_tb2, launch_heat3d_tb2, /*push_arg=*/1};

}  // namespace pk
