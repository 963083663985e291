// sgemm_tc.cu -- C4: FP32 GEMM C = A * B on the 5th-generation tensor cores
// (tcgen05 + TMEM + TMA, CTA pairs), 3xTF32 split for FP32-level accuracy.
//
// PAPER.md P:L995-1005 (§9.1 "Matmul computes the product of two dense,
// quadratic matrices ... The second matrix of the product is read column-wise
// by each thread"); reading Q17: row-major C = A B, alpha = 1, beta = 0.
//
// Split (reading Q17): x = hi + lo with hi = x truncated to TF32 (low 13
// mantissa bits cleared, exactly representable), lo = round_tf32(x - hi);
//   C = A_hi B_hi + A_hi B_lo + A_lo B_hi     (the A_lo B_lo term is < 2^-20 relative)
// accumulated in FP32, no split-K (so a P-way row partition is bit-identical to the
// 1-way launch).
//
// ONE kernel per partition, reading the fp32 operands straight from HBM -- no split
// pre-pass, no hi/lo scratch (round 1 split A and B into 4 GiB of hi/lo scratch per
// launch and re-streamed both halves; DRAM traffic was 9.4x the algorithmic bytes):
//   * a cluster of 2 CTAs on 2 SMs computes a 256 x 256 C tile with
//     tcgen05.mma.cta_group::2 (M = 256, N = 256, K = 8): each CTA holds its 128 rows of
//     A and HALF of the B tile (128 columns), so the pair streams the B tile once and
//     each SM's shared memory carries half of it -- the operand and converter traffic
//     a single-CTA 128 x 256 tile could not sustain (ncu: the shared-memory pipe was the
//     limit at 1 CTA, tensor pipe 68 %);
//   * TMA loads the raw fp32 tiles: A 128 x 16 (K-major, 64-B swizzle) and the B half
//     16 x 128 straight from row-major B as four 32-column MN-major boxes in the
//     128-B / 32-B-atom swizzle (the tf32 kind accepts MN-major B in that layout, so no
//     transpose);
//   * kind::tf32 ignores the low 13 mantissa bits of its fp32 operands, so the raw tile
//     IS the hi operand; ten converter warps per CTA write lo = round_tf32(x - hi) of
//     every element into a second buffer of the same layout (an elementwise pass);
//   * the leader CTA's single MMA thread issues hi.hi, hi.lo, lo.hi per K-step of 8.
//
// Chunked accumulation: the tensor core's FP32 accumulator loses the bits below its
// alignment on every MMA (measured round 1: error / RMS(C) grows LINEARLY with K,
// 3.5e-4 at K = 16384 with one accumulator), so a TMEM accumulator only spans
// KC = 512 of K: the MMA thread alternates between two TMEM accumulators and the
// epilogue warps add each finished chunk into FP32 registers (round-to-nearest).
//
// Diagonal chunk order: tile-row pair r of R starts its K loop at chunk floor(r *
// nchunks / R) and wraps around.  The order is a function of the tile's position only
// (pairs are aligned to even global tile rows), so a P-way row partition stays
// bit-identical to the 1-way launch, and with P row slabs of B (linear
// H2D, or the slabs the previous GEMM of an iteration wrote) a partition starts on the
// chunks it holds itself while the other slabs arrive.
//
// Streamed B (LaunchInfo::arrival, runtime "streamed operand"): the runtime copies the
// stale granules of B on a side stream while this kernel runs; the TMA producers poll
// the granule's arrival flag before the first load of a chunk -- the operand all-gather
// fused into the GEMM's pipeline (P:L999-1004 names that redistribution as Matmul's
// scaling limit).
//
// Per CTA, 12 warps:
//   warp 0    TMA producer (6 stages of 32 KB: raw A, raw B half, lo A, lo B half)
//   warp 1    MMA issuer (leader CTA only: one thread, tcgen05.mma.cta_group::2.kind::tf32)
//   warps 2-11 converters, one slice of every stage each (warp 2 also allocates TMEM:
//             2 x 256 columns, cta_group::2); warps 4-11 are also the epilogue
//             (tcgen05.ld 32x32b -> FP32 running sums -> global), draining chunk j-1
//             early in chunk j
// A pair whose second tile row lies outside the partition (odd row counts) runs with a
// "phantom" CTA: its A box is fully out of bounds (zero fill, nothing read) and it
// stores nothing.
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>

#include "../runtime/builtins.h"
#include "launch_util.h"
#include "trace.cuh"
#include "ptx.cuh"
#include "tma_host.h"

namespace pk {
namespace {

#ifndef PK_SGEMM_DIAG
#define PK_SGEMM_DIAG 8
#endif
constexpr int BM = 128, BN = 256, BK = 16, STAGES = 6;  // BM: rows per CTA (256 per pair)
constexpr int BNH = BN / 2;                         // B columns held by each CTA of the pair
constexpr int A_TILE = BM * BK * 4;                 // 8 KB
constexpr int B_TILE = BNH * BK * 4;                // 8 KB: this CTA's half of the B tile
constexpr int RAW_BYTES = A_TILE + B_TILE;          // 16 KB: what TMA writes per stage and CTA
constexpr int STAGE_BYTES = 2 * RAW_BYTES;          // + the lo copy of both tiles
constexpr int B_GROUP = 32;                         // N columns per 128-B swizzle box
constexpr int B_GROUP_BYTES = BK * 128;             // 2 KB: one box of 16 K rows x 128 B
constexpr int kThreads = 384;
constexpr int EPI_COLS = BN / 2;                    // columns per epilogue thread
constexpr int TMEM_COLS = 2 * BN;                   // two accumulators
constexpr int KC_BLOCKS = 32;                       // K per TMEM accumulator chunk = 32 * BK = 512
constexpr int kConvWarps = 10;                      // warps 2..11 convert (4..11 are also the epilogue)
constexpr size_t SMEM_BYTES = (size_t)STAGES * STAGE_BYTES + 1024 + 256;

// lo = round_tf32(x - hi), round to nearest even: one native F2FP.TF32 (cvt.rna -- ties
// away -- is emulated in 3 instructions); the bound |lo - (x - hi)| <= 2^-22 |x| is the same
__device__ __forceinline__ uint32_t lo_tf32(uint32_t x) {
    const float hi = __uint_as_float(x & 0xFFFFE000u);
    const float r = __uint_as_float(x) - hi;  // exact
    uint32_t t;
    asm("cvt.rn.tf32.f32 %0, %1;" : "=r"(t) : "f"(r));
    return t;
}
__device__ __forceinline__ uint4 lds128(uint32_t a) {
    uint4 v;
    asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(a));
    return v;
}
__device__ __forceinline__ void sts128(uint32_t a, uint4 v) {
    asm volatile("st.shared.v4.u32 [%0], {%1,%2,%3,%4};" ::"r"(a), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
}

// ---------------------------------------------------------------- tcgen05 helpers
// K-major, SWIZZLE_64B canonical layout (A): rows of 64 B, 8-row atoms of 512 B
__device__ __forceinline__ uint64_t umma_desc_k_sw64(uint32_t smem_addr) {
    uint64_t d = 0;
    d |= (uint64_t)((smem_addr >> 4) & 0x3FFFu);        // start address
    d |= (uint64_t)1u << 16;                            // LBO (unused for swizzled K-major) = 1
    d |= (uint64_t)(512u >> 4) << 32;                   // SBO = 512 B between 8-row groups
    d |= (uint64_t)1u << 46;                            // version = 1 (sm_100)
    d |= (uint64_t)4u << 61;                            // layout = SWIZZLE_64B
    return d;
}
// MN-major 32-bit operands have ONE canonical smem layout on sm_100: 128-B swizzle with
// 32-B atoms (SWIZZLE_128B_BASE32B; TMA: CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B) -- 128-B rows
// of 32 N values, K rows grouped by 4 (512 B, SBO), the next 32 N values (LBO) in the next
// TMA box, B_GROUP_BYTES further
__device__ __forceinline__ uint64_t umma_desc_mn_sw128_32b(uint32_t smem_addr) {
    uint64_t d = 0;
    d |= (uint64_t)((smem_addr >> 4) & 0x3FFFu);
    d |= (uint64_t)((B_GROUP_BYTES >> 4) & 0x3FFFu) << 16;   // LBO: N-group stride
    d |= (uint64_t)(512u >> 4) << 32;                       // SBO: 4-row K-group stride
    d |= (uint64_t)1u << 46;
    d |= (uint64_t)1u << 61;                                // layout = SWIZZLE_128B_BASE32B
    return d;
}

// instruction descriptor: kind::tf32, D = F32, A = B = TF32, A K-major, B MN-major
__host__ __device__ constexpr uint32_t idesc_tf32(int m, int n) {
    return (1u << 4)                   // c_format = F32
           | (2u << 7)                 // a_format = TF32
           | (2u << 10)                // b_format = TF32
           | (0u << 15)                // a_major = K
           | (1u << 16)                // b_major = MN
           | ((uint32_t)(n >> 3) << 17)
           | ((uint32_t)(m >> 4) << 24);
}

// M = 256 across the CTA pair: rows 0-127 from the leader's smem / TMEM, 128-255 from the peer's
__device__ __forceinline__ void umma_tf32_2sm(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                              uint32_t accumulate) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::2.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_d),
        "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate));
}

// completion of the pair's MMAs arrives on the barrier at this offset in BOTH CTAs
__device__ __forceinline__ void umma_commit_pair(uint64_t* bar) {
    asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
                     ptx::smem_u32(bar)),
                 "h"((uint16_t)3)
                 : "memory");
}

// the same shared-memory offset in CTA `rank` of the cluster
__device__ __forceinline__ uint32_t mapa(uint32_t addr, uint32_t rank) {
    uint32_t r;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(addr), "r"(rank));
    return r;
}
// Relaxed remote arrive: one SYNCS instruction.  (.release.cluster compiles to MEMBAR.ALL.GPU +
// ERRBAR + CGAERRBAR before it, microseconds per stage on the forwarding thread.)  What it
// publishes is already ordered: the converters' smem writes are fenced to the async proxy and
// released to the forwarder through the local barrier (acquire on wait); TMEM reads of the
// epilogue are complete (tcgen05.wait::ld) before its arrive.
__device__ __forceinline__ void arrive_cluster(uint32_t cluster_addr) {
    asm volatile("mbarrier.arrive.relaxed.cluster.shared::cluster.b64 _, [%0];" ::"r"(cluster_addr) : "memory");
}
__device__ __forceinline__ uint32_t cluster_rank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ void cluster_sync() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

__device__ __forceinline__ void tma_2d(void* dst, const CUtensorMap* map, int32_t c0, int32_t c1, uint64_t* bar) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(
            ptx::smem_u32(dst)),
        "l"(map), "r"(c0), "r"(c1), "r"(ptx::smem_u32(bar))
        : "memory");
}

__device__ __forceinline__ void tmem_ld16(uint32_t taddr, float (&v)[16]) {
    uint32_t r[16];
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
          "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
        : "r"(taddr));
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
    for (int i = 0; i < 16; ++i) v[i] = __uint_as_float(r[i]);
}

__device__ __forceinline__ uint32_t ld_acquire_u32(const uint32_t* p) {
    uint32_t v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

// chunk of K processed j-th by a tile in tile row `rt` (of `nrt`): diagonal start, wrap.  The
// start is quantised to eighths of K (the row slabs of up to 8 partitions): the pairs running
// at the same time then mostly stream the same B k-slices, which L2 serves once
constexpr int kDiagSlabs = PK_SGEMM_DIAG;
__device__ __forceinline__ int chunk_at(int j, int64_t rt, int64_t nrt, int nchunks) {
    const int c0 = (int)(((rt * kDiagSlabs) / nrt) * nchunks / kDiagSlabs);  // rt / nrt: pair / pairs of the grid
    const int c = c0 + j;
    return c >= nchunks ? c - nchunks : c;
}

// ---------------------------------------------------------------- the GEMM
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(kThreads, 1)
    k_sgemm_tf32x3(const __grid_constant__ CUtensorMap tm_a, const __grid_constant__ CUtensorMap tm_b,
                   float* __restrict__ C, int64_t M, int64_t N, int64_t K, pk_partition part, Arrival arr,
                   const float* a_trace, const float* b_trace) {
    extern __shared__ __align__(1024) unsigned char smem_raw[];
    unsigned char* smem = smem_raw + ((1024u - ((uint32_t)(uintptr_t)smem_raw & 1023u)) & 1023u);
    uint64_t* full = reinterpret_cast<uint64_t*>(smem + (size_t)STAGES * STAGE_BYTES);
    uint64_t* conv = full + STAGES;        // [STAGES]: lo written by this CTA's converters
    uint64_t* conv_peer = conv + STAGES;   // [STAGES] (leader): forwarded "peer converted" signal
    uint64_t* empty = conv_peer + STAGES;  // [STAGES]: the pair's MMAs of the stage are done
    uint64_t* acc_full = empty + STAGES;   // [2]: chunk finished in accumulator a (both CTAs)
    uint64_t* acc_empty = acc_full + 2;    // [2] (leader): accumulator a drained by both epilogues
    uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(acc_empty + 2);

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t rank = cluster_rank();   // 0 = leader (issues the MMAs), 1 = peer
    // Tile pairs: the cluster computes tile rows (2 pr, 2 pr + 1) of one 256-column band.
    // Pairs are aligned to even GLOBAL tile rows, so the pairing and the chunk order do not
    // depend on the partition; grouped rasterisation: the clusters running at the same time
    // cover kGroup pairs x (wave / kGroup) bands, so a B k-slice is read about once per kGroup
    // pairs.  The cluster -> (pair, band) map is a bijection onto the pairs that intersect
    // the partition's box, so the launch computes exactly the blocks [min, max) (Eq. 8-10).
    constexpr int kGroup = 8;
    const int64_t gx = part.max[0] - part.min[0];
    const int64_t p0 = part.min[1] / 2, np = (part.max[1] + 1) / 2 - p0;   // pairs touching [min, max)
    const int64_t L = (int64_t)blockIdx.x / 2;
    const int64_t grp = L / (kGroup * gx);
    const int64_t pg0 = grp * kGroup;
    const int64_t gsz = (np - pg0) < kGroup ? (np - pg0) : kGroup;
    const int64_t in = L - grp * kGroup * gx;
    const int64_t pr = p0 + pg0 + in % gsz;                 // global pair index
    const int64_t rt = 2 * pr + rank;                       // this CTA's global tile row (Eq. 8)
    const bool live = rt >= part.min[1] && rt < part.max[1];   // else a phantom: no A reads, no stores
    const int64_t m0 = rt * BM;
    const int64_t n0 = (int64_t)(part.min[0] + in / gsz) * BN;
    const int64_t nb0 = n0 + (int64_t)rank * BNH;           // this CTA's half of the B columns
    const int64_t npr = (part.grid[1] + 1) / 2;              // pairs of the FULL grid (Eq. 9)
    const int nk = (int)((K + BK - 1) / BK);
    const int nchunks = (nk + KC_BLOCKS - 1) / KC_BLOCKS;

    if (warp == 0 && lane == 0) {
        for (int s = 0; s < STAGES; ++s) {
            ptx::mbar_init(&full[s], 1);
            ptx::mbar_init(&conv[s], kConvWarps);
            ptx::mbar_init(&conv_peer[s], 1);
            ptx::mbar_init(&empty[s], 1);
        }
        for (int a = 0; a < 2; ++a) {
            ptx::mbar_init(&acc_full[a], 1);
            ptx::mbar_init(&acc_empty[a], 2 * 8);   // one arrival per epilogue warp of both CTAs
        }
        ptx::fence_mbar_init();
        asm volatile("prefetch.tensormap [%0];" ::"l"(&tm_a) : "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"(&tm_b) : "memory");
    }
    if (warp == 2) {
        asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                         ptx::smem_u32(tmem_holder)),
                     "r"(TMEM_COLS)
                     : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    cluster_sync();   // both CTAs' barriers initialised and TMEM allocated before any cross-CTA traffic
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tmem = *tmem_holder;

    if (warp == 0 && lane == 0) {
        // ---------------- TMA producer (both CTAs: own A rows, own half of the B band)
        const uint64_t row_bytes = (uint64_t)N * 4;
        const int32_t arow = live ? (int32_t)m0 : (int32_t)M;    // phantom: a fully out-of-bounds box
        int it = 0;
        for (int j = 0; j < nchunks; ++j) {
            const int c = chunk_at(j, pr, npr, nchunks);
            const int kb0 = c * KC_BLOCKS, kb1 = min(kb0 + KC_BLOCKS, nk);
            if (arr.wait) {
                // streamed B: every granule the chunk's rows touch must have landed
                const uint64_t g0 = (uint64_t)kb0 * BK * row_bytes / arr.granule;
                const uint64_t g1 = ((uint64_t)min((int64_t)kb1 * BK, K) * row_bytes - 1) / arr.granule;
                for (uint64_t g = g0; g <= g1 && g < (uint64_t)kMaxGranules; ++g)
                    if ((arr.wait >> g) & 1ull) {
                        const long long t0 = clock64();
                        while (ld_acquire_u32(arr.flags + g) == 0u) {
                            __nanosleep(128);
                            // a copy that never lands is a runtime bug: fail loudly, do not hang
                            if (clock64() - t0 > 60000000000ll) __trap();
                        }
                    }
                asm volatile("fence.proxy.async.global;" ::: "memory");  // generic acquire -> TMA reads
            }
            for (int kb = kb0; kb < kb1; ++kb, ++it) {
                const int s = it % STAGES;
                const uint32_t ph = (it / STAGES) & 1u;
                ptx::mbar_wait(&empty[s], ph ^ 1u);
                unsigned char* st = smem + (size_t)s * STAGE_BYTES;
                ptx::mbar_arrive_expect_tx(&full[s], RAW_BYTES);
                const int32_t kc = kb * BK;
                tma_2d(st, &tm_a, kc, arow, &full[s]);
#pragma unroll
                for (int g = 0; g < BNH / B_GROUP; ++g)
                    tma_2d(st + A_TILE + g * B_GROUP_BYTES, &tm_b, (int32_t)(nb0 + g * B_GROUP), kc, &full[s]);
                if (live) PK_TRACE_BOX(a_trace, M, K, kc, BK, m0, BM, 0);
                PK_TRACE_BOX(b_trace, K, N, nb0, BNH, kc, BK, 0);
            }
        }
    } else if (warp == 1) {
        // ---------------- MMA issuer: one thread of the leader CTA, for the pair.  In the peer
        // CTA this thread forwards "stage converted" to the leader: one remote arrive per
        // stage (ten, one per converter warp, each behind a GPU-scope membar when they were
        // release.cluster arrives: ncu, 40 % of the stall samples)
        if (rank == 1 && lane == 0) {
            const uint32_t fwd = mapa(ptx::smem_u32(conv_peer), 0);
            for (int it = 0; it < nk; ++it) {
                const int s = it % STAGES;
                ptx::mbar_wait(&conv[s], (it / STAGES) & 1u);
                arrive_cluster(fwd + 8u * (uint32_t)s);
            }
        }
        if (rank == 0 && lane == 0) {
            constexpr uint32_t idesc = idesc_tf32(2 * BM, BN);
            int it = 0;
            for (int j = 0; j < nchunks; ++j) {
                const int c = chunk_at(j, pr, npr, nchunks);
                const int kb0 = c * KC_BLOCKS, kb1 = min(kb0 + KC_BLOCKS, nk);
                const int a = j & 1;
                if (j >= 2)  // accumulator a still holds chunk j-2 until both epilogues drained it
                    ptx::mbar_wait(&acc_empty[a], (uint32_t)((j / 2 - 1) & 1));
                const uint32_t acc = tmem + (uint32_t)(a * BN);
                for (int kb = kb0; kb < kb1; ++kb, ++it) {
                    const int s = it % STAGES;
                    ptx::mbar_wait(&conv[s], (it / STAGES) & 1u);        // own raw + lo tiles ready
                    ptx::mbar_wait(&conv_peer[s], (it / STAGES) & 1u);   // the peer's too
                    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
                    const uint32_t st = ptx::smem_u32(smem + (size_t)s * STAGE_BYTES);
#pragma unroll
                    for (int kk = 0; kk < BK / 8; ++kk) {
                        const uint64_t ahi = umma_desc_k_sw64(st + kk * 32);            // 8 TF32 = 32 B along K
                        const uint64_t alo = umma_desc_k_sw64(st + RAW_BYTES + kk * 32);
                        const uint64_t bhi = umma_desc_mn_sw128_32b(st + A_TILE + kk * 1024);  // next 8 K rows
                        const uint64_t blo = umma_desc_mn_sw128_32b(st + RAW_BYTES + A_TILE + kk * 1024);
                        umma_tf32_2sm(acc, ahi, bhi, idesc, (kb == kb0 && kk == 0) ? 0u : 1u);
                        umma_tf32_2sm(acc, ahi, blo, idesc, 1u);
                        umma_tf32_2sm(acc, alo, bhi, idesc, 1u);
                    }
                    umma_commit_pair(&empty[s]);  // frees the stage in both CTAs when these MMAs complete
                }
                umma_commit_pair(&acc_full[a]);
            }
        }
    } else if (warp >= 2) {
        // ---------------- converters (warps 2..11): lo = round_tf32(x - hi) of every raw element,
        // same layout, each warp a contiguous slice of the stage.  Warps 4..11 are also the
        // epilogue: they drain chunk j-1's accumulator once they have converted the first
        // stages of chunk j (the MMA then works on chunk j, so chunk j-1 is complete or about to
        // be), which leaves the 2 dedicated converter warps alone only for the drain.
        const int cw = warp - 2;                                  // converter index 0..9
        const int u0 = (RAW_BYTES / 16) * cw / kConvWarps, u1 = (RAW_BYTES / 16) * (cw + 1) / kConvWarps;
        const bool epi = warp >= 4;
        const int q = warp & 3;                     // TMEM lane quarter of this warp (epilogue)
        const int half = (warp - 4) >> 2;           // column half of the tile (epilogue)
        const uint32_t accempty_leader = mapa(ptx::smem_u32(acc_empty), 0);
        float sum[EPI_COLS];
#pragma unroll
        for (int i = 0; i < EPI_COLS; ++i) sum[i] = 0.f;
        auto drain = [&](int jd) {
            const int a = jd & 1;
            ptx::mbar_wait(&acc_full[a], (uint32_t)((jd / 2) & 1));
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
#pragma unroll
            for (int c = 0; c < EPI_COLS; c += 16) {
                float v[16];
                tmem_ld16(tmem + ((uint32_t)(32 * q) << 16) + (uint32_t)(a * BN + half * EPI_COLS + c), v);
#pragma unroll
                for (int i = 0; i < 16; ++i) sum[c + i] += v[i];   // round-to-nearest FP32 add, chunk order
            }
            asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
            __syncwarp();
            if (lane == 0) arrive_cluster(accempty_leader + 8u * (uint32_t)a);
        };
        int it = 0;
        for (int j = 0; j < nchunks; ++j) {
            const int c = chunk_at(j, pr, npr, nchunks);
            const int nst = min(c * KC_BLOCKS + KC_BLOCKS, nk) - c * KC_BLOCKS;
            for (int x = 0; x < nst; ++x, ++it) {
                const int s = it % STAGES;
                ptx::mbar_wait(&full[s], (it / STAGES) & 1u);
                // shared-space addresses: LDS/STS (a generic pointer here compiled to LD.E/ST.E)
                const uint32_t base = ptx::smem_u32(smem + (size_t)s * STAGE_BYTES);
                for (int u = u0 + lane; u < u1; u += 32) {
                    const uint4 v = lds128(base + 16u * (uint32_t)u);
                    sts128(base + RAW_BYTES + 16u * (uint32_t)u,
                           make_uint4(lo_tf32(v.x), lo_tf32(v.y), lo_tf32(v.z), lo_tf32(v.w)));
                }
                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // generic writes -> tensor core
                __syncwarp();
                if (lane == 0) ptx::mbar_arrive(&conv[s]);
                if (epi && j >= 1 && x == min(STAGES, nst) - 1) drain(j - 1);
            }
        }
        if (epi) {
            drain(nchunks - 1);
            const int64_t row = m0 + 32 * q + lane;
            if (live && row < M) {
                const int64_t c0 = n0 + half * EPI_COLS;
                float* dst = C + row * N + c0;
#pragma unroll
                for (int c = 0; c < EPI_COLS; c += 4) {
                    if (c0 + c + 4 <= N && (N % 4) == 0) {
                        *reinterpret_cast<float4*>(dst + c) = make_float4(sum[c], sum[c + 1], sum[c + 2], sum[c + 3]);
                        PK_TRACE_W(dst + c, 16);
                    } else {
                        for (int i = 0; i < 4; ++i)
                            if (c0 + c + i < N) {
                                dst[c + i] = sum[c + i];
                                PK_TRACE_W(dst + c + i, 4);
                            }
                    }
                }
            }
        }
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    cluster_sync();   // the leader's MMAs read the peer's smem; remote arrivals target the leader
    if (warp == 2) {
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(TMEM_COLS) : "memory");
    }
}

// ---------------------------------------------------------------- host side
// 2-D fp32 tensor map: dims {inner, outer}, box {box_inner, box_outer}
bool make_map(CUtensorMap* m, const float* base, int64_t outer, int64_t inner, uint32_t box_inner, uint32_t box_outer,
              CUtensorMapSwizzle swz) {
    EncodeTiledFn enc = tma_encode_fn();
    if (!enc) return false;
    cuuint64_t dims[2] = {(cuuint64_t)inner, (cuuint64_t)outer};
    cuuint64_t strides[1] = {(cuuint64_t)inner * 4};
    cuuint32_t box[2] = {box_inner, box_outer};
    cuuint32_t estr[2] = {1, 1};
    return enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, (void*)base, dims, strides, box, estr,
               CU_TENSOR_MAP_INTERLEAVE_NONE, swz, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

int describe_sgemm(pk_ctx c, pk_kernel k) {
    // scalars: 0 = M, 1 = N, 2 = K.  Logical block (bx, by) = C tile rows
    // [128 by, +128) x cols [256 bx, +256), guarded; it reads the A row band over
    // all of K and the B column band over all of K (B "read column-wise").
    pk_affine_access a{};
    a.ndim = 2;
    a.dim[0] = DimMap(1, E(BM), E(BM), E(0), PK_DIM_GUARD, E(0), S(0));
    a.dim[1] = DimMap(-1, E(0), S(2), E(0), 0);
    if (int r = pk_declare_affine_access(c, k, 0, PK_READ, &a)) return r;
    pk_affine_access b{};
    b.ndim = 2;
    b.dim[0] = DimMap(-1, E(0), S(2), E(0), 0);
    b.dim[1] = DimMap(0, E(BN), E(BN), E(0), PK_DIM_GUARD, E(0), S(1));
    if (int r = pk_declare_affine_access(c, k, 1, PK_READ, &b)) return r;
    pk_affine_access w{};
    w.ndim = 2;
    w.dim[0] = DimMap(1, E(BM), E(BM), E(0), PK_DIM_GUARD, E(0), S(0));
    w.dim[1] = DimMap(0, E(BN), E(BN), E(0), PK_DIM_GUARD, E(0), S(1));
    return pk_declare_affine_access(c, k, 2, PK_WRITE, &w);
}

// streamed-B granule: whole 512-row K chunks of B (so a chunk waits for whole granules),
// as many per granule as keep the count <= kMaxGranules
uint64_t sgemm_granule(const int64_t* sc, int ns) {
    if (ns < 3 || sc[1] < 1 || sc[2] < 1) return 0;
    const int64_t N = sc[1], K = sc[2];
    const int64_t kc = (int64_t)KC_BLOCKS * BK;
    const int64_t nch = (K + kc - 1) / kc;
    const int64_t per = (nch + kMaxGranules - 1) / kMaxGranules;
    return (uint64_t)(per * kc) * (uint64_t)N * 4u;
}

cudaError_t launch_sgemm(const LaunchInfo& li) {
    if (li.nscalars < 3) return cudaErrorInvalidValue;
    int64_t M = li.scalars[0], N = li.scalars[1], K = li.scalars[2];
    // TMA: row strides of A (K) and B (N) must be 16-byte multiples
    if (M < 1 || N < 1 || K < 4 || K % 4 || N % 4) return cudaErrorInvalidValue;
    if (K > (int64_t)KC_BLOCKS * BK * (1 << 20)) return cudaErrorInvalidValue;
    const float* A = (const float*)li.inst[0];
    const float* B = (const float*)li.inst[1];
    float* C = (float*)li.inst[2];
    CUtensorMap tm[2];
    if (!make_map(&tm[0], A, M, K, BK, BM, CU_TENSOR_MAP_SWIZZLE_64B) ||
        !make_map(&tm[1], B, K, N, B_GROUP, BK, CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B))
        return cudaErrorInvalidValue;
    KernelDevInfo kd;   // per device: the opt-in above 48 KB is a (function, device) attribute
    cudaError_t e = prepare_kernel((const void*)k_sgemm_tf32x3, li.device, SMEM_BYTES, kThreads, &kd, false);
    if (e != cudaSuccess) return e;
    Arrival arr = li.arrival;
    if (arr.wait && (!arr.flags || arr.granule == 0)) return cudaErrorInvalidValue;
    // one 2-CTA cluster per (tile-row pair, 256-column band) that intersects the partition box
    const int64_t gx = li.part.max[0] - li.part.min[0];
    const int64_t np = (li.part.max[1] + 1) / 2 - li.part.min[1] / 2;
    if (gx <= 0 || np <= 0) return cudaSuccess;
    if (2 * gx * np > 0x7fffffffll) return cudaErrorInvalidValue;
    void* argv[] = {&tm[0], &tm[1], &C, &M, &N, &K, (void*)&li.part, &arr, (void*)&li.inst[0], (void*)&li.inst[1]};
    return cudaLaunchKernel((const void*)k_sgemm_tf32x3, dim3((unsigned)(2 * gx * np)), dim3(kThreads), argv,
                            SMEM_BYTES, li.stream);
}

}  // namespace

const Builtin kBuiltinSgemm = {"sgemm_tf32x3", (const void*)k_sgemm_tf32x3, 6,
                               {PK_ARG_BUFFER, PK_ARG_BUFFER, PK_ARG_BUFFER, PK_ARG_SCALAR, PK_ARG_SCALAR,
                                PK_ARG_SCALAR},
                               -1, describe_sgemm, launch_sgemm, /*push_arg=*/-1, /*stream_arg=*/1,
                               sgemm_granule};

}  // namespace pk
