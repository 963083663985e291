// sgemm_tc.cu -- C4: FP32 GEMM C = A * B on the 5th-generation tensor cores
// (tcgen05 + TMEM + TMA), 3xTF32 split for FP32-level accuracy.
//
// PAPER.md P:L995-1005 (§9.1 "Matmul computes the product of two dense,
// quadratic matrices ... The second matrix of the product is read column-wise
// by each thread"); reading Q17: row-major C = A B, alpha = 1, beta = 0.
//
// Split (reading Q17): x = hi + lo with hi = x truncated to TF32 (low 13
// mantissa bits cleared, exactly representable), lo = round_tf32(x - hi);
//   C = A_hi B_hi + A_hi B_lo + A_lo B_hi     (the A_lo B_lo term is < 2^-20 relative)
// accumulated in FP32, fixed K order, no split-K (so a P-way row partition is
// bit-identical to the 1-way launch).
//
// Chunked accumulation: the tensor core's FP32 accumulator loses the bits below
// its alignment on every MMA (measured: the error relative to RMS(C) grows
// LINEARLY with K -- 2.3e-5 at K = 1024, 3.5e-4 at K = 16384, 1.4e-3 at 65536 for a
// single TMEM accumulator, i.e. each element drifts toward zero by ~2^-23 of its
// running value per MMA).  So the TMEM accumulator only spans KC = 512 of K: the
// MMA warp alternates between two TMEM accumulators, and the epilogue warps add
// each finished chunk into FP32 registers (round-to-nearest) while the next chunk
// is being computed.  The error then grows with the chunk length, not with K.
//
// Per partitioned launch the launcher runs, on the partition's stream:
//   1. k_split_rows   : A rows of this partition -> A_hi, A_lo (M x K, K-major)
//   2. k_split_transp : all of B (K x N) -> Bt_hi, Bt_lo (N x K, K-major)
//   3. k_sgemm_tf32x3 : one CTA per 128 x 256 C tile (logical block), 12 warps:
//        warp 0   TMA producer (cp.async.bulk.tensor.2d, 64-B swizzle, 4 stages)
//        warp 1   MMA issuer (one thread: tcgen05.mma.cta_group::1.kind::tf32,
//                 M = 128, N = 256, K = 8 per instruction, 3 per K-step)
//        warp 2   TMEM allocator (2 x 256 columns: two 128 x 256 FP32 accumulators)
//        warps 4-11 epilogue (tcgen05.ld 32x32b -> FP32 running sums in registers,
//                 128 per thread = half a C row -> global)
// (N = 128 tiles with 4 epilogue warps were tried for the chunked accumulation:
// shared-memory bound, 181 vs 258 TF/s: operand reads + TMA fills exceed 128 B/clk.)
// Scratch (hi/lo operands) is private to the launch, allocated per stream.
#include <cuda.h>
#include <cuda_runtime.h>

#include <mutex>
#include <unordered_map>

#include "../runtime/builtins.h"
#include "launch_util.h"
#include "trace.cuh"
#include "ptx.cuh"

namespace pk {
namespace {

constexpr int BM = 128, BN = 256, BK = 16, STAGES = 4;
constexpr int A_TILE = BM * BK * 4;                 // 8 KB
constexpr int B_TILE = BN * BK * 4;                 // 16 KB
constexpr int STAGE_BYTES = 2 * A_TILE + 2 * B_TILE; // 48 KB
constexpr int kThreads = 384;                       // 4 role warps + 8 epilogue warps
constexpr int EPI_COLS = BN / 2;                    // columns per epilogue thread
constexpr int TMEM_COLS = 2 * BN;                   // two accumulators
constexpr int KC_BLOCKS = 32;                       // K per TMEM accumulator chunk = 32 * BK = 512
constexpr size_t SMEM_BYTES = (size_t)STAGES * STAGE_BYTES + 1024 + 256;

// ---------------------------------------------------------------- split kernels
__device__ __forceinline__ void split_tf32(float x, float& hi, float& lo) {
    hi = __uint_as_float(__float_as_uint(x) & 0xFFFFE000u);
    const float r = x - hi;  // exact
    uint32_t t;
    asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(t) : "f"(r));
    lo = __uint_as_float(t);
}

__global__ void k_split_rows(const float* __restrict__ x, float* __restrict__ hi, float* __restrict__ lo,
                             int64_t r0, int64_t r1, int64_t cols) {
    const int64_t n = (r1 - r0) * cols;
    const int64_t base = r0 * cols;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        float h, l;
        split_tf32(x[base + i], h, l);
        PK_TRACE_R(x + base + i, 4);
        hi[base + i] = h;
        lo[base + i] = l;
    }
}

// B (K x N, row-major) -> Bt_hi, Bt_lo (N x K, row-major) via 32 x 32 smem tiles, for the
// column band [nb0, nb1) the partition's C tiles read (n0 = nb0 + 32 blockIdx.x)
__global__ void k_split_transp(const float* __restrict__ b, float* __restrict__ bthi, float* __restrict__ btlo,
                               int64_t K, int64_t N, int64_t nb0, int64_t nb1) {
    __shared__ float th[32][33], tl[32][33];
    const int64_t k0 = blockIdx.y * 32, n0 = nb0 + blockIdx.x * 32;
    for (int r = threadIdx.y; r < 32; r += blockDim.y) {
        const int64_t k = k0 + r, n = n0 + threadIdx.x;
        float h = 0.f, l = 0.f;
        if (k < K && n < nb1) {
            split_tf32(b[k * N + n], h, l);
            PK_TRACE_R(b + k * N + n, 4);
        }
        th[r][threadIdx.x] = h;
        tl[r][threadIdx.x] = l;
    }
    __syncthreads();
    for (int r = threadIdx.y; r < 32; r += blockDim.y) {
        const int64_t n = n0 + r, k = k0 + threadIdx.x;
        if (k < K && n < nb1) {
            bthi[n * K + k] = th[threadIdx.x][r];
            btlo[n * K + k] = tl[threadIdx.x][r];
        }
    }
}

// ---------------------------------------------------------------- tcgen05 helpers
__device__ __forceinline__ uint64_t umma_desc_k_sw64(uint32_t smem_addr) {
    // K-major, SWIZZLE_64B canonical layout: rows of 64 B, 8-row atoms of 512 B.
    uint64_t d = 0;
    d |= (uint64_t)((smem_addr >> 4) & 0x3FFFu);        // start address
    d |= (uint64_t)1u << 16;                            // LBO (unused for swizzled K-major) = 1
    d |= (uint64_t)(512u >> 4) << 32;                   // SBO = 512 B between 8-row groups
    d |= (uint64_t)1u << 46;                            // version = 1 (sm_100)
    d |= (uint64_t)4u << 61;                            // layout = SWIZZLE_64B
    return d;
}

// instruction descriptor: kind::tf32, D = F32, A = B = TF32, both K-major, M = 128, N = 256
__host__ __device__ constexpr uint32_t idesc_tf32(int m, int n) {
    return (1u << 4)                   // c_format = F32
           | (2u << 7)                 // a_format = TF32
           | (2u << 10)                // b_format = TF32
           | ((uint32_t)(n >> 3) << 17)
           | ((uint32_t)(m >> 4) << 24);
}

__device__ __forceinline__ void umma_tf32(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                          uint32_t accumulate) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_d),
        "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate));
}

__device__ __forceinline__ void umma_commit(uint64_t* bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                     ptx::smem_u32(bar))
                 : "memory");
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

__device__ __forceinline__ void tmem_ld32(uint32_t taddr, float (&v)[32]) {
    uint32_t r[32];
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
        "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
          "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
          "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
          "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
        : "r"(taddr));
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
    for (int i = 0; i < 32; ++i) v[i] = __uint_as_float(r[i]);
}

// ---------------------------------------------------------------- the GEMM
__global__ void __launch_bounds__(kThreads, 1)
    k_sgemm_tf32x3(const __grid_constant__ CUtensorMap tm_ahi, const __grid_constant__ CUtensorMap tm_alo,
                   const __grid_constant__ CUtensorMap tm_bhi, const __grid_constant__ CUtensorMap tm_blo,
                   float* __restrict__ C, int64_t M, int64_t N, int64_t K, pk_partition part) {
    extern __shared__ __align__(1024) unsigned char smem_raw[];
    unsigned char* smem = (unsigned char*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
    uint64_t* full = reinterpret_cast<uint64_t*>(smem + (size_t)STAGES * STAGE_BYTES);
    uint64_t* empty = full + STAGES;
    uint64_t* acc_full = empty + STAGES;   // [2]: chunk finished in accumulator a
    uint64_t* acc_empty = acc_full + 2;    // [2]: accumulator a drained by the epilogue
    uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(acc_empty + 2);

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    // Grouped rasterisation: the CTAs running at the same time cover kGroup tile
    // rows x (wave / kGroup) tile columns, so each B panel k-slice is read from
    // HBM once per kGroup rows (not once per row) and each A slice once per wave.
    // The CTA -> logical tile map is a bijection onto the partition's box, so the
    // launch still computes exactly the blocks [min, max) (Eq. 8-10).
    constexpr int kGroup = 16;
    const int64_t gx = part.max[0] - part.min[0], gy = part.max[1] - part.min[1];
    const int64_t L = (int64_t)blockIdx.y * gridDim.x + blockIdx.x;
    const int64_t grp = L / (kGroup * gx);
    const int64_t row0 = grp * kGroup;
    const int64_t gsz = (gy - row0) < kGroup ? (gy - row0) : kGroup;
    const int64_t in = L - grp * kGroup * gx;
    const int64_t m0 = (int64_t)(part.min[1] + row0 + in % gsz) * BM;  // Eq. 8
    const int64_t n0 = (int64_t)(part.min[0] + in / gsz) * BN;
    const int nk = (int)((K + BK - 1) / BK);

    if (warp == 0 && lane == 0) {
        for (int s = 0; s < STAGES; ++s) {
            ptx::mbar_init(&full[s], 1);
            ptx::mbar_init(&empty[s], 1);
        }
        for (int a = 0; a < 2; ++a) {
            ptx::mbar_init(&acc_full[a], 1);
            ptx::mbar_init(&acc_empty[a], 8);   // one arrival per epilogue warp
        }
        ptx::fence_mbar_init();
        asm volatile("prefetch.tensormap [%0];" ::"l"(&tm_ahi) : "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"(&tm_alo) : "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"(&tm_bhi) : "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"(&tm_blo) : "memory");
    }
    if (warp == 2) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                         ptx::smem_u32(tmem_holder)),
                     "r"(TMEM_COLS)
                     : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tmem = *tmem_holder;

    if (warp == 0 && lane == 0) {
        // ---------------- TMA producer
        for (int kb = 0; kb < nk; ++kb) {
            const int s = kb % STAGES;
            const uint32_t ph = (kb / STAGES) & 1u;
            ptx::mbar_wait(&empty[s], ph ^ 1u);
            unsigned char* st = smem + (size_t)s * STAGE_BYTES;
            ptx::mbar_arrive_expect_tx(&full[s], STAGE_BYTES);
            const int32_t kc = kb * BK;
            tma_2d(st, &tm_ahi, kc, (int32_t)m0, &full[s]);
            tma_2d(st + A_TILE, &tm_alo, kc, (int32_t)m0, &full[s]);
            tma_2d(st + 2 * A_TILE, &tm_bhi, kc, (int32_t)n0, &full[s]);
            tma_2d(st + 2 * A_TILE + B_TILE, &tm_blo, kc, (int32_t)n0, &full[s]);
        }
    } else if (warp == 1 && lane == 0) {
        // ---------------- MMA issuer (single thread)
        constexpr uint32_t idesc = idesc_tf32(BM, BN);
        for (int kb = 0; kb < nk; ++kb) {
            const int s = kb % STAGES;
            const uint32_t ph = (kb / STAGES) & 1u;
            const int chunk = kb / KC_BLOCKS, a = chunk & 1;
            const bool first = kb % KC_BLOCKS == 0;
            if (first && chunk >= 2) {  // accumulator a still holds chunk-2 until the epilogue drained it
                ptx::mbar_wait(&acc_empty[a], (uint32_t)((chunk / 2 - 1) & 1));
            }
            ptx::mbar_wait(&full[s], ph);
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
            const uint32_t st = ptx::smem_u32(smem + (size_t)s * STAGE_BYTES);
            const uint32_t acc = tmem + (uint32_t)(a * BN);
#pragma unroll
            for (int kk = 0; kk < BK / 8; ++kk) {
                const uint32_t ko = kk * 32;  // 8 TF32 = 32 B along K inside the 64-B swizzle row
                const uint64_t ahi = umma_desc_k_sw64(st + ko), alo = umma_desc_k_sw64(st + A_TILE + ko);
                const uint64_t bhi = umma_desc_k_sw64(st + 2 * A_TILE + ko);
                const uint64_t blo = umma_desc_k_sw64(st + 2 * A_TILE + B_TILE + ko);
                umma_tf32(acc, ahi, bhi, idesc, (first && kk == 0) ? 0u : 1u);
                umma_tf32(acc, ahi, blo, idesc, 1u);
                umma_tf32(acc, alo, bhi, idesc, 1u);
            }
            umma_commit(&empty[s]);  // frees the smem stage when these MMAs complete
            if (kb % KC_BLOCKS == KC_BLOCKS - 1 || kb == nk - 1) umma_commit(&acc_full[a]);
        }
    } else if (warp >= 4) {
        // ---------------- epilogue: chunk accumulators -> FP32 running sums -> global
        const int q = warp & 3;                     // TMEM lane quarter of this warp
        const int half = (warp - 4) >> 2;           // column half of the tile
        const int64_t row = m0 + 32 * q + lane;
        const int nchunks = (nk + KC_BLOCKS - 1) / KC_BLOCKS;
        float sum[EPI_COLS];
#pragma unroll
        for (int i = 0; i < EPI_COLS; ++i) sum[i] = 0.f;
        for (int chunk = 0; chunk < nchunks; ++chunk) {
            const int a = chunk & 1;
            ptx::mbar_wait(&acc_full[a], (uint32_t)((chunk / 2) & 1));
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
#pragma unroll
            for (int c = 0; c < EPI_COLS; c += 16) {
                float v[16];
                tmem_ld16(tmem + ((uint32_t)(32 * q) << 16) + (uint32_t)(a * BN + half * EPI_COLS + c), v);
#pragma unroll
                for (int i = 0; i < 16; ++i) sum[c + i] += v[i];   // round-to-nearest FP32 add
            }
            asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
            __syncwarp();
            if (lane == 0) ptx::mbar_arrive(&acc_empty[a]);
        }
        if (row < M) {
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
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (warp == 2) {
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(TMEM_COLS) : "memory");
    }
}

// ---------------------------------------------------------------- host side
using EncodeTiled = CUresult (*)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                 const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                 CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

EncodeTiled get_encode() {
    static EncodeTiled fn = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
        void* p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = (EncodeTiled)p;
    });
    return fn;
}

bool make_map(CUtensorMap* m, const float* base, int64_t rows, int64_t cols, int box_rows) {
    EncodeTiled enc = get_encode();
    if (!enc) return false;
    cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)rows};
    cuuint64_t strides[1] = {(cuuint64_t)cols * 4};
    cuuint32_t box[2] = {BK, (cuuint32_t)box_rows};
    cuuint32_t estr[2] = {1, 1};
    return enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, (void*)base, dims, strides, box, estr,
               CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_64B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

struct Scratch {
    float *ahi = nullptr, *alo = nullptr, *bhi = nullptr, *blo = nullptr;
};

// hi/lo operand scratch: context-owned per partition (grow-only, see context_scratch)
cudaError_t get_scratch(const LaunchInfo& li, size_t a_elems, size_t b_elems, Scratch* sc) {
    cudaError_t e = cudaSuccess;
    if (!(sc->ahi = (float*)context_scratch(li, 0, a_elems * 4, &e))) return e;
    if (!(sc->alo = (float*)context_scratch(li, 1, a_elems * 4, &e))) return e;
    if (!(sc->bhi = (float*)context_scratch(li, 2, b_elems * 4, &e))) return e;
    if (!(sc->blo = (float*)context_scratch(li, 3, b_elems * 4, &e))) return e;
    return cudaSuccess;
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

cudaError_t launch_sgemm(const LaunchInfo& li) {
    if (li.nscalars < 3) return cudaErrorInvalidValue;
    int64_t M = li.scalars[0], N = li.scalars[1], K = li.scalars[2];
    if (M < 1 || N < 1 || K < 4 || K % 4) return cudaErrorInvalidValue;  // TMA row stride: 16-B multiple
    const float* A = (const float*)li.inst[0];
    const float* B = (const float*)li.inst[1];
    float* C = (float*)li.inst[2];
    Scratch scr;
    Scratch* sc = &scr;
    cudaError_t e = get_scratch(li, (size_t)M * K, (size_t)N * K, &scr);
    if (e != cudaSuccess) return e;
    // 1. split this partition's A rows; 2. split + transpose all of B
    const int64_t r0 = (int64_t)li.part.min[1] * BM, r1 = std::min<int64_t>((int64_t)li.part.max[1] * BM, M);
    if (r1 > r0) {
        k_split_rows<<<1184, 256, 0, li.stream>>>(A, sc->ahi, sc->alo, r0, r1, K);
        if ((e = cudaGetLastError()) != cudaSuccess) return e;
    }
    // only the B column band of this partition's C tiles (tile partitions split N too)
    const int64_t nb0 = (int64_t)li.part.min[0] * BN, nb1 = std::min<int64_t>((int64_t)li.part.max[0] * BN, N);
    dim3 tg((unsigned)((nb1 - nb0 + 31) / 32), (unsigned)((K + 31) / 32));
    if (nb1 > nb0) k_split_transp<<<tg, dim3(32, 8), 0, li.stream>>>(B, sc->bhi, sc->blo, K, N, nb0, nb1);
    if ((e = cudaGetLastError()) != cudaSuccess) return e;
    // 3. tensor-core GEMM over the partition's C tiles
    CUtensorMap tm[4];
    if (!make_map(&tm[0], sc->ahi, M, K, BM) || !make_map(&tm[1], sc->alo, M, K, BM) ||
        !make_map(&tm[2], sc->bhi, N, K, BN) || !make_map(&tm[3], sc->blo, N, K, BN))
        return cudaErrorInvalidValue;
    KernelDevInfo kd;   // per device: the opt-in above 48 KB is a (function, device) attribute
    if ((e = prepare_kernel((const void*)k_sgemm_tf32x3, li.device, SMEM_BYTES, kThreads, &kd)) != cudaSuccess)
        return e;
    void* argv[] = {&tm[0], &tm[1], &tm[2], &tm[3], &C, &M, &N, &K, (void*)&li.part};
    return cudaLaunchKernel((const void*)k_sgemm_tf32x3, li.grid, dim3(kThreads), argv, SMEM_BYTES, li.stream);
}

}  // namespace

const Builtin kBuiltinSgemm = {"sgemm_tf32x3", (const void*)k_sgemm_tf32x3, 6,
                               {PK_ARG_BUFFER, PK_ARG_BUFFER, PK_ARG_BUFFER, PK_ARG_SCALAR, PK_ARG_SCALAR,
                                PK_ARG_SCALAR},
                               -1, describe_sgemm, launch_sgemm};

}  // namespace pk
