// racecheck_bulk_ring.cu -- minimal reproducer for the racecheck reports on the Hotspot rings
// (VERDICT r1 #8).  One producer thread fills a 4-slot shared-memory ring with bulk copies
// (global -> shared, completion counted on a per-slot "full" mbarrier); one consumer warp waits
// on "full", reads the slot, and releases it on a per-slot "empty" mbarrier that the producer
// waits on before refilling.  This is the canonical TMA pipeline: every read of a slot happens
// after the phase of its full barrier that the copy completes, every refill after the empty
// phase the readers complete.  The result is checked on the host (sum of all elements).
//   mode 0: 1-D cp.async.bulk (non-tensor), as the Hotspot rings use
//   mode 1: cp.async.bulk.tensor through a tensor map (2-D: 4 rows of 256 floats per slot), as the
//           Heat rings use
// Run each under compute-sanitizer --tool racecheck.
//   nvcc -gencode arch=compute_100a,code=sm_100a -o rr scripts/racecheck_bulk_ring.cu -lcuda && ./rr 0 && ./rr 1
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>
#include <vector>

constexpr int kSlots = 4, kSlotFloats = 1024, kRows = 64;

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t n) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(n) : "memory");
}
__device__ __forceinline__ void mbar_expect(uint64_t* b, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* b) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t par) {
    asm volatile(
        "{\n\t.reg .pred p;\nW:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t@!p bra W;\n}" ::"r"(
            smem_u32(b)),
        "r"(par)
        : "memory");
}

__global__ void ring(const float* __restrict__ src, float* out, const __grid_constant__ CUtensorMap tm, int mode) {
    __shared__ __align__(128) float buf[kSlots][kSlotFloats];
    __shared__ uint64_t full[kSlots], empty[kSlots];
    if (threadIdx.x == 0) {
        for (int s = 0; s < kSlots; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], 1);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (threadIdx.x == 32) {  // producer (warp 1, lane 0)
        for (int r = 0; r < kRows; ++r) {
            const int s = r % kSlots;
            mbar_wait(&empty[s], ((r / kSlots) & 1) ^ 1);
            mbar_expect(&full[s], kSlotFloats * 4);
            if (mode == 0)
                asm volatile(
                    "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                        smem_u32(buf[s])),
                    "l"(src + (size_t)r * kSlotFloats), "r"(kSlotFloats * 4), "r"(smem_u32(&full[s]))
                    : "memory");
            else
                asm volatile(
                    "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, "
                    "%3}], [%4];" ::"r"(smem_u32(buf[s])),
                    "l"(&tm), "r"(0), "r"(r * 4), "r"(smem_u32(&full[s]))
                    : "memory");
        }
    } else if (threadIdx.x < 32) {  // consumer warp 0
        float acc = 0.f;
        for (int r = 0; r < kRows; ++r) {
            const int s = r % kSlots;
            mbar_wait(&full[s], (r / kSlots) & 1);
            for (int i = threadIdx.x; i < kSlotFloats; i += 32) acc += buf[s][i];
            __syncwarp();
            if (threadIdx.x == 0) mbar_arrive(&empty[s]);
        }
        atomicAdd(out, acc);
    }
}

int main(int argc, char** argv) {
    const int mode = argc > 1 ? atoi(argv[1]) : 0;
    const size_t n = (size_t)kRows * kSlotFloats;
    std::vector<float> h(n);
    double ref = 0;
    for (size_t i = 0; i < n; ++i) {
        h[i] = (float)(i % 7);
        ref += h[i];
    }
    float *d, *out;
    cudaMalloc(&d, n * 4);
    cudaMalloc(&out, 4);
    cudaMemcpy(d, h.data(), n * 4, cudaMemcpyHostToDevice);
    cudaMemset(out, 0, 4);
    CUtensorMap tm{};
    // the same data as rows of 256 floats: one 256 x 4 box fills one 1024-float slot
    cuuint64_t dims2[2] = {256, n / 256};
    cuuint64_t str2[1] = {256 * 4};
    cuuint32_t box2[2] = {256, 4};
    cuuint32_t es2[2] = {1, 1};
    CUresult cr = cuTensorMapEncodeTiled(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, d, dims2, str2, box2, es2,
                                         CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                                         CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (mode == 1 && cr != CUDA_SUCCESS) {
        printf("tensor map encode failed %d\n", (int)cr);
        return 1;
    }
    ring<<<1, 64>>>(d, out, tm, mode);
    float got = 0;
    cudaMemcpy(&got, out, 4, cudaMemcpyDeviceToHost);
    printf("mode %d (%s): sum %.0f, expected %.0f, %s (%s)\n", mode, mode ? "tensor bulk copy" : "1-D bulk copy", got,
           ref, got == (float)ref ? "correct" : "WRONG", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
