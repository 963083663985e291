// ce_probe.cu -- which transfer operations make progress while every SM is held by a
// kernel that spins?  (The streamed-operand path overlaps B copies with a GEMM whose CTAs
// poll arrival flags; an operation that needs an SM could then never run: deadlock.)
// The spinners poll a flag in mapped pinned host memory that only the HOST sets, after
// it has watched (for up to 1 s) whether the operation under test completed.  Also: are
// stream memory operations capturable into a CUDA graph?
//   nvcc -gencode arch=compute_100a,code=sm_100a -o scripts/ce_probe.bin scripts/ce_probe.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>

#include <chrono>
#include <cstdio>
#include <thread>

__global__ void spin(const volatile unsigned* release) {
    extern __shared__ unsigned char sm[];  // one CTA per SM: nothing else can be resident
    sm[threadIdx.x] = 0;
    while (*release == 0u) __nanosleep(500);
}

int main() {
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const size_t smem = 200 * 1024;
    cudaFuncSetAttribute(spin, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    unsigned* release;  // mapped pinned host word
    cudaHostAlloc(&release, 4, cudaHostAllocMapped);
    unsigned* release_d;
    cudaHostGetDevicePointer(&release_d, release, 0);
    volatile unsigned* hflag;  // mapped pinned host word written by a stream memory op
    cudaHostAlloc((void**)&hflag, 4, cudaHostAllocMapped);
    unsigned* hflag_d;
    cudaHostGetDevicePointer(&hflag_d, (void*)hflag, 0);
    unsigned* dflag;
    cudaMalloc(&dflag, 4);
    const size_t n = 64 << 20;
    void *a, *b, *h;
    cudaMalloc(&a, n);
    cudaMalloc(&b, n);
    cudaHostAlloc(&h, n, 0);
    cudaStream_t s1, s2;
    cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking);
    cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking);
    const char* names[] = {"cuStreamWriteValue32 to mapped host memory", "cuStreamWriteValue32 to device memory",
                           "cudaMemcpyAsync D2D (same device) 64 MB", "cudaMemcpyAsync D2H 64 MB (pinned)",
                           "cudaMemcpyAsync H2D 64 MB (pinned)", "cudaMemcpy2DAsync D2D 64 MB"};
    for (int mode = 0; mode < 6; ++mode) {
        *release = 0;
        *hflag = 0;
        cudaDeviceSynchronize();
        spin<<<sms, 128, smem, s1>>>(release_d);
        std::this_thread::sleep_for(std::chrono::milliseconds(50));  // let the spinners occupy every SM
        cudaEvent_t done;
        cudaEventCreateWithFlags(&done, cudaEventDisableTiming);
        switch (mode) {
            case 0: cuStreamWriteValue32((CUstream)s2, (CUdeviceptr)hflag_d, 1u, CU_STREAM_WRITE_VALUE_DEFAULT); break;
            case 1: cuStreamWriteValue32((CUstream)s2, (CUdeviceptr)dflag, 1u, CU_STREAM_WRITE_VALUE_DEFAULT); break;
            case 2: cudaMemcpyAsync(b, a, n, cudaMemcpyDeviceToDevice, s2); break;
            case 3: cudaMemcpyAsync(h, a, n, cudaMemcpyDeviceToHost, s2); break;
            case 4: cudaMemcpyAsync(b, h, n, cudaMemcpyHostToDevice, s2); break;
            case 5: cudaMemcpy2DAsync(b, 4096, a, 4096, 4096, n / 4096, cudaMemcpyDeviceToDevice, s2); break;
        }
        cudaEventRecord(done, s2);
        const auto t0 = std::chrono::steady_clock::now();
        bool ok = false;
        double ms = 0;
        while ((ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count()) < 1000) {
            if (mode == 0 ? *hflag == 1u : cudaEventQuery(done) == cudaSuccess) { ok = true; break; }
        }
        *release = 1;  // let the spinners go
        cudaDeviceSynchronize();
        printf("%-46s while %d CTAs hold every SM: %s (%.2f ms)\n", names[mode], sms,
               ok ? "COMPLETED" : "blocked until the SMs were released", ms);
        cudaEventDestroy(done);
    }
    // stream memory operations inside a stream capture
    cudaGraph_t g = nullptr;
    cudaStreamBeginCapture(s2, cudaStreamCaptureModeRelaxed);
    CUresult r1 = cuStreamWriteValue32((CUstream)s2, (CUdeviceptr)dflag, 0u, CU_STREAM_WRITE_VALUE_DEFAULT);
    cudaMemcpyAsync(b, a, 1 << 20, cudaMemcpyDeviceToDevice, s2);
    CUresult r2 = cuStreamWriteValue32((CUstream)s2, (CUdeviceptr)dflag, 7u, CU_STREAM_WRITE_VALUE_DEFAULT);
    cudaError_t ce = cudaStreamEndCapture(s2, &g);
    cudaGraphExec_t ex = nullptr;
    cudaError_t ie = g ? cudaGraphInstantiate(&ex, g, 0) : cudaErrorUnknown;
    unsigned v = 0;
    if (ex) {
        cudaMemset(dflag, 0, 4);
        cudaGraphLaunch(ex, s2);
        cudaStreamSynchronize(s2);
        cudaMemcpy(&v, dflag, 4, cudaMemcpyDeviceToHost);
    }
    printf("capture of cuStreamWriteValue32: rc %d/%d, end %s, instantiate %s, flag after replay = %u\n", (int)r1,
           (int)r2, cudaGetErrorString(ce), cudaGetErrorString(ie), v);
    return 0;
}
