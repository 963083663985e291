// builtins.h -- registry of the library's hand-written sm_100a kernels.
#pragma once

#include <cuda_runtime.h>

#include "pk_api.h"

namespace pk {

// Halo push (PK_MODE_PUSH): bytes [lo[i], hi[i]) of the kernel's push-capable output
// instance are ALSO stored at dst[i] + offset (another partition's instance of the same
// buffer, same layout; a peer GPU's memory over NVLink or an IPC mapping) by the kernel
// that produces them.  Passed to the kernel by value.
constexpr int kMaxPush = 16;
struct PushList {
    int32_t n;
    int32_t pad;
    uint64_t lo[kMaxPush], hi[kMaxPush];
    uint64_t dst[kMaxPush];
};

// Streamed operand (Builtin::stream_arg): the copies that make that argument valid on
// the partition run on a side stream WHILE the kernel runs -- the transfer overlapped
// with the computation it feeds (the B operand broadcast of C4).  The copy
// of granule g (bytes [g * granule, (g + 1) * granule) of the instance) stores 1 into
// flags[g] when it has landed; bit g of `wait` tells the kernel to poll flags[g]
// (acquire) before it reads that granule.  wait == 0: nothing is in flight.
constexpr int kMaxGranules = 64;
struct Arrival {
    const uint32_t* flags;   // device words [kMaxGranules] of this partition
    uint64_t wait;
    uint64_t granule;        // bytes
};

// Everything a launcher needs for one partition (Fig. 4 lines 10-19).
struct LaunchInfo {
    const void* fn;
    dim3 grid;                 // partition grid: max - min (Eq. 10)
    dim3 block;
    size_t smem;
    cudaStream_t stream;
    int device;
    void* const* inst;         // [nargs] instance pointers (nullptr for scalars)
    const void* const* args;   // [nargs] user arg pointers (scalar values)
    const int64_t* scalars;
    int nscalars;
    pk_partition part;
    const PushList* push = nullptr;  // halo push of the push-capable output (nullptr / n = 0: none)
    pk_ctx ctx = nullptr;            // owning context and partition index (context_scratch)
    int part_index = -1;
    Arrival arrival = {nullptr, 0, 0};  // streamed operand (Builtin::stream_arg), if any
};

// Device scratch of a launcher (e.g. N-body partial sums), owned by the context per
// (partition, slot) on the partition's device.  Grow-only: a smaller request reuses the
// block; a larger one allocates a new block and RETIRES the old one, which stays
// allocated until pk_finalize because a memoised graph may still replay into it.
// Returns nullptr on failure (*err set).
void* context_scratch(const LaunchInfo& li, int slot, size_t bytes, cudaError_t* err);
constexpr int kScratchSlots = 4;
using LauncherFn = cudaError_t (*)(const LaunchInfo&);

struct Builtin {
    const char* name;
    const void* fn;
    int nargs;
    int32_t kinds[PK_MAX_ARGS];
    int32_t partition_dim;
    // declares the kernel's access taps through pk_declare_affine_access
    int (*describe)(pk_ctx, pk_kernel);
    LauncherFn launcher;       // nullptr = generic cudaLaunchKernel
    int32_t push_arg = -1;     // output buffer argument the kernel can halo-push (LaunchInfo::push), -1: none
    // input argument the kernel can consume while its copies are in flight (LaunchInfo::arrival),
    // -1: none; stream_granule(scalars) = the granule in bytes (<= kMaxGranules granules per buffer)
    int32_t stream_arg = -1;
    uint64_t (*stream_granule)(const int64_t* scalars, int nscalars) = nullptr;
};

const Builtin* find_builtin(const char* name);
const Builtin* find_builtin_by_fn(const void* fn);
LauncherFn find_builtin_launcher(const void* fn);
int32_t find_builtin_push_arg(const void* fn);

// Per-kernel-file registration (defined in kernels/*.cu)
extern const Builtin kBuiltinJacobi2d;
extern const Builtin kBuiltinJacobi2dTb;     // jacobi2d_tb (K sweeps per launch, ghost zones)
extern const Builtin kBuiltinHotspot2d;     // hotspot2d_regs (register window)
extern const Builtin kBuiltinHotspot2dTma;  // hotspot2d (TMA bulk ring, default)
extern const Builtin kBuiltinHotspot2dTb2;  // hotspot2d_tb2 (two sweeps per launch)
extern const Builtin kBuiltinHotspot2dTbk;  // hotspot2d_tbk (K = 2..4 sweeps per launch, scalar 3)
extern const Builtin kBuiltinHeat3d;
extern const Builtin kBuiltinHeat3dTma;      // heat3d (TMA plane ring, default); kBuiltinHeat3d = heat3d_regs
extern const Builtin kBuiltinHeat3dTb2;      // heat3d_tb2 (two sweeps per launch)
extern const Builtin kBuiltinHeat3dTb3;      // heat3d_tb3 (three sweeps per launch)
extern const Builtin kBuiltinNbody;
extern const Builtin kBuiltinSgemm;          // sgemm_tf32x3 (tcgen05 3xTF32)

// Strided halo copy on the destination's SMs (kernels/halo_copy.cu): nslab slabs
// (stride `slice`) of `rows` pieces (stride `pitch`) of `len` bytes, dst <- src.
cudaError_t launch_strided_copy(char* dst, const char* src, uint64_t len, uint64_t pitch, uint64_t rows,
                                uint64_t slice, uint64_t nslab, int sm_count, cudaStream_t stream);

// Epoch flags of the peer-memory SPMD transport on the SMs (fallback of the stream
// memory operations): wait until *flags[i] >= targets[i] for all i; store *flag = v.
cudaError_t launch_flag_wait(const uint64_t* const* flags, const uint64_t* targets, int n, cudaStream_t stream);
cudaError_t launch_flag_write(uint64_t* flag, uint64_t v, cudaStream_t stream);

// Descriptor helpers used by the kernel files' describe() functions.
inline pk_expr E(int64_t c0) {
    pk_expr e{};
    e.c0 = c0;
    return e;
}
inline pk_expr S(int s, int64_t coef = 1, int64_t c0 = 0) {  // coef * scalars[s] + c0
    pk_expr e{};
    e.c0 = c0;
    e.c_scalar[s] = coef;
    return e;
}
inline pk_expr BD(int w, int64_t coef = 1) {  // coef * blockDim[w]
    pk_expr e{};
    e.c_blockdim[w] = coef;
    return e;
}
inline pk_dim_map DimMap(int grid_dim, pk_expr scale, pk_expr extent, pk_expr offset,
                         uint32_t flags, pk_expr glo = E(0), pk_expr ghi = E(0)) {
    pk_dim_map d{};
    d.grid_dim = grid_dim;
    d.flags = flags;
    d.scale = scale;
    d.extent = extent;
    d.offset = offset;
    d.guard_lo = glo;
    d.guard_hi = ghi;
    return d;
}

}  // namespace pk
