// runtime.cu -- the C-ABI of include/pk_api.h: virtual buffers, kernel model
// records, the Fig. 4 launch replacement (partition -> regions -> stale plan ->
// transfers -> partitioned launches -> tracker update), D2H/H2D translation.
//
// Process model: one host process drives every partition (the paper's single
// rewritten host program, §8.4).  A partition is a virtual device:
// several may share one physical GPU (each with its own full-size instance), so
// P-way partitioning and its transfers are exercised on any GPU count.
//
// Ordering replaces the global barrier of Fig. 4 line 8 by a
// cross-stream event DAG per (buffer, partition) instance:
//   RAW  a copy out of (b,q) waits for the last writer of (b,q);
//   WAR  any write into (b,p) -- kernel or incoming copy -- waits for the copies
//        that read (b,p) since its last write ("readers").
// PK_MODE_GLOBAL_BARRIER restores the literal host-side barrier.
#include <cuda.h>
#include <cuda_runtime.h>
#include <dlfcn.h>

#include <algorithm>
#include <array>
#include <chrono>
#include <ctime>
#include <cstddef>
#include <cstdio>
#include <cstring>
#include <memory>
#include <string>
#include <unordered_map>
#include <vector>

#include <nvtx3/nvToolsExt.h>

#include "../core/host_core.h"
#include "../kernels/trace.cuh"
#include "builtins.h"
#include "pk_api.h"

using namespace pk;

// ---- access recording (libpk_trace.so only; kernels/trace.cuh) ----
#ifdef PK_TRACE_ACCESS
#include <mutex>
__device__ pk::trace::Table g_pk_trace;
namespace {
struct TraceInst {
    const void* base;
    uint64_t bytes;
    uint32_t* bits[2];
};
std::mutex g_trace_mu;
std::vector<TraceInst> g_trace;  // every registered instance of every context (one device)
cudaError_t trace_upload() {
    pk::trace::Table t{};
    t.n = (int32_t)g_trace.size();
    for (size_t i = 0; i < g_trace.size(); ++i) {
        t.base[i] = (uint64_t)(uintptr_t)g_trace[i].base;
        t.bytes[i] = g_trace[i].bytes;
        t.bits[i][0] = g_trace[i].bits[0];
        t.bits[i][1] = g_trace[i].bits[1];
    }
    cudaError_t e = cudaDeviceSynchronize();
    if (e == cudaSuccess) e = cudaMemcpyToSymbol(g_pk_trace, &t, sizeof t);
    return e;
}
cudaError_t trace_add(const void* base, uint64_t bytes) {
    std::lock_guard<std::mutex> g(g_trace_mu);
    if (g_trace.size() >= (size_t)pk::trace::kMaxInst) return cudaErrorMemoryAllocation;
    TraceInst ti{base, bytes, {nullptr, nullptr}};
    const size_t wb = ((bytes / 4 + 31) / 32) * 4;
    for (int k = 0; k < 2; ++k) {
        cudaError_t e = cudaMalloc(&ti.bits[k], wb ? wb : 4);
        if (e == cudaSuccess) e = cudaMemset(ti.bits[k], 0, wb ? wb : 4);
        if (e != cudaSuccess) return e;
    }
    g_trace.push_back(ti);
    return trace_upload();
}
void trace_remove(const void* base) {
    std::lock_guard<std::mutex> g(g_trace_mu);
    for (size_t i = 0; i < g_trace.size(); ++i)
        if (g_trace[i].base == base) {
            cudaFree(g_trace[i].bits[0]);
            cudaFree(g_trace[i].bits[1]);
            g_trace.erase(g_trace.begin() + i);
            trace_upload();
            return;
        }
}
}  // namespace
#endif

namespace {

thread_local std::string g_err;

int fail(int code, const std::string& msg) {
    g_err = msg;
    return code;
}
int fail(const Status& s) { return fail(s.code, s.msg); }

#define PK_CUDA(call)                                                                   \
    do {                                                                                \
        cudaError_t e_ = (call);                                                        \
        if (e_ != cudaSuccess)                                                          \
            return fail(PK_ERR_CUDA, std::string(#call) + ": " + cudaGetErrorName(e_) + \
                                         " (" + cudaGetErrorString(e_) + ")");          \
    } while (0)

// NVTX ranges per phase of the launch replacement (SURVEY.md §5 tracing): visible in
// Nsight Systems / ncu --nvtx; NVTX v3 is header-only and costs a branch without a tool.
struct NvtxPhase {
    bool open = false;
    explicit NvtxPhase(const char* name) { next(name); }
    void next(const char* name) {
        if (open) nvtxRangePop();
        nvtxRangePushA(name);
        open = true;
    }
    ~NvtxPhase() {
        if (open) nvtxRangePop();
    }
};

uint64_t thread_cpu_ns() {
    timespec ts;
    clock_gettime(CLOCK_THREAD_CPUTIME_ID, &ts);
    return (uint64_t)ts.tv_sec * 1000000000ull + (uint64_t)ts.tv_nsec;
}

uint64_t now_ns() {
    return (uint64_t)std::chrono::duration_cast<std::chrono::nanoseconds>(
               std::chrono::steady_clock::now().time_since_epoch())
        .count();
}

enum : uint8_t { W_NONE = 0, W_KERNEL = 1, W_COPY = 2 };

// ---- NCCL, loaded at run time (only multi-process SPMD contexts need it) ----
struct NcclId {
    char internal[128];  // layout of ncclUniqueId
};
struct NcclApi {
    bool ok = false;
    int (*GetUniqueId)(NcclId*) = nullptr;
    int (*CommInitRank)(void** comm, int nranks, NcclId id, int rank) = nullptr;
    int (*CommInitAll)(void** comms, int ndev, const int* devlist) = nullptr;  // optional (one process)
    int (*CommDestroy)(void* comm) = nullptr;
    int (*Send)(const void*, size_t, int, int, void*, cudaStream_t) = nullptr;
    int (*Recv)(void*, size_t, int, int, void*, cudaStream_t) = nullptr;
    int (*AllGather)(const void*, void*, size_t, int, void*, cudaStream_t) = nullptr;
    int (*GroupStart)() = nullptr;
    int (*GroupEnd)() = nullptr;
    const char* (*GetErrorString)(int) = nullptr;
};
constexpr int kNcclUint8 = 1;  // ncclUint8

NcclApi load_nccl();
const NcclApi& nccl() {  // process-wide (not device-scoped); thread-safe static initialisation
    static const NcclApi api = load_nccl();
    return api;
}
NcclApi load_nccl() {
    NcclApi api;
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) {
        const char* p = getenv("PK_NCCL_LIB");
        if (p) h = dlopen(p, RTLD_NOW | RTLD_GLOBAL);
    }
    if (!h) return api;
    api.GetUniqueId = (int (*)(NcclId*))dlsym(h, "ncclGetUniqueId");
    api.CommInitRank = (int (*)(void**, int, NcclId, int))dlsym(h, "ncclCommInitRank");
    api.CommDestroy = (int (*)(void*))dlsym(h, "ncclCommDestroy");
    api.CommInitAll = (int (*)(void**, int, const int*))dlsym(h, "ncclCommInitAll");
    api.Send = (int (*)(const void*, size_t, int, int, void*, cudaStream_t))dlsym(h, "ncclSend");
    api.Recv = (int (*)(void*, size_t, int, int, void*, cudaStream_t))dlsym(h, "ncclRecv");
    api.AllGather = (int (*)(const void*, void*, size_t, int, void*, cudaStream_t))dlsym(h, "ncclAllGather");
    api.GroupStart = (int (*)())dlsym(h, "ncclGroupStart");
    api.GroupEnd = (int (*)())dlsym(h, "ncclGroupEnd");
    api.GetErrorString = (const char* (*)(int))dlsym(h, "ncclGetErrorString");
    api.ok = api.GetUniqueId && api.CommInitRank && api.CommDestroy && api.Send && api.Recv && api.AllGather &&
             api.GroupStart &&
             api.GroupEnd && api.GetErrorString;
    return api;
}

struct Buffer {
    bool alive = false;
    int ndim = 0;
    int64_t shape[PK_MAX_DIMS] = {0, 0, 0, 0};
    int eb = 0;
    uint64_t bytes = 0;
    bool owned = false;
    std::vector<void*> inst;
    Tracker tracker;
    std::vector<uint8_t> last_writer;  // per partition
    std::vector<uint64_t> readers;     // per partition: mask of partitions whose ev_copy must precede a write
    // SPMD over peer memory (pk_init_spmd_ipc): replicated epoch bookkeeping
    std::vector<uint64_t> ep_mod;      // [q]: epoch of the last device write of (b,q); 0 = settled
    std::vector<uint8_t> ep_kind;      // [q]: W_KERNEL / W_COPY (which flag word signals it)
    std::vector<uint64_t> ep_read;     // [q*P + r]: epoch at which r last copied out of (b,q); 0 = none
    std::vector<void*> ipc_base;       // [q]: mapped base of a remote instance (cudaIpcCloseMemHandle)
    // halo push (PK_MODE_PUSH)
    std::vector<RangeList> last_read;  // [p]: bytes p read in the last launch that read this buffer (prediction)
    std::vector<uint64_t> pushers;     // [p]: partitions whose kernels pushed into (b,p) (event RAW, 1 process)
    std::vector<uint64_t> ep_push;     // [p*P+q]: epoch of q's last push into (b,p) (peer-memory SPMD)
    std::vector<uint64_t> ep_kread;    // [p]: epoch of p's last kernel that read b (peer-memory SPMD, push WAR)
};

struct Tap {
    int arg;
    int mode;
    pk_affine_access acc;
};

struct Kernel {
    std::string name;
    const void* fn = nullptr;
    int nargs = 0;
    int32_t kinds[PK_MAX_ARGS] = {};
    int32_t partition_dim = -1;
    int32_t tiles[3] = {0, 0, 0};  // (tx, ty, tz) tile partition; 0 = 1-D split
    std::vector<Tap> taps;
    LauncherFn launcher = nullptr;
    int32_t push_arg = -1;  // output buffer argument the kernel can halo-push (builtin capability)
    int32_t stream_arg = -1;  // input argument consumed while its copies are in flight (builtin capability)
    uint64_t (*stream_granule)(const int64_t*, int) = nullptr;
    uint64_t version = 0;  // bumps when taps change (region cache key)
};

struct ArgRegions {
    RangeList r, w;
};
struct Regions {
    bool empty;
    int64_t box[6];
    std::vector<ArgRegions> args;  // [nargs]
};

struct CopyOp {
    int64_t buf;
    int src, dst;
    uint64_t b, e;
};

struct TimedLaunch {
    cudaEvent_t start, stop;
    int part;
    uint64_t launch_id;
    bool graph = false;  // events around a replayed graph launch (whole launch), not one kernel
    int nlaunch = 1;     // partitioned launches inside that graph (pk_launch_sequence)
};

}  // namespace

struct pk_ctx_s {
    int P = 0;
    int rank = 0, world = 1;
    uint32_t init_flags = 0;
    uint32_t mode = 0;
    bool host_only = false;
    std::vector<int> dev, prank;
    std::vector<int> sm_count;  // per partition's device (halo copy kernel grid)
    std::vector<uint8_t> peer;  // [p*P + q]: p's device can address q's instances (same GPU or peer access on)
    bool sm_reach(int p, int q) const { return ipc || peer.empty() || peer[(size_t)p * P + q]; }
    std::vector<cudaStream_t> stream;
    std::vector<cudaEvent_t> ev_kernel, ev_copy;
    std::vector<uint8_t> kernel_recorded;  // [p]: ev_kernel[p] recorded since the hazards were last cleared
    std::vector<Buffer> bufs;
    std::vector<Kernel> kernels;
    pk_stats stats{};
    std::vector<CopyOp> last_plan;                               // built by the eager path
    std::shared_ptr<const std::vector<CopyOp>> replay_plan;       // set by a graph replay
    std::unordered_map<std::string, std::shared_ptr<std::vector<Regions>>> region_cache;
    std::vector<TimedLaunch> pending_timing;
    std::vector<std::vector<cudaEvent_t>> event_pool;  // per partition (device-bound)
    uint64_t launch_counter = 0;
    int cur_device = -1;
    cudaEvent_t timer_start = nullptr, timer_stop = nullptr;
    bool timer_running = false;
    int first_local = -1;    // lowest partition owned by this rank
    int nlocal = 0;          // partitions owned by this rank
    void* comm = nullptr;    // ncclComm_t (SPMD only)
    // one process, P partitions on P distinct GPUs: ncclComm_t per partition from ncclCommInitAll
    // (created at the first whole-buffer read; ag_state -1 = not tried, 0 = unavailable, 1 = ready)
    std::vector<void*> ag_comm;
    int ag_state = -1;
    // SPMD over peer memory (pk_init_spmd_ipc)
    bool ipc = false;
    pk_host_allgather_fn allgather = nullptr;
    void* ag_user = nullptr;
    uint64_t* flag_local = nullptr;      // device words [kFlagCopied, kFlagDone] of this rank
    std::vector<uint64_t*> flag;         // [p]: flag words of partition p's rank (mapped)
    std::vector<void*> flag_mapped;      // [p]: mapped bases to close
    uint64_t epoch = 0;                  // replicated launch epoch (flags are compared GEQ)
    bool flags_on_sm = false;            // epoch flags by SM kernels instead of stream memory operations
    std::vector<uint8_t> flag_on_peer_gpu;  // [p]: p's flag words live on another physical GPU
    std::unordered_map<std::string, std::pair<void*, int>> ipc_maps;  // handle -> (mapped base, refs)
    // steady-state graph replay (pk_api.h, PK_MODE_NO_GRAPHS)
    struct Memo {
        int seen = 0;
        cudaGraphExec_t exec = nullptr;
        struct Post { int64_t buf; SegState state; uint64_t fp; };
        std::vector<Post> pre;   // tracker states before the launch (checked on a hit: the key holds only hashes)
        std::vector<Post> post;  // tracker states after the launch (shared, restored by pointer)
        std::shared_ptr<const std::vector<CopyOp>> plan;
        pk_stats delta{};
    };
    std::unordered_map<std::string, Memo> memo;
    // launcher scratch (pk::context_scratch): [p][slot] = (pointer, bytes); retired blocks
    // stay allocated until pk_finalize (memoised graphs may still reference them)
    std::vector<std::array<std::pair<void*, size_t>, kScratchSlots>> scratch;
    std::vector<std::pair<int, void*>> scratch_retired;  // (device, pointer)
    bool graph_mode = false;  // all work is ordered on stream[first_local]
    bool graphs_broken = false;  // a capture / instantiation failed once: launch eagerly from now on
    bool capturing = false;      // inside a stream capture (no timing events: they would be graph nodes)
    cudaEvent_t ev_fork = nullptr;
    std::vector<cudaEvent_t> ev_join;
    // streamed operands (Builtin::stream_arg): per partition a side stream for the copies
    // that overlap the kernel, its fork/join events and kMaxGranules arrival flag words
    std::vector<cudaStream_t> side;
    std::vector<cudaEvent_t> ev_side_fork, ev_side_done;
    std::vector<uint32_t*> arrive_flags;
    // stream pieces whose source shares the destination's GPU too (off by default: measured on
    // a B200, a same-device D2D copy crawls while the consuming kernel holds every SM, whereas a
    // peer copy runs on the NVLink copy engines; PK_STREAM_SAME_DEVICE=1 at pk_init, for tests)
    bool stream_same_dev = false;

    bool local(int p) const { return prank[p] == rank; }
    int set_device(int d) {
        if (d != cur_device) {
            cudaError_t e = cudaSetDevice(d);
            if (e != cudaSuccess)
                return fail(PK_ERR_CUDA, std::string("cudaSetDevice: ") + cudaGetErrorName(e));
            cur_device = d;
        }
        return PK_OK;
    }
};

namespace {

bool valid_buf(pk_ctx c, pk_buf b) { return c && b >= 0 && b < (int64_t)c->bufs.size() && c->bufs[b].alive; }
bool valid_kernel(pk_ctx c, pk_kernel k) { return c && k >= 0 && k < (int64_t)c->kernels.size(); }

// ---- SPMD over peer memory (pk_init_spmd_ipc) ----
constexpr int kFlagCopied = 0;  // incoming copies of epoch E complete
constexpr int kFlagDone = 1;    // partition kernel of epoch E complete

// Driver entry points, resolved through the runtime at first use (the library does
// not link libcuda, so host-only contexts load on machines without a driver).
struct DriverApi {
    bool ok = false;
    CUresult (*WaitValue64)(CUstream, CUdeviceptr, cuuint64_t, unsigned) = nullptr;
    CUresult (*WriteValue64)(CUstream, CUdeviceptr, cuuint64_t, unsigned) = nullptr;
    CUresult (*WriteValue32)(CUstream, CUdeviceptr, cuuint32_t, unsigned) = nullptr;
    CUresult (*GetAddressRange)(CUdeviceptr*, size_t*, CUdeviceptr) = nullptr;
    CUresult (*GetErrorName)(CUresult, const char**) = nullptr;
};
DriverApi load_drv();
const DriverApi& drv() {  // process-wide driver entry points; thread-safe static initialisation
    static const DriverApi d = load_drv();
    return d;
}
DriverApi load_drv() {
    DriverApi d;
    auto get = [](const char* name, void** fn) {
        cudaDriverEntryPointQueryResult q;
        return cudaGetDriverEntryPointByVersion(name, fn, CUDART_VERSION, cudaEnableDefault, &q) == cudaSuccess &&
               q == cudaDriverEntryPointSuccess && *fn;
    };
    d.ok = get("cuStreamWaitValue64", (void**)&d.WaitValue64) && get("cuStreamWriteValue64", (void**)&d.WriteValue64) &&
           get("cuStreamWriteValue32", (void**)&d.WriteValue32) &&
           get("cuMemGetAddressRange", (void**)&d.GetAddressRange) && get("cuGetErrorName", (void**)&d.GetErrorName);
    return d;
}

#define PK_CU(call)                                                                        \
    do {                                                                                   \
        if (!drv().ok) return fail(PK_ERR_CUDA, "CUDA driver entry points unavailable");  \
        CUresult e_ = drv().call;                                                          \
        if (e_ != CUDA_SUCCESS) {                                                          \
            const char* s_ = nullptr;                                                      \
            drv().GetErrorName(e_, &s_);                                                   \
            return fail(PK_ERR_CUDA, std::string(#call) + ": " + (s_ ? s_ : "CUresult")); \
        }                                                                                  \
    } while (0)

int host_allgather(pk_ctx c, const void* send, void* recv, size_t n) {
    if (!c->allgather || c->allgather(c->ag_user, send, recv, n) != 0)
        return fail(PK_ERR_INVALID, "host all-gather callback failed");
    return PK_OK;
}

// Every rank's enqueued work is complete when this returns (local drain + host barrier).
int ipc_barrier(pk_ctx c) {
    for (int p = 0; p < c->P; ++p) {
        if (!c->local(p)) continue;
        if (int r = c->set_device(c->dev[p])) return r;
        PK_CUDA(cudaStreamSynchronize(c->stream[p]));
    }
    char s = 0;
    std::vector<char> all(c->world);
    return host_allgather(c, &s, all.data(), 1);
}

// After a barrier nothing is in flight anywhere: no epoch needs waiting for.
void ipc_settle(pk_ctx c) {
    for (Buffer& B : c->bufs)
        if (B.alive) {
            std::fill(B.ep_mod.begin(), B.ep_mod.end(), 0ull);
            std::fill(B.ep_read.begin(), B.ep_read.end(), 0ull);
            std::fill(B.ep_push.begin(), B.ep_push.end(), 0ull);
            std::fill(B.ep_kread.begin(), B.ep_kread.end(), 0ull);
        }
}

// Map a remote allocation (the same handle may back several buffers: reference counted).
int ipc_open(pk_ctx c, const cudaIpcMemHandle_t& h, void** out) {
    std::string key((const char*)&h, sizeof h);
    auto it = c->ipc_maps.find(key);
    if (it != c->ipc_maps.end()) {
        it->second.second += 1;
        *out = it->second.first;
        return PK_OK;
    }
    void* m = nullptr;
    PK_CUDA(cudaIpcOpenMemHandle(&m, h, cudaIpcMemLazyEnablePeerAccess));
    c->ipc_maps[key] = {m, 1};
    *out = m;
    return PK_OK;
}

void ipc_close(pk_ctx c, void* base) {
    for (auto it = c->ipc_maps.begin(); it != c->ipc_maps.end(); ++it)
        if (it->second.first == base) {
            if (--it->second.second == 0) {
                cudaIpcCloseMemHandle(base);
                c->ipc_maps.erase(it);
            }
            return;
        }
}

// Per-stream wait list: the max epoch needed from each partition's two flag words.
// Flags in this GPU's memory (ranks sharing the device) are waited for with stream
// memory operations (cuStreamWaitValue64, processed by the stream front end, no SM).
// Flags on another GPU are polled by the 1-thread SM kernel with system-scope
// acquire loads over NVLink (peer loads are the documented path; PK_FLAGS_MEMOP_PEER
// opts into stream memory operations on peer addresses instead).  If the driver
// refuses a memory operation the context switches to the SM kernels for good
// (PK_FLAGS_SM forces them everywhere).
struct FlagWaits {
    std::vector<uint64_t> need;  // [q*2 + word]
    explicit FlagWaits(int P) : need(2 * P, 0) {}
    void add(int q, int word, uint64_t e) { need[2 * q + word] = std::max(need[2 * q + word], e); }
    int issue(pk_ctx c, cudaStream_t s) {
        std::vector<const uint64_t*> fl;
        std::vector<uint64_t> tg;
        for (size_t i = 0; i < need.size(); ++i)
            if (need[i]) {
                const uint64_t* f = c->flag[i / 2] + (i % 2);
                if (!c->flags_on_sm && !c->flag_on_peer_gpu[i / 2]) {
                    CUresult e = drv().ok ? drv().WaitValue64((CUstream)s, (CUdeviceptr)f, need[i],
                                                              CU_STREAM_WAIT_VALUE_GEQ)
                                          : CUDA_ERROR_NOT_SUPPORTED;
                    if (e == CUDA_SUCCESS) continue;
                    c->flags_on_sm = true;
                }
                fl.push_back(f);
                tg.push_back(need[i]);
            }
        if (!fl.empty()) PK_CUDA(launch_flag_wait(fl.data(), tg.data(), (int)fl.size(), s));
        return PK_OK;
    }
};

int ipc_signal(pk_ctx c, int p, int word, uint64_t e) {
    uint64_t* f = c->flag_local + word;
    if (!c->flags_on_sm) {
        CUresult r = drv().ok ? drv().WriteValue64((CUstream)c->stream[p], (CUdeviceptr)f, e,
                                                   CU_STREAM_WRITE_VALUE_DEFAULT)
                              : CUDA_ERROR_NOT_SUPPORTED;
        if (r == CUDA_SUCCESS) return PK_OK;
        c->flags_on_sm = true;
    }
    PK_CUDA(launch_flag_write(f, e, c->stream[p]));
    return PK_OK;
}

// cudaMemcpy2DAsync / cudaMemcpy3DPeerAsync pitch bound (beyond it: one copy per piece)
constexpr uint64_t kMaxCopyPitch = 1ull << 30;
// strided runs of pieces up to this size go through the SM halo-copy kernel
constexpr uint64_t kNarrowPiece = 256;

int choose_source(uint64_t mask, int p, int P) {
    // reading Q5: nearest holder, ties to the lower index
    int best = -1, bestd = 1 << 30;
    for (int q = 0; q < P; ++q) {
        if (!((mask >> q) & 1)) continue;
        int d = q > p ? q - p : p - q;
        if (d < bestd) { bestd = d; best = q; }
    }
    return best;
}

// when every partition reads a whole buffer whose holders are exactly
// the linear slabs in rank order (N-body positions each step, GEMM B once), the
// plan for that buffer is P(P-1) copies, slab q -> every p != q: one all-gather.
// Returns the buffers whose plan entries form exactly that pattern (equal slabs).
std::vector<int64_t> allgather_buffers(const std::vector<CopyOp>& plan, int P,
                                       const std::vector<Buffer>& bufs) {
    std::vector<int64_t> out;
    if (P < 2) return out;
    std::unordered_map<int64_t, std::vector<const CopyOp*>> by;
    for (const CopyOp& o : plan) by[o.buf].push_back(&o);
    for (auto& kv : by) {
        const Buffer& B = bufs[kv.first];
        const uint64_t n = B.bytes / B.eb;
        if (n % P || kv.second.size() != (size_t)P * (P - 1)) continue;
        const uint64_t slab = n / P * B.eb;
        std::vector<uint8_t> seen((size_t)P * P, 0);
        bool ok = true;
        for (const CopyOp* o : kv.second) {
            if (o->src == o->dst || o->b != (uint64_t)o->src * slab || o->e != (uint64_t)(o->src + 1) * slab ||
                seen[(size_t)o->src * P + o->dst]++) {
                ok = false;
                break;
            }
        }
        if (ok) out.push_back(kv.first);
    }
    std::sort(out.begin(), out.end());
    return out;
}

int split_dim(const int32_t grid[3], int forced) {
    if (forced >= 0 && forced <= 2) return forced;
    for (int w = 2; w >= 0; --w)
        if (grid[w] > 1) return w;
    return 0;
}

// a1: partition p of the grid, box6 = (zmin,zmax,ymin,ymax,xmin,xmax)
void partition_box(const int32_t grid[3], int P, int p, int w, int64_t box[6]) {
    int64_t lo[3] = {0, 0, 0}, hi[3] = {grid[0], grid[1], grid[2]};
    int64_t g = hi[w];
    lo[w] = (p * g) / P;
    hi[w] = ((p + 1) * g) / P;
    box[0] = lo[2]; box[1] = hi[2];
    box[2] = lo[1]; box[3] = hi[1];
    box[4] = lo[0]; box[5] = hi[0];
}

// a1 with a tile shape (tx, ty, tz), tx*ty*tz == P: partition p is tile
// (p % tx, (p / tx) % ty, p / (tx*ty)), each grid dim split like partition_box
void tile_box(const int32_t grid[3], const int32_t tiles[3], int p, int64_t box[6]) {
    const int idx[3] = {p % tiles[0], (p / tiles[0]) % tiles[1], p / (tiles[0] * tiles[1])};
    int64_t lo[3], hi[3];
    for (int d = 0; d < 3; ++d) {
        lo[d] = (int64_t)idx[d] * grid[d] / tiles[d];
        hi[d] = (int64_t)(idx[d] + 1) * grid[d] / tiles[d];
    }
    box[0] = lo[2]; box[1] = hi[2];
    box[2] = lo[1]; box[3] = hi[1];
    box[4] = lo[0]; box[5] = hi[0];
}

void kernel_box(const Kernel& K, const int32_t grid[3], int P, int p, int64_t box[6]) {
    if (K.tiles[0] > 0) tile_box(grid, K.tiles, p, box);
    else partition_box(grid, P, p, split_dim(grid, K.partition_dim), box);
}

bool box_empty(const int64_t box[6]) { return box[0] >= box[1] || box[2] >= box[3] || box[4] >= box[5]; }

Status arg_ranges(const Kernel& k, int arg, int want_mode, const int64_t box[6], const Buffer& buf,
                  const EvalEnv& env, RangeList* out) {
    out->clear();
    RangeList tmp;
    for (const Tap& t : k.taps) {
        if (t.arg != arg) continue;
        bool is_read = t.mode == PK_READ || t.mode == PK_MAY_WRITE;
        bool is_write = t.mode == PK_WRITE || t.mode == PK_MAY_WRITE;
        if ((want_mode == PK_READ && !is_read) || (want_mode == PK_WRITE && !is_write)) continue;
        Status st = tap_ranges(t.acc, box, buf.ndim, buf.shape, buf.eb, env, &tmp);
        if (!st.ok()) return st;
        out->insert(out->end(), tmp.begin(), tmp.end());
    }
    canonicalize(out);
    return Status::Ok();
}

std::string region_key(const Kernel& k, int64_t kid, const int32_t grid[3], const int32_t block[3],
                       const int64_t* scalars, int ns, int P, const std::vector<const Buffer*>& bound) {
    std::string key;
    key.reserve(256);
    auto put = [&key](const void* p, size_t n) { key.append((const char*)p, n); };
    put(&kid, sizeof kid);
    put(&k.version, sizeof k.version);
    put(grid, 12);
    put(block, 12);
    put(&P, sizeof P);
    put(&ns, sizeof ns);
    if (ns) put(scalars, sizeof(int64_t) * ns);
    for (const Buffer* b : bound) {
        int64_t z = 0;
        if (!b) { put(&z, sizeof z); continue; }
        put(&b->ndim, sizeof b->ndim);
        put(b->shape, sizeof(int64_t) * b->ndim);
        put(&b->eb, sizeof b->eb);
    }
    return key;
}

}  // namespace

// ====================================================================== ABI
extern "C" {

const char* pk_last_error(void) { return g_err.c_str(); }
const char* pk_version(void) { return "pk 0.1 (sm_100a)"; }

int pk_nccl_unique_id(void* out, size_t bytes) {
    if (!out || bytes < sizeof(NcclId)) return fail(PK_ERR_INVALID, "need a 128-byte buffer");
    const NcclApi& n = nccl();
    if (!n.ok) return fail(PK_ERR_NCCL, "libnccl.so.2 could not be loaded (set PK_NCCL_LIB)");
    NcclId id;
    int r = n.GetUniqueId(&id);
    if (r) return fail(PK_ERR_NCCL, std::string("ncclGetUniqueId: ") + n.GetErrorString(r));
    std::memcpy(out, &id, sizeof id);
    return PK_OK;
}

static int init_impl(const pk_init_params* prm, const void* nccl_id, pk_host_allgather_fn ag, void* ag_user,
                     pk_ctx* out);

int pk_init(const pk_init_params* prm, pk_ctx* out) { return init_impl(prm, nullptr, nullptr, nullptr, out); }
int pk_init_spmd(const pk_init_params* prm, const void* nccl_id, pk_ctx* out) {
    return init_impl(prm, nccl_id, nullptr, nullptr, out);
}
int pk_init_spmd_ipc(const pk_init_params* prm, pk_host_allgather_fn ag, void* user, pk_ctx* out) {
    if (!ag) return fail(PK_ERR_INVALID, "pk_init_spmd_ipc needs a host all-gather callback");
    return init_impl(prm, nullptr, ag, user, out);
}

static int init_impl(const pk_init_params* prm, const void* nccl_id, pk_host_allgather_fn ag, void* ag_user,
                     pk_ctx* out) {
    if (!prm || !out) return fail(PK_ERR_INVALID, "null argument");
    if (prm->nparts < 1 || prm->nparts > PK_MAX_PARTS)
        return fail(PK_ERR_INVALID, "nparts must be in [1, 64]");
    if (prm->world_size < 1 || prm->my_rank < 0 || prm->my_rank >= prm->world_size)
        return fail(PK_ERR_INVALID, "bad rank/world_size");
    std::unique_ptr<pk_ctx_s> c(new pk_ctx_s());
    c->P = prm->nparts;
    c->rank = prm->my_rank;
    c->world = prm->world_size;
    c->init_flags = prm->flags;
    c->stream_same_dev = getenv("PK_STREAM_SAME_DEVICE") != nullptr;
    c->host_only = prm->flags & PK_INIT_HOST_ONLY;
    c->ipc = ag != nullptr && c->world > 1;
    c->allgather = ag;
    c->ag_user = ag_user;
    c->dev.assign(c->P, 0);
    c->prank.assign(c->P, 0);
    for (int p = 0; p < c->P; ++p) {
        if (prm->part_rank) {
            if (prm->part_rank[p] < 0 || prm->part_rank[p] >= c->world)
                return fail(PK_ERR_INVALID, "part_rank out of range");
            c->prank[p] = prm->part_rank[p];
        }
    }
    c->first_local = -1;
    for (int p = 0; p < c->P; ++p)
        if (c->local(p)) {
            if (c->first_local < 0) c->first_local = p;
            c->nlocal++;
        }
    if (c->ipc) {
        // collective handshake: every rank must describe the same partition -> rank map
        struct Cfg { int64_t P, world, map_hash, host_only; } mine{c->P, c->world, 1469598103934665603ll,
                                                                   (int64_t)c->host_only};
        for (int p = 0; p < c->P; ++p) mine.map_hash = (mine.map_hash ^ c->prank[p]) * 1099511628211ll;
        std::vector<Cfg> all(c->world);
        if (int r = host_allgather(c.get(), &mine, all.data(), sizeof mine)) return r;
        for (const Cfg& x : all)
            if (std::memcmp(&x, &mine, sizeof mine) != 0)
                return fail(PK_ERR_INVALID, "ranks disagree on nparts / world_size / part_rank / host-only");
    }
    if (!c->host_only) {
        int nlocal = 0;
        for (int p = 0; p < c->P; ++p) nlocal += c->local(p);
        if (c->world > 1 && nlocal != 1)
            return fail(PK_ERR_STATE, "SPMD execution needs exactly one partition per rank");
        if (c->world > 1 && !nccl_id && !c->ipc)
            return fail(PK_ERR_INVALID, "SPMD execution needs an NCCL unique id (or pk_init_spmd_ipc)");
        int ndev = 0;
        PK_CUDA(cudaGetDeviceCount(&ndev));
        if (ndev < 1) return fail(PK_ERR_CUDA, "no CUDA device");
        for (int p = 0; p < c->P; ++p) {
            if (!c->local(p)) continue;
            c->dev[p] = prm->part_device ? prm->part_device[p] : (c->world > 1 ? 0 : p % ndev);
            if (c->dev[p] < 0 || c->dev[p] >= ndev) return fail(PK_ERR_INVALID, "part_device out of range");
        }
        // peer access between every pair of distinct local devices in use
        std::vector<int> used;
        for (int p = 0; p < c->P; ++p)
            if (c->local(p)) used.push_back(c->dev[p]);
        std::sort(used.begin(), used.end());
        used.erase(std::unique(used.begin(), used.end()), used.end());
        // devices without peer access (no NVLink / P2P) still get copy-engine copies
        // (cudaMemcpyPeerAsync stages them); only SM-side peer loads and stores -- the
        // narrow-halo copy kernel and PK_MODE_PUSH -- need the pair enabled (c->peer)
        std::vector<std::pair<int, int>> enabled;
        for (int a : used)
            for (int b : used) {
                if (a == b) continue;
                int can = 0;
                PK_CUDA(cudaDeviceCanAccessPeer(&can, a, b));
                if (!can) continue;
                PK_CUDA(cudaSetDevice(a));
                cudaError_t e = cudaDeviceEnablePeerAccess(b, 0);
                if (e == cudaErrorPeerAccessAlreadyEnabled) cudaGetLastError();
                else if (e != cudaSuccess)
                    return fail(PK_ERR_CUDA, std::string("cudaDeviceEnablePeerAccess: ") + cudaGetErrorName(e));
                enabled.push_back({a, b});
            }
        c->peer.assign((size_t)c->P * c->P, 0);
        for (int p = 0; p < c->P; ++p)
            for (int q = 0; q < c->P; ++q)
                if (c->local(p) && c->local(q))
                    c->peer[(size_t)p * c->P + q] =
                        c->dev[p] == c->dev[q] ||
                        std::find(enabled.begin(), enabled.end(), std::make_pair(c->dev[p], c->dev[q])) != enabled.end();
        c->stream.resize(c->P);
        c->ev_kernel.resize(c->P);
        c->ev_copy.resize(c->P);
        c->event_pool.resize(c->P);
        c->ev_join.assign(c->P, nullptr);
        c->kernel_recorded.assign(c->P, 0);
        c->sm_count.assign(c->P, 148);
        for (int p = 0; p < c->P; ++p) {
            if (!c->local(p)) continue;
            PK_CUDA(cudaSetDevice(c->dev[p]));
            PK_CUDA(cudaDeviceGetAttribute(&c->sm_count[p], cudaDevAttrMultiProcessorCount, c->dev[p]));
            PK_CUDA(cudaStreamCreateWithFlags(&c->stream[p], cudaStreamNonBlocking));
            PK_CUDA(cudaEventCreateWithFlags(&c->ev_kernel[p], cudaEventDisableTiming));
            PK_CUDA(cudaEventCreateWithFlags(&c->ev_copy[p], cudaEventDisableTiming));
            PK_CUDA(cudaEventCreateWithFlags(&c->ev_join[p], cudaEventDisableTiming));
            c->cur_device = c->dev[p];
        }
        PK_CUDA(cudaSetDevice(c->dev[c->first_local]));
        PK_CUDA(cudaEventCreateWithFlags(&c->ev_fork, cudaEventDisableTiming));
        c->cur_device = c->dev[c->first_local];
        if (c->ipc) {
            c->flags_on_sm = getenv("PK_FLAGS_SM") != nullptr;
            // which ranks sit on another physical GPU (their flags are polled by SM kernels)
            cudaDeviceProp prop;
            PK_CUDA(cudaGetDeviceProperties(&prop, c->dev[c->first_local]));
            std::vector<cudaUUID_t> uu(c->world);
            if (int r = host_allgather(c.get(), &prop.uuid, uu.data(), sizeof(cudaUUID_t))) return r;
            const bool memop_peer = getenv("PK_FLAGS_MEMOP_PEER") != nullptr;
            c->flag_on_peer_gpu.assign(c->P, 0);
            for (int p = 0; p < c->P; ++p)
                c->flag_on_peer_gpu[p] = !memop_peer && std::memcmp(&uu[c->prank[p]], &prop.uuid, sizeof(cudaUUID_t)) != 0;
            // epoch flag words of this rank, mapped by every other rank
            if (int r = c->set_device(c->dev[c->first_local])) return r;
            PK_CUDA(cudaMalloc((void**)&c->flag_local, 256));
            PK_CUDA(cudaMemset(c->flag_local, 0, 256));
            PK_CUDA(cudaDeviceSynchronize());
            cudaIpcMemHandle_t h;
            PK_CUDA(cudaIpcGetMemHandle(&h, c->flag_local));
            std::vector<cudaIpcMemHandle_t> all(c->world);
            if (int r = host_allgather(c.get(), &h, all.data(), sizeof h)) return r;
            c->flag.assign(c->P, nullptr);
            c->flag_mapped.assign(c->P, nullptr);
            for (int p = 0; p < c->P; ++p) {
                if (c->local(p)) { c->flag[p] = c->flag_local; continue; }
                void* m = nullptr;
                if (int r = ipc_open(c.get(), all[c->prank[p]], &m)) return r;
                c->flag[p] = (uint64_t*)m;
                c->flag_mapped[p] = m;
            }
        } else if (c->world > 1) {
            const NcclApi& n = nccl();
            if (!n.ok) return fail(PK_ERR_NCCL, "libnccl.so.2 could not be loaded (set PK_NCCL_LIB)");
            if (int r = c->set_device(c->dev[c->first_local])) return r;
            NcclId id;
            std::memcpy(&id, nccl_id, sizeof id);
            int r = n.CommInitRank(&c->comm, c->world, id, c->rank);
            if (r) return fail(PK_ERR_NCCL, std::string("ncclCommInitRank: ") + n.GetErrorString(r));
        }
    }
    *out = c.release();
    return PK_OK;
}

static void clear_hazards(pk_ctx c) {
    std::fill(c->kernel_recorded.begin(), c->kernel_recorded.end(), (uint8_t)0);
    for (Buffer& B : c->bufs)
        if (B.alive) {
            std::fill(B.last_writer.begin(), B.last_writer.end(), (uint8_t)W_NONE);
            std::fill(B.readers.begin(), B.readers.end(), 0ull);
            std::fill(B.pushers.begin(), B.pushers.end(), 0ull);
        }
}

int pk_synchronize(pk_ctx c) {
    if (!c) return fail(PK_ERR_INVALID, "null ctx");
    if (c->host_only) return PK_OK;
    for (int p = 0; p < c->P; ++p) {
        if (!c->local(p)) continue;
        if (int r = c->set_device(c->dev[p])) return r;
        PK_CUDA(cudaStreamSynchronize(c->stream[p]));
    }
    // nothing is in flight any more: event hazards and graph mode are void
    c->graph_mode = false;
    clear_hazards(c);
    return PK_OK;
}

// Graph mode: every partition stream's tail is joined into stream[p0] so that a
// replayed graph (launched on p0, forking to the other streams internally) is
// ordered after everything enqueued before it.
static int enter_graph_mode(pk_ctx c) {
    if (c->graph_mode) return PK_OK;
    const int p0 = c->first_local;
    for (int p = 0; p < c->P; ++p) {
        if (!c->local(p) || p == p0) continue;
        if (int r = c->set_device(c->dev[p])) return r;
        PK_CUDA(cudaEventRecord(c->ev_join[p], c->stream[p]));
        if (int r = c->set_device(c->dev[p0])) return r;
        PK_CUDA(cudaStreamWaitEvent(c->stream[p0], c->ev_join[p], 0));
    }
    c->graph_mode = true;
    clear_hazards(c);  // stream order on p0 now covers every hazard
    return PK_OK;
}

// Leave graph mode before eager work: every stream waits for p0's tail.
static int exit_graph_mode(pk_ctx c) {
    if (!c->graph_mode) return PK_OK;
    const int p0 = c->first_local;
    if (int r = c->set_device(c->dev[p0])) return r;
    PK_CUDA(cudaEventRecord(c->ev_fork, c->stream[p0]));
    for (int p = 0; p < c->P; ++p) {
        if (!c->local(p) || p == p0) continue;
        if (int r = c->set_device(c->dev[p])) return r;
        PK_CUDA(cudaStreamWaitEvent(c->stream[p], c->ev_fork, 0));
    }
    c->graph_mode = false;
    clear_hazards(c);
    return PK_OK;
}

static void clear_memo(pk_ctx c) {
    for (auto& kv : c->memo)
        if (kv.second.exec) cudaGraphExecDestroy(kv.second.exec);
    c->memo.clear();
}

int pk_timer_begin(pk_ctx c) {
    if (!c) return fail(PK_ERR_INVALID, "null ctx");
    if (c->host_only) return fail(PK_ERR_STATE, "host-only context has no device timer");
    const int p0 = c->first_local;
    if (!c->timer_start) {
        for (cudaEvent_t* e : {&c->timer_start, &c->timer_stop}) {
            if (int r = c->set_device(c->dev[p0])) return r;
            PK_CUDA(cudaEventCreate(e));
        }
    }
    if (int r = c->set_device(c->dev[p0])) return r;
    PK_CUDA(cudaEventRecord(c->timer_start, c->stream[p0]));
    for (int p = 0; p < c->P; ++p) {
        if (!c->local(p) || p == p0) continue;
        if (int r = c->set_device(c->dev[p])) return r;
        PK_CUDA(cudaStreamWaitEvent(c->stream[p], c->timer_start, 0));
    }
    c->timer_running = true;
    return PK_OK;
}

int pk_timer_end(pk_ctx c, double* ms) {
    if (!c || !ms) return fail(PK_ERR_INVALID, "null argument");
    if (c->host_only || !c->timer_running) return fail(PK_ERR_STATE, "timer not running");
    const int p0 = c->first_local;
    for (int p = 0; p < c->P; ++p) {
        if (!c->local(p) || p == p0) continue;
        if (int r = c->set_device(c->dev[p])) return r;
        PK_CUDA(cudaEventRecord(c->ev_kernel[p], c->stream[p]));
        if (int r = c->set_device(c->dev[p0])) return r;
        PK_CUDA(cudaStreamWaitEvent(c->stream[p0], c->ev_kernel[p], 0));
    }
    if (int r = c->set_device(c->dev[p0])) return r;
    PK_CUDA(cudaEventRecord(c->timer_stop, c->stream[p0]));
    PK_CUDA(cudaEventSynchronize(c->timer_stop));
    float f = 0.f;
    PK_CUDA(cudaEventElapsedTime(&f, c->timer_start, c->timer_stop));
    *ms = f;
    c->timer_running = false;
    return PK_OK;
}

static int drain_timing(pk_ctx c) {
    for (TimedLaunch& t : c->pending_timing) {
        if (int r = c->set_device(c->dev[t.part])) return r;
        PK_CUDA(cudaEventSynchronize(t.stop));
        float ms = 0.f;
        PK_CUDA(cudaEventElapsedTime(&ms, t.start, t.stop));
        if (t.graph) {
            c->stats.graph_launch_ms += ms;
            c->stats.timed_graph_launches += t.nlaunch;
        } else {
            c->stats.kernel_ms += ms;
            c->stats.timed_kernels += 1;
        }
        c->event_pool[t.part].push_back(t.start);
        c->event_pool[t.part].push_back(t.stop);
    }
    // per launch: max over partitions
    std::unordered_map<uint64_t, double> mx;
    for (TimedLaunch& t : c->pending_timing) {
        if (t.graph) continue;
        float ms = 0.f;
        cudaEventElapsedTime(&ms, t.start, t.stop);
        double& v = mx[t.launch_id];
        v = std::max(v, (double)ms);
    }
    for (auto& kv : mx) c->stats.kernel_ms_max_launch += kv.second;
    c->stats.timed_eager_launches += mx.size();
    c->pending_timing.clear();
    return PK_OK;
}

int pk_finalize(pk_ctx c) {
    if (!c) return PK_OK;
    if (!c->host_only) {
        pk_synchronize(c);
        drain_timing(c);
        if (c->ipc) {
            // nobody may still read our instances / flags; unmap theirs before they free them
            ipc_barrier(c);
            for (Buffer& B : c->bufs)
                if (B.alive)
                    for (int p = 0; p < c->P; ++p)
                        if (B.ipc_base[p]) { ipc_close(c, B.ipc_base[p]); B.ipc_base[p] = nullptr; B.inst[p] = nullptr; }
            for (void* m : c->flag_mapped)
                if (m) ipc_close(c, m);
            ipc_barrier(c);
            if (c->flag_local) { cudaSetDevice(c->dev[c->first_local]); cudaFree(c->flag_local); }
        }
#ifdef PK_TRACE_ACCESS
        for (Buffer& B : c->bufs)
            if (B.alive)
                for (int p = 0; p < c->P; ++p)
                    if (B.inst[p] && c->local(p)) trace_remove(B.inst[p]);
#endif
        for (size_t b = 0; b < c->bufs.size(); ++b) {
            Buffer& B = c->bufs[b];
            if (B.alive && B.owned)
                for (int p = 0; p < c->P; ++p)
                    if (B.inst[p] && c->local(p)) { cudaSetDevice(c->dev[p]); cudaFree(B.inst[p]); }
        }
        clear_memo(c);
        for (size_t p = 0; p < c->scratch.size(); ++p)
            for (auto& s : c->scratch[p])
                if (s.first) { cudaSetDevice(c->dev[p]); cudaFree(s.first); }
        for (auto& r : c->scratch_retired) { cudaSetDevice(r.first); cudaFree(r.second); }
        for (size_t p = 0; p < c->side.size(); ++p)
            if (c->side[p]) {
                cudaSetDevice(c->dev[p]);
                cudaStreamDestroy(c->side[p]);
                cudaEventDestroy(c->ev_side_fork[p]);
                cudaEventDestroy(c->ev_side_done[p]);
                cudaFree(c->arrive_flags[p]);
            }
        for (int p = 0; p < c->P; ++p) {
            if (!c->local(p)) continue;
            cudaSetDevice(c->dev[p]);
            cudaStreamDestroy(c->stream[p]);
            cudaEventDestroy(c->ev_kernel[p]);
            cudaEventDestroy(c->ev_copy[p]);
            cudaEventDestroy(c->ev_join[p]);
            for (cudaEvent_t e : c->event_pool[p]) cudaEventDestroy(e);
        }
        if (c->ev_fork) { cudaSetDevice(c->dev[c->first_local]); cudaEventDestroy(c->ev_fork); }
        if (c->comm) nccl().CommDestroy(c->comm);
        for (void* cm : c->ag_comm)
            if (cm) nccl().CommDestroy(cm);
        if (c->timer_start) {
            cudaSetDevice(c->dev[c->first_local]);
            cudaEventDestroy(c->timer_start);
            cudaEventDestroy(c->timer_stop);
        }
    }
    delete c;
    return PK_OK;
}

// ------------------------------------------------------------------ buffers
int pk_register_buffer(pk_ctx c, int ndim, const int64_t* shape, int elem_bytes, void* const* dev_ptrs,
                       const void* host_init, pk_buf* out) {
    if (!c || !shape || !out) return fail(PK_ERR_INVALID, "null argument");
    if (ndim < 1 || ndim > PK_MAX_DIMS) return fail(PK_ERR_INVALID, "ndim must be 1..4");
    if (elem_bytes < 1) return fail(PK_ERR_INVALID, "elem_bytes must be >= 1");
    Buffer B;
    B.ndim = ndim;
    B.eb = elem_bytes;
    int64_t n = elem_bytes;
    for (int k = 0; k < ndim; ++k) {
        if (shape[k] < 0) return fail(PK_ERR_INVALID, "negative shape");
        B.shape[k] = shape[k];
        if (!mul_ok(n, shape[k], &n)) return fail(PK_ERR_OVERFLOW, "buffer size overflows int64");
    }
    B.bytes = (uint64_t)n;
    B.inst.assign(c->P, nullptr);
    B.last_writer.assign(c->P, W_NONE);
    B.readers.assign(c->P, 0);
    B.ep_mod.assign(c->P, 0);
    B.ep_kind.assign(c->P, W_NONE);
    B.ep_read.assign((size_t)c->P * c->P, 0);
    B.ipc_base.assign(c->P, nullptr);
    B.last_read.assign(c->P, RangeList{});
    B.pushers.assign(c->P, 0);
    B.ep_push.assign((size_t)c->P * c->P, 0);
    B.ep_kread.assign(c->P, 0);
    const uint64_t all = c->P == 64 ? ~0ull : ((1ull << c->P) - 1);
    B.tracker.init(B.bytes, all);  // reading Q3: undefined contents are valid everywhere
    if (!c->host_only) {
        if (dev_ptrs) {
            for (int p = 0; p < c->P; ++p) {
                if (!c->local(p)) continue;
                if (!dev_ptrs[p] && B.bytes) return fail(PK_ERR_INVALID, "null instance pointer");
                if (((uintptr_t)dev_ptrs[p]) % 16) return fail(PK_ERR_INVALID, "instance not 16-byte aligned");
                B.inst[p] = dev_ptrs[p];
            }
        } else {
            B.owned = true;
            for (int p = 0; p < c->P; ++p) {
                if (!c->local(p) || !B.bytes) continue;
                if (int r = c->set_device(c->dev[p])) return r;
                cudaError_t e = cudaMalloc(&B.inst[p], B.bytes);
                if (e != cudaSuccess) {
                    cudaGetLastError();
                    for (int q = 0; q < p; ++q)
                        if (B.inst[q]) { cudaSetDevice(c->dev[q]); cudaFree(B.inst[q]); }
                    c->cur_device = -1;
                    return fail(PK_ERR_OOM, "cudaMalloc of a buffer instance failed");
                }
            }
        }
    }
    if (c->ipc && !c->host_only) {
        // collective: export this rank's instance, map every other rank's (pulled from later)
        struct Exp {
            cudaIpcMemHandle_t h;
            uint64_t off;
            int64_t valid;
        } mine{};
        const int p0 = c->first_local;
        if (B.bytes) {
            CUdeviceptr base = 0;
            size_t sz = 0;
            if (int r = c->set_device(c->dev[p0])) return r;
            PK_CU(GetAddressRange(&base, &sz, (CUdeviceptr)B.inst[p0]));
            PK_CUDA(cudaIpcGetMemHandle(&mine.h, (void*)base));
            mine.off = (uint64_t)((CUdeviceptr)B.inst[p0] - base);
            mine.valid = 1;
        }
        std::vector<Exp> all(c->world);
        if (int r = host_allgather(c, &mine, all.data(), sizeof mine)) return r;
        for (int q = 0; q < c->P; ++q) {
            if (c->local(q)) continue;
            const Exp& x = all[c->prank[q]];
            if (!x.valid) continue;
            void* m = nullptr;
            if (int r = ipc_open(c, x.h, &m)) return r;
            B.ipc_base[q] = m;
            B.inst[q] = (char*)m + x.off;
        }
    }
#ifdef PK_TRACE_ACCESS
    if (!c->host_only)
        for (int p = 0; p < c->P; ++p)
            if (c->local(p) && B.inst[p] && B.bytes) {
                if (int r = c->set_device(c->dev[p])) return r;
                PK_CUDA(trace_add(B.inst[p], B.bytes));
            }
#endif
    B.alive = true;
    c->bufs.push_back(std::move(B));
    *out = (pk_buf)(c->bufs.size() - 1);
    if (host_init) {
        int r = pk_copy_from_host(c, *out, host_init, c->bufs[*out].bytes);
        if (r) return r;
    }
    return PK_OK;
}

int pk_buffer_instance(pk_ctx c, pk_buf b, int part, void** dev_ptr) {
    if (!valid_buf(c, b) || part < 0 || part >= c->P || !dev_ptr) return fail(PK_ERR_INVALID, "bad argument");
    *dev_ptr = c->bufs[b].inst[part];
    return PK_OK;
}

int pk_unregister_buffer(pk_ctx c, pk_buf b) {
    if (!valid_buf(c, b)) return fail(PK_ERR_INVALID, "bad buffer");
    Buffer& B = c->bufs[b];
    if (!c->host_only) {
        if (int r = pk_synchronize(c)) return r;
        clear_memo(c);  // replay graphs may reference the instances
    }
    if (c->ipc && !c->host_only) {
        // collective: every rank unmaps before any rank frees
        if (int r = ipc_barrier(c)) return r;
        for (int q = 0; q < c->P; ++q)
            if (B.ipc_base[q]) { ipc_close(c, B.ipc_base[q]); B.ipc_base[q] = nullptr; B.inst[q] = nullptr; }
        if (int r = ipc_barrier(c)) return r;
    }
#ifdef PK_TRACE_ACCESS
    for (int p = 0; p < c->P; ++p)
        if (B.inst[p] && c->local(p)) trace_remove(B.inst[p]);
#endif
    if (!c->host_only && B.owned) {
        for (int p = 0; p < c->P; ++p)
            if (B.inst[p] && c->local(p)) {
                if (int r = c->set_device(c->dev[p])) return r;
                PK_CUDA(cudaFree(B.inst[p]));
            }
    }
    B = Buffer();
    return PK_OK;
}

// Wait, on partition p's stream, for every copy that read (b,p) since its last write.
static int wait_readers(pk_ctx c, Buffer& B, int p) {
    uint64_t m = B.readers[p];
    for (int q = 0; m; ++q, m >>= 1) {
        if (!(m & 1) || q == p) continue;
        PK_CUDA(cudaStreamWaitEvent(c->stream[p], c->ev_copy[q], 0));
    }
    B.readers[p] = 0;
    return PK_OK;
}

int pk_copy_from_host(pk_ctx c, pk_buf b, const void* host, size_t bytes) {
    NvtxPhase nv("pk a8 H2D 1:n linear");
    if (!valid_buf(c, b) || !host) return fail(PK_ERR_INVALID, "bad argument");
    Buffer& B = c->bufs[b];
    if (bytes != B.bytes) return fail(PK_ERR_INVALID, "size mismatch (H2D copies the whole virtual buffer)");
    const uint64_t n = B.bytes / B.eb;
    uint64_t t0 = now_ns();
    if (!c->host_only) {
        if (int r = pk_synchronize(c)) return r;  // WAR against everything in flight
        if (c->ipc)                               // ... on every rank (peers may read our slab)
            if (int r = ipc_barrier(c)) return r;
        for (int p = 0; p < c->P; ++p) {
            if (!c->local(p)) continue;
            uint64_t lo = (uint64_t)p * n / c->P * B.eb, hi = (uint64_t)(p + 1) * n / c->P * B.eb;
            if (hi <= lo) continue;
            if (int r = c->set_device(c->dev[p])) return r;
            PK_CUDA(cudaMemcpyAsync((char*)B.inst[p] + lo, (const char*)host + lo, hi - lo,
                                    cudaMemcpyHostToDevice, c->stream[p]));
        }
        if (int r = pk_synchronize(c)) return r;
        if (c->ipc) {  // every slab is in place before any rank pulls from it
            if (int r = ipc_barrier(c)) return r;
            ipc_settle(c);
        }
        for (int p = 0; p < c->P; ++p) { B.last_writer[p] = W_NONE; B.readers[p] = 0; }
    }
    // linear distribution; tracker says slab p lives on p (reading Q2)
    for (int p = 0; p < c->P; ++p) {
        uint64_t lo = (uint64_t)p * n / c->P * B.eb, hi = (uint64_t)(p + 1) * n / c->P * B.eb;
        if (hi > lo) B.tracker.assign(RangeList{Range{lo, hi}}, 1ull << p);
    }
    c->stats.h2d_bytes += B.bytes;
    (void)t0;
    return PK_OK;
}

// Asynchronous H2D (single process): the same 1:n linear distribution, enqueued on
// the partition streams behind what they already hold instead of draining the
// context.  WAR: slab p's copy waits for the copies that read (b,p) on other streams
// (wait_readers); everything else that touches instance p (its kernels, incoming
// copies, D2H pieces) is on stream p already.  RAW: the copy is (b,p)'s last writer.
int pk_copy_from_host_async(pk_ctx c, pk_buf b, const void* host, size_t bytes) {
    if (!valid_buf(c, b) || !host) return fail(PK_ERR_INVALID, "bad argument");
    if (c->host_only || c->world > 1) return pk_copy_from_host(c, b, host, bytes);
    Buffer& B = c->bufs[b];
    if (bytes != B.bytes) return fail(PK_ERR_INVALID, "size mismatch (H2D copies the whole virtual buffer)");
    for (uint64_t m : B.pushers)   // bytes pushed into an instance by another partition's kernel: drain
        if (m) {
            if (int r = pk_synchronize(c)) return r;
            break;
        }
    if (int r = exit_graph_mode(c)) return r;
    const uint64_t n = B.bytes / B.eb;
    for (int p = 0; p < c->P; ++p) {
        uint64_t lo = (uint64_t)p * n / c->P * B.eb, hi = (uint64_t)(p + 1) * n / c->P * B.eb;
        if (hi <= lo || !c->local(p)) continue;
        if (int r = c->set_device(c->dev[p])) return r;
        if (int r = wait_readers(c, B, p)) return r;
        PK_CUDA(cudaMemcpyAsync((char*)B.inst[p] + lo, (const char*)host + lo, hi - lo, cudaMemcpyHostToDevice,
                                c->stream[p]));
        if (c->P > 1) {
            PK_CUDA(cudaEventRecord(c->ev_copy[p], c->stream[p]));
            B.last_writer[p] = W_COPY;
        }
    }
    for (int p = 0; p < c->P; ++p) {
        uint64_t lo = (uint64_t)p * n / c->P * B.eb, hi = (uint64_t)(p + 1) * n / c->P * B.eb;
        if (hi > lo) B.tracker.assign(RangeList{Range{lo, hi}}, 1ull << p);
    }
    c->stats.h2d_bytes += B.bytes;
    return PK_OK;
}

int pk_copy_from_host_for(pk_ctx c, pk_buf b, const void* host, size_t bytes, pk_kernel k, int arg,
                          const int32_t grid[3], const int32_t block[3], const int64_t* scalars, int ns) {
    if (!valid_buf(c, b) || !host || !valid_kernel(c, k) || !grid || !block) return fail(PK_ERR_INVALID, "bad argument");
    if (ns < 0 || ns > PK_MAX_SCALARS || (ns && !scalars)) return fail(PK_ERR_INVALID, "bad scalars");
    Buffer& B = c->bufs[b];
    if (bytes != B.bytes) return fail(PK_ERR_INVALID, "size mismatch (H2D copies the whole virtual buffer)");
    const Kernel& K = c->kernels[k];
    if (arg < 0 || arg >= K.nargs || K.kinds[arg] != PK_ARG_BUFFER) return fail(PK_ERR_INVALID, "bad arg index");
    const int P = c->P;
    EvalEnv env{scalars, ns, {block[0], block[1], block[2]}};
    std::vector<RangeList> U(P);
    RangeList covered;
    for (int p = 0; p < P; ++p) {
        int64_t box[6];
        kernel_box(K, grid, P, p, box);
        if (box_empty(box)) continue;
        Status st = arg_ranges(K, arg, PK_READ, box, B, env, &U[p]);
        if (!st.ok()) return fail(st);
        covered = union_ranges(covered, U[p]);
    }
    // bytes nobody reads keep the linear distribution
    const uint64_t n = B.bytes / B.eb;
    for (int p = 0; p < P; ++p) {
        const uint64_t lo = (uint64_t)p * n / P * B.eb, hi = (uint64_t)(p + 1) * n / P * B.eb;
        uint64_t cur = lo;
        RangeList extra;
        for (const Range& r : covered) {
            if (r.e <= cur) continue;
            if (r.b >= hi) break;
            if (r.b > cur) extra.push_back(Range{cur, std::min(r.b, hi)});
            cur = std::max(cur, r.e);
            if (cur >= hi) break;
        }
        if (cur < hi) extra.push_back(Range{cur, hi});
        if (!extra.empty()) U[p] = union_ranges(U[p], extra);
    }
    if (!c->host_only) {
        if (int r = pk_synchronize(c)) return r;
        if (c->ipc)
            if (int r = ipc_barrier(c)) return r;
        for (int p = 0; p < P; ++p) {
            if (!c->local(p)) continue;
            if (int r = c->set_device(c->dev[p])) return r;
            for (const Range& r : U[p])
                PK_CUDA(cudaMemcpyAsync((char*)B.inst[p] + r.b, (const char*)host + r.b, r.e - r.b,
                                        cudaMemcpyHostToDevice, c->stream[p]));
        }
        if (int r = pk_synchronize(c)) return r;
        if (c->ipc) {
            if (int r = ipc_barrier(c)) return r;
            ipc_settle(c);
        }
        for (int p = 0; p < P; ++p) { B.last_writer[p] = W_NONE; B.readers[p] = 0; }
    }
    B.tracker.init(B.bytes, 0);
    for (int p = 0; p < P; ++p)
        if (!U[p].empty()) B.tracker.add_bit(U[p], p);
    for (int p = 0; p < P; ++p) c->stats.h2d_bytes += total_bytes(U[p]);
    return PK_OK;
}

static int sync_to_host_spmd(pk_ctx c, Buffer& B, void* host) {
    // collective n:1 gather to rank 0: segments rank 0's partition lacks are sent
    // by their lowest holder straight into rank 0's instance, which then holds them
    int r0 = -1;
    for (int p = 0; p < c->P; ++p)
        if (c->prank[p] == 0) { r0 = p; break; }
    if (r0 < 0) return fail(PK_ERR_STATE, "rank 0 owns no partition");
    struct Piece { uint64_t b, e; int src; };
    std::vector<Piece> pieces;
    RangeList received;
    for (const Seg& s : B.tracker.segments()) {
        int src = ((s.mask >> r0) & 1) ? r0 : -1;
        for (int q = 0; q < c->P && src < 0; ++q)
            if ((s.mask >> q) & 1) src = q;
        if (src < 0) return fail(PK_ERR_STATE, "segment held by no partition");
        if (!pieces.empty() && pieces.back().src == src && pieces.back().e == s.b) pieces.back().e = s.e;
        else pieces.push_back({s.b, s.e, src});
    }
    const NcclApi& n = nccl();
    const bool is_root = c->rank == 0;
    if (int r = c->set_device(c->dev[c->first_local])) return r;
    n.GroupStart();
    for (const Piece& pc : pieces) {
        if (pc.src == r0) continue;
        received.push_back(Range{pc.b, pc.e});
        int r = 0;
        if (c->local(pc.src))
            r = n.Send((const char*)B.inst[pc.src] + pc.b, pc.e - pc.b, kNcclUint8, 0, c->comm, c->stream[pc.src]);
        else if (is_root)
            r = n.Recv((char*)B.inst[r0] + pc.b, pc.e - pc.b, kNcclUint8, c->prank[pc.src], c->comm, c->stream[r0]);
        if (r) { n.GroupEnd(); return fail(PK_ERR_NCCL, std::string("ncclSend/Recv: ") + n.GetErrorString(r)); }
    }
    if (int r = n.GroupEnd()) return fail(PK_ERR_NCCL, std::string("ncclGroupEnd: ") + n.GetErrorString(r));
    if (is_root)
        PK_CUDA(cudaMemcpyAsync(host, B.inst[r0], B.bytes, cudaMemcpyDeviceToHost, c->stream[r0]));
    if (int r = pk_synchronize(c)) return r;
    if (!(c->mode & PK_MODE_SINGLE_OWNER)) {  // replicated on every rank: r0 now holds what it received
        canonicalize(&received);
        B.tracker.add_bit(received, r0);
    }
    c->stats.d2h_bytes += is_root ? B.bytes : 0;
    return PK_OK;
}

static int sync_to_host_ipc(pk_ctx c, Buffer& B, void* host) {
    // collective n:1 gather to rank 0 over peer memory: rank 0 pulls every segment its
    // partition lacks from the lowest holder's mapped instance into its own instance
    // (same tracker semantics as the NCCL variant), then copies the whole buffer down
    int r0 = -1;
    for (int p = 0; p < c->P; ++p)
        if (c->prank[p] == 0) { r0 = p; break; }
    if (r0 < 0) return fail(PK_ERR_STATE, "rank 0 owns no partition");
    if (int r = ipc_barrier(c)) return r;  // every rank's writes are complete
    RangeList received;
    struct Piece { uint64_t b, e; int src; };
    std::vector<Piece> pieces;
    for (const Seg& s : B.tracker.segments()) {
        int src = ((s.mask >> r0) & 1) ? r0 : -1;
        for (int q = 0; q < c->P && src < 0; ++q)
            if ((s.mask >> q) & 1) src = q;
        if (src < 0) return fail(PK_ERR_STATE, "segment held by no partition");
        if (!pieces.empty() && pieces.back().src == src && pieces.back().e == s.b) pieces.back().e = s.e;
        else pieces.push_back({s.b, s.e, src});
    }
    for (const Piece& pc : pieces) {
        if (pc.src == r0) continue;
        received.push_back(Range{pc.b, pc.e});
        if (c->rank != 0) continue;
        if (int r = c->set_device(c->dev[r0])) return r;
        PK_CUDA(cudaMemcpyAsync((char*)B.inst[r0] + pc.b, (const char*)B.inst[pc.src] + pc.b, pc.e - pc.b,
                                cudaMemcpyDefault, c->stream[r0]));
    }
    if (c->rank == 0) {
        if (int r = c->set_device(c->dev[r0])) return r;
        PK_CUDA(cudaMemcpyAsync(host, B.inst[r0], B.bytes, cudaMemcpyDeviceToHost, c->stream[r0]));
    }
    if (int r = ipc_barrier(c)) return r;  // nobody overwrites what rank 0 read
    ipc_settle(c);
    if (!(c->mode & PK_MODE_SINGLE_OWNER)) {
        canonicalize(&received);
        B.tracker.add_bit(received, r0);
    }
    c->stats.d2h_bytes += c->rank == 0 ? B.bytes : 0;
    return PK_OK;
}

static int sync_to_host(pk_ctx c, pk_buf b, void* host, size_t bytes, bool async) {
    NvtxPhase nv("pk a8 D2H n:1 gather");
    if (!valid_buf(c, b)) return fail(PK_ERR_INVALID, "bad argument");
    Buffer& B = c->bufs[b];
    if (bytes != B.bytes) return fail(PK_ERR_INVALID, "size mismatch (D2H gathers the whole virtual buffer)");
    if (c->host_only) return fail(PK_ERR_STATE, "host-only context holds no data");
    if (!host && (c->world == 1 || c->rank == 0)) return fail(PK_ERR_INVALID, "null host buffer");
    if (c->world > 1) return c->ipc ? sync_to_host_ipc(c, B, host) : sync_to_host_spmd(c, B, host);
    // bytes pushed into an instance by another partition's kernel: drain everything first
    for (uint64_t m : B.pushers)
        if (m) {
            if (int r = pk_synchronize(c)) return r;
            break;
        }
    // replay graphs run on stream[p0]: fork the other streams from its tail first
    if (int r = exit_graph_mode(c)) return r;
    // query all segments, copy each from a partition that holds it.
    struct Piece { uint64_t b, e; int src; };
    std::vector<Piece> pieces;
    for (const Seg& s : B.tracker.segments()) {
        int src = -1;
        for (int q = 0; q < c->P; ++q)
            if (((s.mask >> q) & 1) && c->local(q)) { src = q; break; }
        if (src < 0) return fail(PK_ERR_STATE, "segment held by no local partition");
        if (!pieces.empty() && pieces.back().src == src && pieces.back().e == s.b) pieces.back().e = s.e;
        else pieces.push_back({s.b, s.e, src});
    }
    for (const Piece& pc : pieces) {
        if (int r = c->set_device(c->dev[pc.src])) return r;
        PK_CUDA(cudaMemcpyAsync((char*)host + pc.b, (const char*)B.inst[pc.src] + pc.b, pc.e - pc.b,
                                cudaMemcpyDeviceToHost, c->stream[pc.src]));
    }
    c->stats.d2h_bytes += B.bytes;
    return async ? PK_OK : pk_synchronize(c);
}

int pk_sync_to_host(pk_ctx c, pk_buf b, void* host, size_t bytes) { return sync_to_host(c, b, host, bytes, false); }

// Asynchronous D2H (single process, not with PK_MODE_PUSH): the pieces are enqueued on
// the streams of the partitions that hold them, behind their writers; the host buffer
// is complete after pk_synchronize.  A later write into a piece's instance is on the
// same stream, so it cannot overtake the copy.
int pk_sync_to_host_async(pk_ctx c, pk_buf b, void* host, size_t bytes) {
    if (c && (c->world > 1 || (c->mode & PK_MODE_PUSH))) return pk_sync_to_host(c, b, host, bytes);
    return sync_to_host(c, b, host, bytes, true);
}

// ------------------------------------------------------------------ kernels
int pk_register_kernel(pk_ctx c, const char* name, const void* fn, int nargs, const int32_t* arg_kind,
                       int32_t partition_dim, pk_kernel* out) {
    if (!c || !out || !arg_kind) return fail(PK_ERR_INVALID, "null argument");
    if (nargs < 0 || nargs > PK_MAX_ARGS) return fail(PK_ERR_INVALID, "nargs must be 0..16");
    if (partition_dim < -1 || partition_dim > 2) return fail(PK_ERR_INVALID, "partition_dim must be -1..2");
    Kernel k;
    k.name = name ? name : "";
    k.fn = fn;
    k.launcher = find_builtin_launcher(fn);  // a builtin __global__ keeps its own launch geometry
    k.push_arg = find_builtin_push_arg(fn);
    if (const Builtin* bi = find_builtin_by_fn(fn)) {
        k.stream_arg = bi->stream_arg;
        k.stream_granule = bi->stream_granule;
    }
    k.nargs = nargs;
    k.partition_dim = partition_dim;
    for (int i = 0; i < nargs; ++i) {
        if (arg_kind[i] != PK_ARG_BUFFER && arg_kind[i] != PK_ARG_SCALAR)
            return fail(PK_ERR_INVALID, "arg_kind must be PK_ARG_BUFFER or PK_ARG_SCALAR");
        k.kinds[i] = arg_kind[i];
    }
    c->kernels.push_back(std::move(k));
    *out = (pk_kernel)(c->kernels.size() - 1);
    return PK_OK;
}

int pk_declare_affine_access(pk_ctx c, pk_kernel k, int arg, int mode, const pk_affine_access* tap) {
    if (!valid_kernel(c, k) || !tap) return fail(PK_ERR_INVALID, "bad kernel or null tap");
    Kernel& K = c->kernels[k];
    if (arg < 0 || arg >= K.nargs || K.kinds[arg] != PK_ARG_BUFFER)
        return fail(PK_ERR_INVALID, "arg_index is not a buffer argument");
    if (mode != PK_READ && mode != PK_WRITE && mode != PK_MAY_WRITE) return fail(PK_ERR_INVALID, "bad mode");
    if (tap->ndim < 1 || tap->ndim > PK_MAX_DIMS) return fail(PK_ERR_INVALID, "tap ndim must be 1..4");
    int used[3] = {0, 0, 0};
    for (int d = 0; d < tap->ndim; ++d) {
        int g = tap->dim[d].grid_dim;
        if (g < -1 || g > 2) return fail(PK_ERR_INVALID, "grid_dim must be -1..2");
        if (g >= 0 && used[g]++) return fail(PK_ERR_INVALID, "a grid dimension drives two array dimensions");
    }
    K.taps.push_back(Tap{arg, mode, *tap});
    K.version++;
    return PK_OK;
}

const void* pk_builtin_fn(const char* name) {
    const Builtin* b = find_builtin(name);
    return b ? b->fn : nullptr;
}

int pk_builtin_kernel(pk_ctx c, const char* name, pk_kernel* out) {
    const Builtin* b = find_builtin(name);
    if (!b) return fail(PK_ERR_INVALID, std::string("unknown builtin kernel '") + (name ? name : "") + "'");
    int r = pk_register_kernel(c, b->name, b->fn, b->nargs, b->kinds, b->partition_dim, out);
    if (r) return r;
    c->kernels[*out].launcher = b->launcher;
    return b->describe(c, *out);
}

int pk_set_partition_shape(pk_ctx c, pk_kernel k, const int32_t tiles[3]) {
    if (!valid_kernel(c, k)) return fail(PK_ERR_INVALID, "bad kernel");
    Kernel& K = c->kernels[k];
    if (!tiles || (tiles[0] == 0 && tiles[1] == 0 && tiles[2] == 0)) {
        K.tiles[0] = K.tiles[1] = K.tiles[2] = 0;
    } else {
        if (tiles[0] < 1 || tiles[1] < 1 || tiles[2] < 1)
            return fail(PK_ERR_INVALID, "tile counts must be >= 1 (or all 0 for the 1-D split)");
        if ((int64_t)tiles[0] * tiles[1] * tiles[2] != c->P)
            return fail(PK_ERR_INVALID, "tx*ty*tz must equal the number of partitions");
        for (int d = 0; d < 3; ++d) K.tiles[d] = tiles[d];
    }
    K.version++;  // region cache + launch memo keys
    return PK_OK;
}

int pk_partition_grid(pk_ctx c, pk_kernel k, const int32_t grid[3], int part, int64_t part_out[6]) {
    if (!valid_kernel(c, k) || !grid || !part_out || part < 0 || part >= c->P)
        return fail(PK_ERR_INVALID, "bad argument");
    kernel_box(c->kernels[k], grid, c->P, part, part_out);
    return PK_OK;
}

int pk_enumerate(pk_ctx c, pk_kernel k, int arg, int mode, pk_buf b, const int64_t part[6],
                 const int32_t block[3], const int64_t* scalars, int ns, pk_range_cb cb, void* user) {
    if (!valid_kernel(c, k) || !valid_buf(c, b) || !part || !block || !cb) return fail(PK_ERR_INVALID, "bad argument");
    if (ns < 0 || ns > PK_MAX_SCALARS || (ns && !scalars)) return fail(PK_ERR_INVALID, "bad scalars");
    const Kernel& K = c->kernels[k];
    if (arg < 0 || arg >= K.nargs) return fail(PK_ERR_INVALID, "bad arg index");
    EvalEnv env{scalars, ns, {block[0], block[1], block[2]}};
    RangeList r;
    Status st = arg_ranges(K, arg, mode == PK_WRITE ? PK_WRITE : PK_READ, part, c->bufs[b], env, &r);
    if (!st.ok()) return fail(st);
    for (const Range& x : r) cb(user, x.b, x.e);
    return PK_OK;
}

int pk_tracker_dump(pk_ctx c, pk_buf b, pk_segment_cb cb, void* user) {
    if (!valid_buf(c, b) || !cb) return fail(PK_ERR_INVALID, "bad argument");
    for (const Seg& s : c->bufs[b].tracker.segments()) cb(user, s.b, s.e, s.mask);
    return PK_OK;
}

int pk_last_plan(pk_ctx c, pk_copy_cb cb, void* user) {
    if (!c || !cb) return fail(PK_ERR_INVALID, "bad argument");
    for (const CopyOp& o : c->replay_plan ? *c->replay_plan : c->last_plan) cb(user, o.buf, o.src, o.dst, o.b, o.e);
    return PK_OK;
}

int pk_get_stats(pk_ctx c, pk_stats* out) {
    if (!c || !out) return fail(PK_ERR_INVALID, "bad argument");
    if (!c->host_only && !c->pending_timing.empty())
        if (int r = drain_timing(c)) return r;
    *out = c->stats;
    return PK_OK;
}

int pk_reset_stats(pk_ctx c) {
    if (!c) return fail(PK_ERR_INVALID, "bad argument");
    if (!c->host_only && !c->pending_timing.empty())
        if (int r = drain_timing(c)) return r;
    c->stats = pk_stats{};
    return PK_OK;
}

int pk_set_mode(pk_ctx c, uint32_t flags) {
    if (!c) return fail(PK_ERR_INVALID, "bad argument");
    if (flags & ~0x1FFu) return fail(PK_ERR_INVALID, "unknown mode flag");
    if ((flags & PK_MODE_PUSH) && !c->host_only && !c->ipc)
        for (int p = 0; p < c->P; ++p)
            for (int q = 0; q < c->P; ++q)
                if (c->local(p) && c->local(q) && !c->sm_reach(p, q))
                    return fail(PK_ERR_INVALID, "PK_MODE_PUSH needs peer access between devices " +
                                                    std::to_string(c->dev[p]) + " and " + std::to_string(c->dev[q]));
    c->mode = flags;
    return PK_OK;
}
uint32_t pk_get_mode(pk_ctx c) { return c ? c->mode : 0; }

// ------------------------------------------------------------------ Fig. 4
static int launch_eager(pk_ctx c, pk_kernel k, const int32_t grid[3], const int32_t block[3], size_t smem,
                        const void* const* args, const int64_t* scalars, int ns);

static void add_stats(pk_stats& a, const pk_stats& d, int sign) {
    a.launches += sign * d.launches;
    a.kernel_launches += sign * d.kernel_launches;
    a.copies += sign * d.copies;
    a.strided_copies += sign * d.strided_copies;
    a.copy_kernels += sign * d.copy_kernels;
    a.stale_bytes += sign * d.stale_bytes;
    a.moved_bytes += sign * d.moved_bytes;
    a.pushed_bytes += sign * d.pushed_bytes;
    a.collectives += sign * d.collectives;
    a.streamed_bytes += sign * d.streamed_bytes;
    for (int i = 0; i < 16; ++i)
        for (int j = 0; j < 16; ++j) a.pair_bytes[i][j] += sign * d.pair_bytes[i][j];
}

namespace {
// One partitioned launch as the memoised launch path sees it.
struct LaunchReq {
    pk_kernel k;
    const int32_t* grid;
    const int32_t* block;
    size_t smem;
    const void* const* args;
    const int64_t* scalars;
    int ns;
};
}  // namespace

static int check_launch(pk_ctx c, const LaunchReq& d) {
    if (!valid_kernel(c, d.k) || !d.grid || !d.block) return fail(PK_ERR_INVALID, "bad argument");
    if (d.ns < 0 || d.ns > PK_MAX_SCALARS || (d.ns && !d.scalars)) return fail(PK_ERR_INVALID, "bad scalars");
    return PK_OK;
}

// n partitioned launches in order, memoised as ONE graph: the key is every launch's
// identity plus the pre-launch tracker state of every buffer bound by any of them; the
// first sighting runs eagerly, the second is captured (transfers, kernels and event edges
// of all n launches), later sightings with the same pre-state replay it and restore the
// recorded post-states.  n = 1 is pk_launch_partitioned.
static int launch_memo(pk_ctx c, const LaunchReq* d, int n) {
    const uint32_t mode = c->mode;
    auto eager_all = [&]() -> int {
        for (int i = 0; i < n; ++i)
            if (int r = launch_eager(c, d[i].k, d[i].grid, d[i].block, d[i].smem, d[i].args, d[i].scalars, d[i].ns))
                return r;
        return PK_OK;
    };
    // builtin launchers take every scalar from `scalars`, so the key below captures the launch
    // (contexts that all-gathered through NCCL launch eagerly: collectives stay out of captures)
    bool can_graph = !c->host_only && c->world == 1 && c->nlocal >= 1 && !c->graphs_broken && c->ag_comm.empty() &&
                     !(mode & (PK_MODE_GLOBAL_BARRIER | PK_MODE_NO_GRAPHS));
    for (int i = 0; i < n && can_graph; ++i) {
        const Kernel& K = c->kernels[d[i].k];
        can_graph = K.nargs && d[i].args && K.launcher;
    }
    if (!can_graph) {
        if (!c->host_only)
            if (int r = exit_graph_mode(c)) return r;
        return eager_all();
    }
    // ---- memo key: launch identities + pre-launch tracker state of every bound buffer ----
    uint64_t t0 = now_ns();
    std::string key;
    key.reserve(256 * n);
    auto put = [&key](const void* p, size_t sz) { key.append((const char*)p, sz); };
    put(&n, sizeof n);
    const uint32_t kmode = mode & ~(uint32_t)PK_MODE_TIME_KERNELS;  // timing events sit outside the graph
    put(&kmode, sizeof kmode);
    std::vector<int64_t> bids;
    for (int i = 0; i < n; ++i) {
        const LaunchReq& q = d[i];
        const Kernel& K = c->kernels[q.k];
        put(&q.k, sizeof q.k);
        put(&K.version, sizeof K.version);
        put(q.grid, 12);
        put(q.block, 12);
        put(&q.smem, sizeof q.smem);
        put(&q.ns, sizeof q.ns);
        if (q.ns) put(q.scalars, sizeof(int64_t) * q.ns);
        for (int a = 0; a < K.nargs; ++a) {
            if (K.kinds[a] == PK_ARG_BUFFER) {
                if (!q.args[a]) return fail(PK_ERR_INVALID, "null buffer argument");
                const pk_buf b = *(const pk_buf*)q.args[a];
                if (!valid_buf(c, b))
                    return fail(PK_ERR_INVALID, "argument " + std::to_string(a) + " is not a live buffer");
                put(&b, sizeof b);
                if (std::find(bids.begin(), bids.end(), b) == bids.end()) bids.push_back(b);
            }
        }
    }
    for (int64_t b : bids) {
        const uint64_t f = c->bufs[b].tracker.fingerprint();
        put(&f, sizeof f);
    }
    auto it = c->memo.find(key);
    if (it != c->memo.end()) {
        // the key holds 64-bit fingerprints of the tracker states: confirm the states
        // themselves (pointer equality, as states are shared copy-on-write, else contents)
        bool same = it->second.pre.size() == bids.size();
        for (size_t i = 0; same && i < bids.size(); ++i) {
            const auto& pr = it->second.pre[i];
            const SegState cur = c->bufs[bids[i]].tracker.state();
            same = pr.buf == bids[i] && (pr.state == cur || (pr.state && cur && *pr.state == *cur));
        }
        if (!same) {  // fingerprint collision: forget the entry, launch eagerly
            if (it->second.exec) cudaGraphExecDestroy(it->second.exec);
            c->memo.erase(it);
            it = c->memo.end();
        }
    }
    std::vector<pk_ctx_s::Memo::Post> pre_states;
    pre_states.reserve(bids.size());
    for (int64_t b : bids) {
        const Tracker& T = c->bufs[b].tracker;
        pre_states.push_back({b, T.state(), T.fingerprint()});
    }
    if (it != c->memo.end() && it->second.exec) {
        // ---- replay: one graph launch + restore the memoised tracker states ----
        NvtxPhase nv("pk graph replay");
        pk_ctx_s::Memo& m = it->second;
        if (int r = enter_graph_mode(c)) return r;
        const int p0 = c->first_local;
        if (int r = c->set_device(c->dev[p0])) return r;
        cudaEvent_t e0 = nullptr, e1 = nullptr;
        if (mode & PK_MODE_TIME_KERNELS) {  // the whole replayed graph, on the stream it runs on
            auto& pool = c->event_pool[p0];
            for (cudaEvent_t* e : {&e0, &e1}) {
                if (!pool.empty()) { *e = pool.back(); pool.pop_back(); }
                else PK_CUDA(cudaEventCreate(e));
            }
            PK_CUDA(cudaEventRecord(e0, c->stream[p0]));
        }
        PK_CUDA(cudaGraphLaunch(m.exec, c->stream[p0]));
        if (mode & PK_MODE_TIME_KERNELS) {
            PK_CUDA(cudaEventRecord(e1, c->stream[p0]));
            TimedLaunch tl{e0, e1, p0, c->launch_counter};
            tl.graph = true;
            tl.nlaunch = n;
            c->pending_timing.push_back(tl);
        }
        for (auto& ps : m.post) c->bufs[ps.buf].tracker.set_state(ps.state, ps.fp);
        c->replay_plan = m.plan;
        add_stats(c->stats, m.delta, 1);
        c->stats.graph_replays += n;
        c->launch_counter += n;
        c->stats.host_ns_issue += now_ns() - t0;
        return PK_OK;
    }
    const bool capture = it != c->memo.end() && it->second.seen >= 1;
    pk_stats before = c->stats;
    int rc;
    if (!capture) {
        if (int r = exit_graph_mode(c)) return r;
        rc = eager_all();
        if (rc) return rc;
    } else {
        // ---- capture the launches once into a multi-stream graph ----
        // host state the eager path mutates, restored if capture or instantiation fails
        std::vector<std::vector<RangeList>> saved_last_read;
        std::vector<std::vector<uint64_t>> saved_pushers;
        for (int64_t b : bids) {
            saved_last_read.push_back(c->bufs[b].last_read);
            saved_pushers.push_back(c->bufs[b].pushers);
        }
        const uint64_t saved_counter = c->launch_counter;
        auto fall_back = [&](const std::string& why) -> int {
            // a failed capture enqueued nothing: undo the bookkeeping and run eagerly, and
            // keep this context on the eager path (no silent retry of a failing capture)
            for (size_t i = 0; i < bids.size(); ++i) {
                Buffer& B = c->bufs[bids[i]];
                B.tracker.set_state(pre_states[i].state, pre_states[i].fp);
                B.last_read = saved_last_read[i];
                B.pushers = saved_pushers[i];
            }
            c->stats = before;
            c->launch_counter = saved_counter;
            c->graphs_broken = true;
            c->stats.graph_fallbacks += 1;
            g_err = why;
            clear_memo(c);
            c->graph_mode = false;  // capture ended; stream[p0] already follows every stream's tail
            if (int r = exit_graph_mode(c)) return r;
            return eager_all();
        };
        if (int r = enter_graph_mode(c)) return r;
        const int p0 = c->first_local;
        if (int r = c->set_device(c->dev[p0])) return r;
        PK_CUDA(cudaStreamBeginCapture(c->stream[p0], cudaStreamCaptureModeRelaxed));
        cudaError_t ce = cudaEventRecord(c->ev_fork, c->stream[p0]);
        for (int p = 0; p < c->P && ce == cudaSuccess; ++p)
            if (c->local(p) && p != p0) {
                c->set_device(c->dev[p]);
                ce = cudaStreamWaitEvent(c->stream[p], c->ev_fork, 0);
            }
        c->capturing = true;
        rc = ce == cudaSuccess ? eager_all() : fail(PK_ERR_CUDA, std::string("graph fork: ") + cudaGetErrorName(ce));
        c->capturing = false;
        if (rc == PK_OK && getenv("PK_DEBUG_FAIL_CAPTURE"))  // test hook: exercise the eager fallback
            rc = fail(PK_ERR_CUDA, "PK_DEBUG_FAIL_CAPTURE");
        for (int p = 0; p < c->P && rc == PK_OK; ++p)
            if (c->local(p) && p != p0) {
                c->set_device(c->dev[p]);
                ce = cudaEventRecord(c->ev_join[p], c->stream[p]);
                c->set_device(c->dev[p0]);
                if (ce == cudaSuccess) ce = cudaStreamWaitEvent(c->stream[p0], c->ev_join[p], 0);
                if (ce != cudaSuccess) rc = fail(PK_ERR_CUDA, std::string("graph join: ") + cudaGetErrorName(ce));
            }
        c->set_device(c->dev[p0]);
        cudaGraph_t g = nullptr;
        cudaError_t ee = cudaStreamEndCapture(c->stream[p0], &g);
        clear_hazards(c);  // events recorded during capture are graph nodes, not real records
        if (rc || ee != cudaSuccess) {
            if (g) cudaGraphDestroy(g);
            cudaGetLastError();
            if (rc == PK_ERR_WRITE_OVERLAP || rc == PK_ERR_INVALID || rc == PK_ERR_OUT_OF_BOUNDS ||
                rc == PK_ERR_OVERFLOW)
                return rc;  // a user error, not a capture problem: same answer eagerly
            const int r = fall_back(std::string("graph capture failed: ") +
                                    (rc ? g_err : std::string(cudaGetErrorName(ee))));
            if (r) return r;
            goto record;
        }
        {
            cudaGraphExec_t ex = nullptr;
            ee = cudaGraphInstantiate(&ex, g, 0);
            cudaGraphDestroy(g);
            if (ee != cudaSuccess) {
                cudaGetLastError();
                const int r = fall_back(std::string("cudaGraphInstantiate: ") + cudaGetErrorName(ee));
                if (r) return r;
                goto record;
            }
            PK_CUDA(cudaGraphLaunch(ex, c->stream[p0]));
            if (c->memo.size() > 256) clear_memo(c);
            c->memo[key].exec = ex;
            c->stats.graph_captures += n;
        }
    }
record:
    if (c->graphs_broken) return PK_OK;  // eager from now on: nothing to memoise
    pk_ctx_s::Memo& m = c->memo[key];
    m.pre = std::move(pre_states);
    m.seen += 1;
    m.plan = std::make_shared<const std::vector<CopyOp>>(c->last_plan);
    m.delta = c->stats;
    add_stats(m.delta, before, -1);
    m.delta.graph_replays = m.delta.graph_captures = 0;
    m.post.clear();
    for (int64_t b : bids) {
        const Tracker& T = c->bufs[b].tracker;
        m.post.push_back({b, T.state(), T.fingerprint()});
    }
    return PK_OK;
}

namespace {
struct CpuTime {  // thread CPU time of a launch call -> pk_stats.host_cpu_ns
    pk_ctx c;
    uint64_t t0 = thread_cpu_ns();
    ~CpuTime() { c->stats.host_cpu_ns += thread_cpu_ns() - t0; }
};
}  // namespace

int pk_launch_partitioned(pk_ctx c, pk_kernel k, const int32_t grid[3], const int32_t block[3], size_t smem,
                          const void* const* args, const int64_t* scalars, int ns) {
    const LaunchReq d{k, grid, block, smem, args, scalars, ns};
    if (int r = check_launch(c, d)) return r;
    CpuTime cpu_time{c};
    return launch_memo(c, &d, 1);
}

int pk_launch_sequence(pk_ctx c, const pk_launch_desc* launches, int n) {
    if (!c || n < 0 || (n && !launches)) return fail(PK_ERR_INVALID, "bad argument");
    if (n > PK_MAX_SEQUENCE) return fail(PK_ERR_INVALID, "more than PK_MAX_SEQUENCE launches");
    if (n == 0) return PK_OK;
    std::vector<LaunchReq> d(n);
    for (int i = 0; i < n; ++i) {
        const pk_launch_desc& l = launches[i];
        d[i] = LaunchReq{l.kernel, l.grid, l.block, l.smem_bytes, l.args, l.scalars, l.nscalars};
        if (int r = check_launch(c, d[i])) return r;
    }
    CpuTime cpu_time{c};
    return launch_memo(c, d.data(), n);
}

// Streamed operand (Builtin::stream_arg): the stale ranges of buffer `b` bound for partition
// p are copied on p's side stream, granule by granule, while p's kernel runs; after the
// last piece of granule g the stream front end stores 1 into flag g (cuStreamWriteValue32:
// no SM is needed, so a kernel that occupies every SM while it polls cannot starve it).
// The flags are reset on p's stream before the fork, i.e. after p's previous kernel.
// Granules go in the order the consumer needs them: starting after p's own linear slab
// (a row partition of the GEMM starts its K loop on the chunks it holds, see sgemm_tc.cu).
static int issue_streamed(pk_ctx c, int p, int64_t b, const std::vector<CopyOp>& ops, uint64_t granule,
                          Arrival* out) {
    Buffer& B = c->bufs[b];
    if (c->side.empty()) {
        c->side.assign(c->P, nullptr);
        c->ev_side_fork.assign(c->P, nullptr);
        c->ev_side_done.assign(c->P, nullptr);
        c->arrive_flags.assign(c->P, nullptr);
    }
    if (!c->side[p]) {
        PK_CUDA(cudaStreamCreateWithFlags(&c->side[p], cudaStreamNonBlocking));
        PK_CUDA(cudaEventCreateWithFlags(&c->ev_side_fork[p], cudaEventDisableTiming));
        PK_CUDA(cudaEventCreateWithFlags(&c->ev_side_done[p], cudaEventDisableTiming));
        PK_CUDA(cudaMalloc((void**)&c->arrive_flags[p], kMaxGranules * sizeof(uint32_t)));
        PK_CUDA(cudaMemset(c->arrive_flags[p], 0, kMaxGranules * sizeof(uint32_t)));
    }
    uint32_t* flags = c->arrive_flags[p];
    const uint64_t ng = (B.bytes + granule - 1) / granule;
    struct Piece { uint64_t g, b, e; int src; };
    std::vector<Piece> pieces;
    uint64_t need = 0;
    for (const CopyOp& o : ops)
        for (uint64_t x = o.b; x < o.e;) {
            const uint64_t g = x / granule, y = std::min(o.e, (g + 1) * granule);
            pieces.push_back({g, x, y, o.src});
            need |= 1ull << g;
            x = y;
        }
    const uint64_t g0 = std::min<uint64_t>(ng - 1, (uint64_t)(p + 1) * B.bytes / c->P / granule);
    std::stable_sort(pieces.begin(), pieces.end(), [&](const Piece& x, const Piece& y) {
        const uint64_t rx = (x.g + ng - g0) % ng, ry = (y.g + ng - g0) % ng;
        return rx != ry ? rx < ry : x.b < y.b;
    });
    for (uint64_t m = need; m; m &= m - 1)  // granules this launch copies: not arrived yet
        PK_CU(WriteValue32((CUstream)c->stream[p], (CUdeviceptr)(flags + __builtin_ctzll(m)), 0u,
                           CU_STREAM_WRITE_VALUE_DEFAULT));
    PK_CUDA(cudaEventRecord(c->ev_side_fork[p], c->stream[p]));  // after every hazard wait on stream[p]
    PK_CUDA(cudaStreamWaitEvent(c->side[p], c->ev_side_fork[p], 0));
    for (size_t i = 0; i < pieces.size(); ++i) {
        const Piece& x = pieces[i];
        char* dst = (char*)B.inst[p] + x.b;
        const char* src = (const char*)B.inst[x.src] + x.b;
        if (c->dev[x.src] == c->dev[p])
            PK_CUDA(cudaMemcpyAsync(dst, src, x.e - x.b, cudaMemcpyDeviceToDevice, c->side[p]));
        else
            PK_CUDA(cudaMemcpyPeerAsync(dst, c->dev[p], src, c->dev[x.src], x.e - x.b, c->side[p]));
        c->stats.copies += 1;
        c->stats.moved_bytes += x.e - x.b;
        c->stats.streamed_bytes += x.e - x.b;
        if (x.src < 16 && p < 16) c->stats.pair_bytes[x.src][p] += x.e - x.b;
        if (i + 1 == pieces.size() || pieces[i + 1].g != x.g)  // granule complete
            PK_CU(WriteValue32((CUstream)c->side[p], (CUdeviceptr)(flags + x.g), 1u, CU_STREAM_WRITE_VALUE_DEFAULT));
    }
    PK_CUDA(cudaEventRecord(c->ev_copy[p], c->side[p]));
    *out = Arrival{flags, need, granule};
    return PK_OK;
}

// One process, P partitions on P distinct GPUs: one NCCL communicator per
// partition from ncclCommInitAll, rank p = partition p, created at the first whole-buffer
// read.  False (peer copies instead) when partitions share a GPU -- NCCL refuses two ranks on
// one device -- or NCCL is not loadable.
static bool single_process_comms(pk_ctx c) {
    if (c->ag_state >= 0) return c->ag_state == 1;
    c->ag_state = 0;
    const NcclApi& n = nccl();
    if (c->P < 2 || c->world != 1 || c->ipc || !n.ok || !n.CommInitAll) return false;
    for (int p = 0; p < c->P; ++p)
        for (int q = 0; q < p; ++q)
            if (c->dev[p] == c->dev[q]) return false;
    std::vector<void*> comms((size_t)c->P, nullptr);
    if (n.CommInitAll(comms.data(), c->P, c->dev.data()) != 0) return false;
    c->ag_comm = std::move(comms);
    c->ag_state = 1;
    c->cur_device = -1;  // NCCL initialisation switches devices
    return true;
}

// The plan entries of each buffer in `bufs` are exactly "slab q -> every p != q" for P equal
// linear slabs (allgather_buffers): one in-place ncclAllGather per buffer, all partitions in
// one group, each on its partition's stream after pass 1's waits.  NVLS multicast on
// NVSwitch where NCCL selects it.
static int allgather_single_process(pk_ctx c, const std::vector<int64_t>& bufs) {
    const NcclApi& n = nccl();
    const int P = c->P;
    if (int r = n.GroupStart()) return fail(PK_ERR_NCCL, std::string("ncclGroupStart: ") + n.GetErrorString(r));
    for (int64_t b : bufs) {
        const Buffer& B = c->bufs[b];
        const uint64_t slab = B.bytes / P;
        for (int p = 0; p < P; ++p) {
            if (int r = c->set_device(c->dev[p])) { n.GroupEnd(); return r; }
            int r = n.AllGather((const char*)B.inst[p] + (uint64_t)p * slab, B.inst[p], slab, kNcclUint8,
                                c->ag_comm[p], c->stream[p]);
            if (r) { n.GroupEnd(); return fail(PK_ERR_NCCL, std::string("ncclAllGather: ") + n.GetErrorString(r)); }
            c->stats.copies += P - 1;
            c->stats.moved_bytes += (uint64_t)(P - 1) * slab;
            for (int q = 0; q < P && q < 16; ++q)
                if (q != p && p < 16) c->stats.pair_bytes[q][p] += slab;
        }
    }
    const int r = n.GroupEnd();
    c->cur_device = -1;  // NCCL may have switched the current device
    if (r) return fail(PK_ERR_NCCL, std::string("ncclGroupEnd: ") + n.GetErrorString(r));
    return PK_OK;
}

static int launch_eager(pk_ctx c, pk_kernel k, const int32_t grid[3], const int32_t block[3], size_t smem,
                        const void* const* args, const int64_t* scalars, int ns) {
    if (!valid_kernel(c, k) || !grid || !block) return fail(PK_ERR_INVALID, "bad argument");
    if (ns < 0 || ns > PK_MAX_SCALARS || (ns && !scalars)) return fail(PK_ERR_INVALID, "bad scalars");
    const Kernel& K = c->kernels[k];
    if (K.nargs && !args) return fail(PK_ERR_INVALID, "null args");
    for (int w = 0; w < 3; ++w)
        if (grid[w] < 0 || block[w] < 1) return fail(PK_ERR_INVALID, "bad grid/block");
    const int P = c->P;
    // resolve buffer arguments
    std::vector<const Buffer*> bound(K.nargs, nullptr);
    std::vector<int64_t> bid(K.nargs, -1);
    for (int a = 0; a < K.nargs; ++a) {
        if (K.kinds[a] != PK_ARG_BUFFER) continue;
        if (!args[a]) return fail(PK_ERR_INVALID, "null buffer argument");
        pk_buf b = *(const pk_buf*)args[a];
        if (!valid_buf(c, b)) return fail(PK_ERR_INVALID, "argument " + std::to_string(a) + " is not a live buffer");
        bound[a] = &c->bufs[b];
        bid[a] = b;
    }
    const uint32_t mode = c->mode;
    const bool track = !(mode & PK_MODE_NO_TRACKING);
    const bool transfer = track && !(mode & PK_MODE_NO_TRANSFERS);
    const bool single_owner = mode & PK_MODE_SINGLE_OWNER;
    uint64_t t0 = now_ns();
    NvtxPhase nv("pk a1+a2 partition, regions");

    // ---- a1 + a2: partition boxes and regions (cached) ----
    std::shared_ptr<std::vector<Regions>> regs;
    std::string key = region_key(K, k, grid, block, scalars, ns, P, bound);
    auto it = c->region_cache.find(key);
    uint64_t t1 = now_ns();
    if (it != c->region_cache.end()) {
        regs = it->second;
    } else {
        regs = std::make_shared<std::vector<Regions>>(P);
        EvalEnv env{scalars, ns, {block[0], block[1], block[2]}};
        for (int p = 0; p < P; ++p) {
            Regions& R = (*regs)[p];
            kernel_box(K, grid, P, p, R.box);
            R.empty = box_empty(R.box);
            R.args.resize(K.nargs);
            if (R.empty) continue;
            for (int a = 0; a < K.nargs; ++a) {
                if (!bound[a]) continue;
                Status st = arg_ranges(K, a, PK_READ, R.box, *bound[a], env, &R.args[a].r);
                if (st.ok()) st = arg_ranges(K, a, PK_WRITE, R.box, *bound[a], env, &R.args[a].w);
                if (!st.ok()) return fail(st);
            }
        }
        if (c->region_cache.size() > 4096) c->region_cache.clear();
        c->region_cache.emplace(key, regs);
    }
    c->stats.host_ns_partition += t1 - t0;
    uint64_t t2 = now_ns();
    c->stats.host_ns_regions += t2 - t1;
    nv.next("pk a3 stale detection, plan");

    // per (partition, distinct buffer): merged read / write sets
    struct BufSets { int64_t b; RangeList r, w; };
    std::vector<std::vector<BufSets>> sets(P);
    if (track) {
        for (int p = 0; p < P; ++p) {
            const Regions& R = (*regs)[p];
            if (R.empty) continue;
            for (int a = 0; a < K.nargs; ++a) {
                if (!bound[a]) continue;
                BufSets* bs = nullptr;
                for (auto& x : sets[p]) if (x.b == bid[a]) bs = &x;
                if (!bs) { sets[p].push_back(BufSets{bid[a], {}, {}}); bs = &sets[p].back(); }
                if (!R.args[a].r.empty()) bs->r = bs->r.empty() ? R.args[a].r : union_ranges(bs->r, R.args[a].r);
                if (!R.args[a].w.empty()) bs->w = bs->w.empty() ? R.args[a].w : union_ranges(bs->w, R.args[a].w);
            }
        }
        // WAW across partitions: reject before anything happens
        std::unordered_map<int64_t, std::vector<std::pair<Range, int>>> allw;
        for (int p = 0; p < P; ++p)
            for (auto& bs : sets[p])
                for (const Range& x : bs.w) allw[bs.b].push_back({x, p});
        for (auto& kv : allw) {
            auto& v = kv.second;
            std::sort(v.begin(), v.end(), [](const std::pair<Range, int>& a, const std::pair<Range, int>& b) {
                return a.first.b < b.first.b;
            });
            for (size_t i = 1; i < v.size(); ++i)
                if (v[i].first.b < v[i - 1].first.e && v[i].second != v[i - 1].second)
                    return fail(PK_ERR_WRITE_OVERLAP, "partitions " + std::to_string(v[i - 1].second) + " and " +
                                                          std::to_string(v[i].second) +
                                                          " write the same bytes of buffer " + std::to_string(kv.first));
        }
    }

    // ---- a3: stale detection + transfer plan against the pre-launch state ----
    c->last_plan.clear();
    c->replay_plan.reset();
    if (track) {
        for (int p = 0; p < P; ++p) {
            for (auto& bs : sets[p]) {
                const Buffer& B = c->bufs[bs.b];
                for (const Range& x : bs.r) {
                    B.tracker.query(x.b, x.e, [&](uint64_t lo, uint64_t hi, uint64_t m) {
                        if ((m >> p) & 1) return;
                        c->stats.stale_bytes += hi - lo;
                        int q = choose_source(m, p, P);
                        if (!c->last_plan.empty()) {
                            CopyOp& l = c->last_plan.back();
                            if (l.buf == bs.b && l.src == q && l.dst == p && l.e == lo) { l.e = hi; return; }
                        }
                        c->last_plan.push_back(CopyOp{bs.b, q, p, lo, hi});
                    });
                }
            }
        }
        if (!single_owner)  // validity map: a reader becomes a co-holder (reading Q4)
            for (int p = 0; p < P; ++p)
                for (auto& bs : sets[p])
                    if (!bs.r.empty()) c->bufs[bs.b].tracker.add_bit(bs.r, p);
    }
    // ---- halo push plan (PK_MODE_PUSH): predict that the next reader of a written buffer
    // reads what its last reader read; the producing kernel then also stores those bytes
    // straight into the reader's instance (fused, peer stores over NVLink), and the tracker
    // records the reader as a holder, so the next launch finds nothing stale.
    struct PushRec { int64_t b; int q, p; RangeList r; };
    std::vector<PushList> push(P);
    std::vector<PushRec> pushed;
    const int pa = K.push_arg;
    if ((mode & PK_MODE_PUSH) && !single_owner && transfer && pa >= 0 && pa < K.nargs && bound[pa] &&
        (c->world == 1 || c->ipc)) {
        const int64_t b = bid[pa];
        bool read_here = false;  // the buffer must not also be read by this launch
        for (int p = 0; p < P && !read_here; ++p)
            for (auto& bs : sets[p])
                if (bs.b == b && !bs.r.empty()) read_here = true;
        const Buffer& B = c->bufs[b];
        for (int q = 0; q < P && !read_here; ++q) {
            const RangeList* Wq = nullptr;
            for (auto& bs : sets[q])
                if (bs.b == b) Wq = &bs.w;
            if (!Wq || Wq->empty()) continue;
            PushList pl{};
            std::vector<PushRec> recs;
            bool fits = true;
            for (int p = 0; p < P && fits; ++p) {
                if (p == q || B.last_read[p].empty()) continue;
                RangeList x = intersect_ranges(*Wq, B.last_read[p]);
                if (x.empty()) continue;
                for (const Range& r : x) {
                    if (pl.n == kMaxPush || (r.b | r.e) % 4) { fits = false; break; }
                    pl.lo[pl.n] = r.b;
                    pl.hi[pl.n] = r.e;
                    pl.dst[pl.n] = (uint64_t)(uintptr_t)B.inst[p];
                    pl.n++;
                }
                recs.push_back(PushRec{b, q, p, std::move(x)});
            }
            if (!fits || recs.empty()) continue;  // too fragmented: those bytes are pulled as usual
            push[q] = pl;
            for (auto& r : recs) pushed.push_back(std::move(r));
        }
    }

    // NCCL SPMD: whole-buffer reads become one in-place all-gather per buffer
    std::vector<int64_t> ag_bufs;
    if (c->world > 1 && !c->ipc && transfer) {
        ag_bufs = allgather_buffers(c->last_plan, P, c->bufs);
        c->stats.collectives += ag_bufs.size();
    }

    uint64_t t3 = now_ns();
    c->stats.host_ns_plan += t3 - t2;
    nv.next("pk a4+a5 transfers, ordering");
    c->stats.launches += 1;
    const uint64_t launch_id = c->launch_counter++;
    const uint64_t E = c->ipc ? ++c->epoch : 0;  // replicated: identical on every rank

    // ---- a4 + a5: transfers, pulled on the destination stream ----
    // streamed operand: the copies of the kernel's stream_arg buffer overlap its kernel
    std::vector<Arrival> arrival(P, Arrival{nullptr, 0, 0});
    std::vector<uint8_t> side_pending(P, 0);
    int64_t sbuf = -1;
    uint64_t granule = 0;
    if (!c->host_only && transfer && K.stream_arg >= 0 && K.stream_arg < K.nargs && bound[K.stream_arg] &&
        K.stream_granule && c->world == 1 && !c->ipc && drv().ok &&
        !(mode & (PK_MODE_GLOBAL_BARRIER | PK_MODE_NO_OVERLAP))) {
        granule = K.stream_granule(scalars, ns);
        const Buffer& SB = *bound[K.stream_arg];
        bool alone = true;  // the buffer bound to another argument too (C = A A): those reads do not poll
        for (int a = 0; a < K.nargs; ++a)
            if (a != K.stream_arg && bound[a] && bid[a] == bid[K.stream_arg]) alone = false;
        if (alone && granule && (SB.bytes + granule - 1) / granule <= (uint64_t)kMaxGranules)
            sbuf = bid[K.stream_arg];
    }
    // one process driving P distinct GPUs: the same pattern goes to an in-place
    // ncclAllGather over a communicator of the partitions' devices (ncclCommInitAll)
    std::vector<int64_t> ag_local;
    if (c->world == 1 && !c->ipc && !c->host_only && !c->capturing && transfer &&
        !(mode & PK_MODE_NO_COLLECTIVES) && !c->last_plan.empty()) {
        ag_local = allgather_buffers(c->last_plan, P, c->bufs);
        ag_local.erase(std::remove(ag_local.begin(), ag_local.end(), sbuf), ag_local.end());  // streamed instead
        if (!ag_local.empty() && !single_process_comms(c)) ag_local.clear();  // peer copies instead
        c->stats.collectives += ag_local.size();
    }
    if (!c->host_only) {
        if (transfer && !c->last_plan.empty()) {
            // the plan's runs of equal destination [i, j) that this process pulls
            struct Group { size_t i, j; int p; };
            std::vector<Group> groups;
            for (size_t i = 0; i < c->last_plan.size();) {
                const int p = c->last_plan[i].dst;
                size_t j = i;
                while (j < c->last_plan.size() && c->last_plan[j].dst == p) ++j;
                if (c->local(p)) groups.push_back(Group{i, j, p});  // else another rank pulls
                i = j;
            }
            // Pass 1: every destination's waits, before ANY copy of this launch is issued.
            // The plan was made against the pre-launch tracker state (a3), so a copy never
            // reads bytes another copy of the same launch delivers: its RAW is on the source's
            // pre-launch writer, and its WAR on readers of earlier launches.  Waiting here, on
            // events not yet re-recorded by this launch, keeps the destinations' pulls
            // concurrent (waiting inside the issue loop chained partition p's pulls behind
            // p-1's, whose ev_copy had just been re-recorded).
            for (const Group& g : groups) {
                const size_t i = g.i, j = g.j;
                const int p = g.p;
                if (int r = c->set_device(c->dev[p])) return r;
                if (c->ipc) {
                    // peer memory: RAW on the holder's flag word of its last write of (b,q);
                    // WAR on (b,p): readers of earlier launches must have finished copying it
                    FlagWaits fw(P);
                    for (size_t t = i; t < j; ++t) {
                        const CopyOp& o = c->last_plan[t];
                        const Buffer& B = c->bufs[o.buf];
                        if (B.ep_mod[o.src])
                            fw.add(o.src, B.ep_kind[o.src] == W_COPY ? kFlagCopied : kFlagDone, B.ep_mod[o.src]);
                        for (int q = 0; q < P; ++q)  // bytes pushed into (b, src) by q's kernel
                            if (B.ep_push[(size_t)o.src * P + q]) fw.add(q, kFlagDone, B.ep_push[(size_t)o.src * P + q]);
                        for (int r = 0; r < P; ++r)
                            if (B.ep_read[(size_t)p * P + r]) fw.add(r, kFlagCopied, B.ep_read[(size_t)p * P + r]);
                    }
                    if (int r = fw.issue(c, c->stream[p])) return r;
                }
                // WAR on the destination instances + RAW on each source's last writer (kernel
                // or copy, per buffer: two buffers of one source may differ)
                uint64_t waited_k = 0, waited_c = 0;
                for (size_t t = i; t < j; ++t) {
                    const CopyOp& o = c->last_plan[t];
                    if (!c->local(o.src)) continue;
                    Buffer& B = c->bufs[o.buf];
                    if (B.readers[p]) if (int r = wait_readers(c, B, p)) return r;
                    for (uint64_t m = B.pushers[o.src]; m; m &= m - 1) {  // bytes pushed into (b, src)
                        const int q = __builtin_ctzll(m);
                        PK_CUDA(cudaStreamWaitEvent(c->stream[p], c->ev_kernel[q], 0));
                    }
                    const uint8_t lw = B.last_writer[o.src];
                    const uint64_t bit = 1ull << o.src;
                    uint64_t& waited = lw == W_KERNEL ? waited_k : waited_c;
                    if (lw != W_NONE && !(waited & bit)) {
                        PK_CUDA(cudaStreamWaitEvent(c->stream[p], lw == W_KERNEL ? c->ev_kernel[o.src]
                                                                                 : c->ev_copy[o.src], 0));
                        waited |= bit;
                    }
                }
            }
            // one-process multi-GPU: whole-buffer reads as one in-place all-gather per buffer
            if (!ag_local.empty())
                if (int r = allgather_single_process(c, ag_local)) return r;
            // Pass 2: the copies, pulled on the destination stream
            std::vector<size_t> order;
            for (const Group& g : groups) {
                const size_t i = g.i, j = g.j;
                const int p = g.p;
                if (int r = c->set_device(c->dev[p])) return r;
                // group by (buffer, source) in plan order; a run of equal-length pieces at a
                // constant pitch (a tile partition's halo column, NEXT-2) is ONE 2-D copy
                order.resize(j - i);
                for (size_t t = i; t < j; ++t) order[t - i] = t;
                std::stable_sort(order.begin(), order.end(), [&](size_t a, size_t b) {
                    const CopyOp &x = c->last_plan[a], &y = c->last_plan[b];
                    return x.buf != y.buf ? x.buf < y.buf : x.src < y.src;
                });
                // run2d(t): end of the constant-pitch run of equal pieces starting at order[t]
                auto run2d = [&](size_t t, uint64_t* pitch) -> size_t {
                    const CopyOp& o = c->last_plan[order[t]];
                    const uint64_t len = o.e - o.b;
                    auto same = [&](size_t v) {
                        const CopyOp& x = c->last_plan[order[v]];
                        return x.buf == o.buf && x.src == o.src && x.e - x.b == len;
                    };
                    *pitch = 0;
                    size_t u = t + 1;
                    if (u < order.size() && same(u)) *pitch = c->last_plan[order[u]].b - o.b;
                    if (!*pitch || *pitch > kMaxCopyPitch) return t + 1;
                    while (u < order.size() && same(u) &&
                           c->last_plan[order[u]].b == c->last_plan[order[u - 1]].b + *pitch)
                        ++u;
                    return u;
                };
                std::vector<CopyOp> side_ops;
                for (size_t t = 0; t < order.size();) {
                    const CopyOp& o = c->last_plan[order[t]];
                    if (!c->local(o.src) && !c->ipc) { ++t; continue; }
                    if (!ag_local.empty() && std::binary_search(ag_local.begin(), ag_local.end(), o.buf)) {
                        ++t;  // moved by the all-gather above
                        continue;
                    }
                    if (o.buf == sbuf && (c->stream_same_dev || c->dev[o.src] != c->dev[p])) {
                        side_ops.push_back(o);  // streamed: copied on the side stream under the kernel
                        ++t;
                        continue;
                    }
                    const uint64_t len = o.e - o.b;
                    uint64_t pitch = 0;
                    size_t u = run2d(t, &pitch);
                    const size_t rows = u - t;
                    if (rows == 1) pitch = len;
                    // slabs: equal 2-D runs at a constant slice stride (a 3-D tile's halo
                    // column repeated per plane) become ONE 3-D copy
                    size_t nslab = 1;
                    uint64_t slice = 0, prev = o.b;
                    while (rows > 1 && u < order.size()) {
                        const CopyOp& q = c->last_plan[order[u]];
                        if (q.buf != o.buf || q.src != o.src || q.e - q.b != len) break;
                        uint64_t p2 = 0;
                        const size_t w2 = run2d(u, &p2);
                        if (w2 - u != rows || p2 != pitch) break;
                        const uint64_t st = q.b - prev;
                        if (nslab == 1) {
                            if (st % pitch || st / pitch < rows || st > kMaxCopyPitch) break;
                            slice = st;
                        } else if (st != slice) {
                            break;
                        }
                        prev = q.b;
                        ++nslab;
                        u = w2;
                    }
                    Buffer& B = c->bufs[o.buf];
                    char* dst = (char*)B.inst[p] + o.b;
                    const char* src = (const char*)B.inst[o.src] + o.b;
                    // IPC-mapped peer instances are addressed through UVA (cudaMemcpyDefault)
                    const bool same_dev = c->ipc || c->dev[o.src] == c->dev[p];
                    const cudaMemcpyKind dkind = c->ipc ? cudaMemcpyDefault : cudaMemcpyDeviceToDevice;
                    if ((rows > 1 || nslab > 1) && len <= kNarrowPiece && c->sm_reach(p, o.src)) {
                        // narrow strided run (a halo column): pulled by the destination's SMs
                        PK_CUDA(launch_strided_copy(dst, src, len, pitch, rows, slice, nslab, c->sm_count[p],
                                                    c->stream[p]));
                        c->stats.copy_kernels += 1;
                    } else if (nslab > 1) {
                        const size_t ysz = slice / pitch;
                        if (same_dev) {
                            cudaMemcpy3DParms pp = {};
                            pp.srcPtr = make_cudaPitchedPtr((void*)src, pitch, len, ysz);
                            pp.dstPtr = make_cudaPitchedPtr(dst, pitch, len, ysz);
                            pp.extent = make_cudaExtent(len, rows, nslab);
                            pp.kind = dkind;
                            PK_CUDA(cudaMemcpy3DAsync(&pp, c->stream[p]));
                        } else {
                            cudaMemcpy3DPeerParms pp = {};
                            pp.srcPtr = make_cudaPitchedPtr((void*)src, pitch, len, ysz);
                            pp.dstPtr = make_cudaPitchedPtr(dst, pitch, len, ysz);
                            pp.srcDevice = c->dev[o.src];
                            pp.dstDevice = c->dev[p];
                            pp.extent = make_cudaExtent(len, rows, nslab);
                            PK_CUDA(cudaMemcpy3DPeerAsync(&pp, c->stream[p]));
                        }
                    } else if (rows == 1) {
                        if (same_dev)
                            PK_CUDA(cudaMemcpyAsync(dst, src, len, dkind, c->stream[p]));
                        else
                            PK_CUDA(cudaMemcpyPeerAsync(dst, c->dev[p], src, c->dev[o.src], len, c->stream[p]));
                    } else if (same_dev) {
                        PK_CUDA(cudaMemcpy2DAsync(dst, pitch, src, pitch, len, rows, dkind, c->stream[p]));
                    } else {
                        cudaMemcpy3DPeerParms pp = {};
                        pp.srcPtr = make_cudaPitchedPtr((void*)src, pitch, len, rows);
                        pp.dstPtr = make_cudaPitchedPtr(dst, pitch, len, rows);
                        pp.srcDevice = c->dev[o.src];
                        pp.dstDevice = c->dev[p];
                        pp.extent = make_cudaExtent(len, rows, 1);
                        PK_CUDA(cudaMemcpy3DPeerAsync(&pp, c->stream[p]));
                    }
                    const uint64_t moved = len * rows * nslab;
                    c->stats.copies += 1;
                    c->stats.strided_copies += rows > 1;
                    c->stats.moved_bytes += moved;
                    if (o.src < 16 && p < 16) c->stats.pair_bytes[o.src][p] += moved;
                    t = u;
                }
                if (!side_ops.empty()) {  // records ev_copy[p] on the side stream
                    if (int r = issue_streamed(c, p, sbuf, side_ops, granule, &arrival[p])) return r;
                    side_pending[p] = 1;
                } else {
                    PK_CUDA(cudaEventRecord(c->ev_copy[p], c->stream[p]));
                }
                if (c->ipc)
                    if (int r = ipc_signal(c, p, kFlagCopied, E)) return r;
            }
            // Pass 3: bookkeeping for the hazards of later work (a copy-in is the instance's
            // last writer; the source gains a reader that its next writer must wait for)
            for (const Group& g : groups)
                for (size_t t = g.i; t < g.j; ++t) {
                    const CopyOp& o = c->last_plan[t];
                    if (!c->local(o.src)) continue;
                    Buffer& B = c->bufs[o.buf];
                    B.readers[o.src] |= 1ull << g.p;
                    B.last_writer[g.p] = W_COPY;
                }
            // SPMD: copies between ranks are NCCL send/recv pairs issued in the
            // global plan order on both sides (one partition per rank, so stream
            // order on that partition covers RAW and both WARs).
            if (c->ipc) {
                // replicated bookkeeping (every rank, every partition): WAR entries of the
                // destinations are consumed, then this launch's reads and copy-writes recorded
                for (const CopyOp& o : c->last_plan) {
                    Buffer& B = c->bufs[o.buf];
                    std::fill(B.ep_read.begin() + (size_t)o.dst * P, B.ep_read.begin() + (size_t)(o.dst + 1) * P, 0ull);
                }
                for (const CopyOp& o : c->last_plan) {
                    Buffer& B = c->bufs[o.buf];
                    B.ep_read[(size_t)o.src * P + o.dst] = E;
                    B.ep_mod[o.dst] = E;
                    B.ep_kind[o.dst] = W_COPY;
                }
            } else if (c->world > 1) {
                const NcclApi& n = nccl();
                bool open = false;
                // whole-buffer reads: one in-place ncclAllGather each (NVLS multicast on NVSwitch)
                for (int64_t b : ag_bufs) {
                    Buffer& B = c->bufs[b];
                    const int me = c->first_local;
                    const uint64_t slab = B.bytes / c->P;
                    if (!open) {
                        if (int r = c->set_device(c->dev[me])) return r;
                        n.GroupStart();
                        open = true;
                    }
                    int r = n.AllGather((const char*)B.inst[me] + (uint64_t)me * slab, B.inst[me], slab, kNcclUint8,
                                        c->comm, c->stream[me]);
                    if (r) { n.GroupEnd(); return fail(PK_ERR_NCCL, std::string("ncclAllGather: ") + n.GetErrorString(r)); }
                    c->stats.copies += P - 1;
                    c->stats.moved_bytes += (uint64_t)(P - 1) * slab;
                    for (int q = 0; q < P && q < 16; ++q)
                        if (q != me && me < 16) c->stats.pair_bytes[q][me] += slab;
                }
                for (const CopyOp& o : c->last_plan) {
                    const bool sl = c->local(o.src), dl = c->local(o.dst);
                    if (sl == dl) continue;
                    if (std::binary_search(ag_bufs.begin(), ag_bufs.end(), o.buf)) continue;
                    if (!open) {
                        if (int r = c->set_device(c->dev[c->first_local])) return r;
                        n.GroupStart();
                        open = true;
                    }
                    Buffer& B = c->bufs[o.buf];
                    int r;
                    if (sl)
                        r = n.Send((const char*)B.inst[o.src] + o.b, o.e - o.b, kNcclUint8, c->prank[o.dst], c->comm,
                                   c->stream[o.src]);
                    else
                        r = n.Recv((char*)B.inst[o.dst] + o.b, o.e - o.b, kNcclUint8, c->prank[o.src], c->comm,
                                   c->stream[o.dst]);
                    if (r) { n.GroupEnd(); return fail(PK_ERR_NCCL, std::string("ncclSend/Recv: ") + n.GetErrorString(r)); }
                    if (dl) {
                        c->stats.copies += 1;
                        c->stats.moved_bytes += o.e - o.b;
                        if (o.src < 16 && o.dst < 16) c->stats.pair_bytes[o.src][o.dst] += o.e - o.b;
                    }
                }
                if (open) {
                    int r = n.GroupEnd();
                    if (r) return fail(PK_ERR_NCCL, std::string("ncclGroupEnd: ") + n.GetErrorString(r));
                }
            }
        }
        if (mode & PK_MODE_GLOBAL_BARRIER) {  // Fig. 4 line 8, literally
            if (int r = pk_synchronize(c)) return r;
            if (c->ipc) {
                if (int r = ipc_barrier(c)) return r;
                ipc_settle(c);
            }
        }
    }
    uint64_t t4 = now_ns();
    nv.next("pk a6 partitioned launches");
    const bool time_k = (mode & PK_MODE_TIME_KERNELS) && !c->capturing;

    // ---- a6: partitioned launches (Eq. 8-10) ----
    bool writes_arg[PK_MAX_ARGS] = {};
    for (int a = 0; a < K.nargs; ++a)
        for (const Tap& t : K.taps)
            if (t.arg == a && t.mode != PK_READ) writes_arg[a] = true;
    if (!c->host_only) {
        // Push hazards, enqueued before ANY kernel of this launch so that ev_kernel[*] still
        // names the previous launch's kernels (no false serialisation within a launch):
        //   RAW  p's kernel reads bytes an earlier kernel of q pushed into (b,p);
        //   WAR  q's kernel pushes into (b,p): p's previous kernel and the copies that read
        //        (b,p) must be done.
        for (int p = 0; p < P; ++p) {
            if ((*regs)[p].empty || !c->local(p)) continue;
            if (int r = c->set_device(c->dev[p])) return r;
            FlagWaits fw(c->ipc ? P : 0);
            for (int a = 0; a < K.nargs; ++a) {
                if (!bound[a]) continue;
                const Buffer& B = c->bufs[bid[a]];
                if (c->ipc) {
                    for (int q = 0; q < P; ++q)
                        if (B.ep_push[(size_t)p * P + q]) fw.add(q, kFlagDone, B.ep_push[(size_t)p * P + q]);
                } else {
                    for (uint64_t m = B.pushers[p]; m; m &= m - 1)
                        PK_CUDA(cudaStreamWaitEvent(c->stream[p], c->ev_kernel[__builtin_ctzll(m)], 0));
                }
            }
            for (const PushRec& pr : pushed) {
                if (pr.q != p) continue;
                const Buffer& B = c->bufs[pr.b];
                if (c->ipc) {
                    if (B.ep_kread[pr.p]) fw.add(pr.p, kFlagDone, B.ep_kread[pr.p]);
                    for (int r = 0; r < P; ++r)
                        if (B.ep_read[(size_t)pr.p * P + r]) fw.add(r, kFlagCopied, B.ep_read[(size_t)pr.p * P + r]);
                } else {
                    if (c->kernel_recorded[pr.p])
                        PK_CUDA(cudaStreamWaitEvent(c->stream[p], c->ev_kernel[pr.p], 0));
                    for (uint64_t m = B.readers[pr.p]; m; m &= m - 1)
                        PK_CUDA(cudaStreamWaitEvent(c->stream[p], c->ev_copy[__builtin_ctzll(m)], 0));
                }
            }
            if (c->ipc)
                if (int r = fw.issue(c, c->stream[p])) return r;
        }
        void* inst[PK_MAX_ARGS];
        void* argv[PK_MAX_ARGS + 1];
        for (int p = 0; p < P; ++p) {
            const Regions& R = (*regs)[p];
            if (R.empty || !c->local(p)) continue;
            if (int r = c->set_device(c->dev[p])) return r;
            if (c->ipc) {
                // WAR across ranks: readers of (b,p) -- this launch's included -- must have
                // finished their copies before p's kernel overwrites b
                FlagWaits fw(P);
                for (int a = 0; a < K.nargs; ++a) {
                    if (!bound[a] || !(writes_arg[a] || !track)) continue;
                    const Buffer& B = c->bufs[bid[a]];
                    for (int r = 0; r < P; ++r)
                        if (B.ep_read[(size_t)p * P + r]) fw.add(r, kFlagCopied, B.ep_read[(size_t)p * P + r]);
                }
                if (int r = fw.issue(c, c->stream[p])) return r;
            }
            // WAR: writes into (b,p) wait for copies that read (b,p)
            if (track) {
                for (auto& bs : sets[p])
                    if (!bs.w.empty() && c->bufs[bs.b].readers[p])
                        if (int r = wait_readers(c, c->bufs[bs.b], p)) return r;
            } else {
                for (int a = 0; a < K.nargs; ++a)
                    if (bound[a] && c->bufs[bid[a]].readers[p])
                        if (int r = wait_readers(c, c->bufs[bid[a]], p)) return r;
            }
            pk_partition part;
            part.min[0] = (int32_t)R.box[4]; part.max[0] = (int32_t)R.box[5];
            part.min[1] = (int32_t)R.box[2]; part.max[1] = (int32_t)R.box[3];
            part.min[2] = (int32_t)R.box[0]; part.max[2] = (int32_t)R.box[1];
            for (int d = 0; d < 3; ++d) part.grid[d] = grid[d];
            for (int a = 0; a < K.nargs; ++a) {
                if (bound[a]) { inst[a] = c->bufs[bid[a]].inst[p]; argv[a] = &inst[a]; }
                else { inst[a] = nullptr; argv[a] = const_cast<void*>(args[a]); }
            }
            argv[K.nargs] = &part;
            dim3 g(part.max[0] - part.min[0], part.max[1] - part.min[1], part.max[2] - part.min[2]);
            dim3 bl(block[0], block[1], block[2]);
            cudaEvent_t e0 = nullptr, e1 = nullptr;
            if (time_k) {
                auto& pool = c->event_pool[p];
                for (cudaEvent_t* e : {&e0, &e1}) {
                    if (!pool.empty()) { *e = pool.back(); pool.pop_back(); }
                    else PK_CUDA(cudaEventCreate(e));
                }
                PK_CUDA(cudaEventRecord(e0, c->stream[p]));
            }
            cudaError_t err;
            if (K.launcher) {
                LaunchInfo li{K.fn, g, bl, smem, c->stream[p], c->dev[p], inst, args, scalars, ns, part,
                              push[p].n ? &push[p] : nullptr, c, p};
                li.arrival = arrival[p];
                err = K.launcher(li);
            } else {
                err = cudaLaunchKernel(K.fn, g, bl, argv, smem, c->stream[p]);
            }
            if (err != cudaSuccess)
                return fail(PK_ERR_CUDA, "launch of '" + K.name + "' on partition " + std::to_string(p) + ": " +
                                             cudaGetErrorName(err) + " (" + cudaGetErrorString(err) + ")");
            if (time_k) {
                PK_CUDA(cudaEventRecord(e1, c->stream[p]));
                c->pending_timing.push_back(TimedLaunch{e0, e1, p, launch_id});
            }
            if (P > 1) {
                PK_CUDA(cudaEventRecord(c->ev_kernel[p], c->stream[p]));
                c->kernel_recorded[p] = 1;
            }
            if (c->ipc)
                if (int r = ipc_signal(c, p, kFlagDone, E)) return r;
            c->stats.kernel_launches += 1;
            for (int a = 0; a < K.nargs; ++a)
                if (bound[a]) {
                    bool writes = false;
                    for (const Tap& t : K.taps)
                        if (t.arg == a && t.mode != PK_READ) writes = true;
                    if (writes || !track) c->bufs[bid[a]].last_writer[p] = (P > 1) ? W_KERNEL : W_NONE;
                }
        }
        // streamed copies rejoin their partition's stream behind its kernel, so everything
        // later on that stream (and a graph's join) is ordered after them
        for (int p = 0; p < P; ++p)
            if (side_pending[p]) {
                if (int r = c->set_device(c->dev[p])) return r;
                PK_CUDA(cudaEventRecord(c->ev_side_done[p], c->side[p]));
                PK_CUDA(cudaStreamWaitEvent(c->stream[p], c->ev_side_done[p], 0));
            }
    } else {
        for (int p = 0; p < P; ++p)
            if (!(*regs)[p].empty && c->local(p)) c->stats.kernel_launches += 1;
    }
    if (c->ipc) {
        // replicated: the kernels' writes consume the WAR entries and become the last writes
        for (int p = 0; p < P; ++p) {
            if ((*regs)[p].empty) continue;
            for (int a = 0; a < K.nargs; ++a) {
                if (!bound[a] || !(writes_arg[a] || !track)) continue;
                Buffer& B = c->bufs[bid[a]];
                std::fill(B.ep_read.begin() + (size_t)p * P, B.ep_read.begin() + (size_t)(p + 1) * P, 0ull);
                B.ep_mod[p] = E;
                B.ep_kind[p] = W_KERNEL;
            }
        }
    }
    uint64_t t5 = now_ns();
    c->stats.host_ns_issue += (t4 - t3) + (t5 - t4);
    nv.next("pk a7 tracker update");

    // ---- a7: tracker update with the write sets, kernels running ----
    if (track)
        for (int p = 0; p < P; ++p)
            for (auto& bs : sets[p])
                if (!bs.w.empty()) c->bufs[bs.b].tracker.assign(bs.w, 1ull << p);
    // pushed bytes are valid on the receiving partition too
    for (const PushRec& pr : pushed) {
        Buffer& B = c->bufs[pr.b];
        B.tracker.add_bit(pr.r, pr.p);
        B.pushers[pr.p] |= 1ull << pr.q;
        if (c->ipc) B.ep_push[(size_t)pr.p * P + pr.q] = E;
        if (c->local(pr.q)) c->stats.pushed_bytes += total_bytes(pr.r);
    }
    // read sets of this launch: the push prediction of the next writer (+ push WAR epochs)
    if (track)
        for (int p = 0; p < P; ++p)
            for (auto& bs : sets[p])
                if (!bs.r.empty()) {
                    Buffer& B = c->bufs[bs.b];
                    B.last_read[p] = bs.r;
                    if (c->ipc) B.ep_kread[p] = E;
                }
    c->stats.host_ns_update += now_ns() - t5;
    return PK_OK;
}

int pk_launch_direct(pk_ctx c, pk_kernel k, const int32_t grid[3], const int32_t block[3], size_t smem,
                     const void* const* args, const int64_t* scalars, int ns) {
    if (!valid_kernel(c, k) || !grid || !block) return fail(PK_ERR_INVALID, "bad argument");
    if (ns < 0 || ns > PK_MAX_SCALARS || (ns && !scalars)) return fail(PK_ERR_INVALID, "bad scalars");
    if (c->host_only || c->P != 1 || c->world != 1)
        return fail(PK_ERR_STATE, "pk_launch_direct: single-partition, single-process device contexts only");
    const Kernel& K = c->kernels[k];
    if (K.nargs && !args) return fail(PK_ERR_INVALID, "null args");
    for (int w = 0; w < 3; ++w)
        if (grid[w] < 0 || block[w] < 1) return fail(PK_ERR_INVALID, "bad grid/block");
    void* inst[PK_MAX_ARGS];
    void* argv[PK_MAX_ARGS + 1];
    for (int a = 0; a < K.nargs; ++a) {
        if (K.kinds[a] == PK_ARG_BUFFER) {
            if (!args[a]) return fail(PK_ERR_INVALID, "null buffer argument");
            const pk_buf b = *(const pk_buf*)args[a];
            if (!valid_buf(c, b)) return fail(PK_ERR_INVALID, "argument " + std::to_string(a) + " is not a live buffer");
            inst[a] = c->bufs[b].inst[0];
            argv[a] = &inst[a];
        } else {
            inst[a] = nullptr;
            argv[a] = const_cast<void*>(args[a]);
        }
    }
    pk_partition part;  // the whole grid: blockIdx' = blockIdx (Eq. 8 with min = 0)
    for (int d = 0; d < 3; ++d) {
        part.min[d] = 0;
        part.max[d] = grid[d];
        part.grid[d] = grid[d];
    }
    argv[K.nargs] = &part;
    if (int r = c->set_device(c->dev[0])) return r;
    const dim3 g(grid[0], grid[1], grid[2]), bl(block[0], block[1], block[2]);
    cudaError_t err;
    if (K.launcher) {
        LaunchInfo li{K.fn, g, bl, smem, c->stream[0], c->dev[0], inst, args, scalars, ns, part, nullptr, c, 0};
        err = K.launcher(li);
    } else {
        err = cudaLaunchKernel(K.fn, g, bl, argv, smem, c->stream[0]);
    }
    if (err != cudaSuccess)
        return fail(PK_ERR_CUDA, "direct launch of '" + K.name + "': " + cudaGetErrorName(err));
    return PK_OK;
}

// ---- access recording (PK_TRACE_ACCESS build) ----
int pk_trace_available(void) {
#ifdef PK_TRACE_ACCESS
    return 1;
#else
    return 0;
#endif
}

int pk_trace_reset(pk_ctx c) {
#ifdef PK_TRACE_ACCESS
    if (!c || c->host_only) return fail(PK_ERR_INVALID, "bad context");
    if (int r = pk_synchronize(c)) return r;
    std::lock_guard<std::mutex> g(g_trace_mu);
    for (const TraceInst& t : g_trace)
        for (int k = 0; k < 2; ++k) PK_CUDA(cudaMemset(t.bits[k], 0, ((t.bytes / 4 + 31) / 32) * 4));
    unsigned long long z = 0;
    PK_CUDA(cudaMemcpyToSymbol(g_pk_trace, &z, sizeof z, offsetof(pk::trace::Table, stray)));
    return PK_OK;
#else
    (void)c;
    return fail(PK_ERR_STATE, "library built without PK_TRACE_ACCESS (load libpk_trace.so)");
#endif
}

int pk_trace_fetch(pk_ctx c, pk_buf b, int part, int kind, uint32_t* words, uint64_t nwords) {
#ifdef PK_TRACE_ACCESS
    if (!valid_buf(c, b) || part < 0 || part >= c->P || kind < 0 || kind > 1 || (nwords && !words))
        return fail(PK_ERR_INVALID, "bad argument");
    if (int r = pk_synchronize(c)) return r;
    const Buffer& B = c->bufs[b];
    std::lock_guard<std::mutex> g(g_trace_mu);
    for (const TraceInst& t : g_trace)
        if (t.base == B.inst[part]) {
            const uint64_t n = (t.bytes / 4 + 31) / 32;
            if (nwords < n) return fail(PK_ERR_INVALID, "bitmap needs " + std::to_string(n) + " words");
            PK_CUDA(cudaMemcpy(words, t.bits[kind], n * 4, cudaMemcpyDeviceToHost));
            return PK_OK;
        }
    return fail(PK_ERR_STATE, "instance is not traced");
#else
    (void)c; (void)b; (void)part; (void)kind; (void)words; (void)nwords;
    return fail(PK_ERR_STATE, "library built without PK_TRACE_ACCESS (load libpk_trace.so)");
#endif
}

int pk_trace_stray(pk_ctx c, uint64_t* out) {
#ifdef PK_TRACE_ACCESS
    if (!c || !out) return fail(PK_ERR_INVALID, "bad argument");
    if (int r = pk_synchronize(c)) return r;
    unsigned long long v = 0;
    PK_CUDA(cudaMemcpyFromSymbol(&v, g_pk_trace, sizeof v, offsetof(pk::trace::Table, stray)));
    *out = v;
    return PK_OK;
#else
    (void)c; (void)out;
    return fail(PK_ERR_STATE, "library built without PK_TRACE_ACCESS (load libpk_trace.so)");
#endif
}

}  // extern "C"

namespace pk {
void* context_scratch(const LaunchInfo& li, int slot, size_t bytes, cudaError_t* err) {
    pk_ctx c = li.ctx;
    *err = cudaSuccess;
    if (!c || li.part_index < 0 || li.part_index >= c->P || slot < 0 || slot >= kScratchSlots) {
        *err = cudaErrorInvalidValue;
        return nullptr;
    }
    if (c->scratch.size() != (size_t)c->P) c->scratch.resize(c->P);
    auto& s = c->scratch[li.part_index][slot];
    if (s.second >= bytes && s.first) return s.first;
    void* p = nullptr;
    // the runtime has selected the partition's device before calling the launcher
    *err = cudaMalloc(&p, bytes ? bytes : 16);
    if (*err != cudaSuccess) return nullptr;
    if (s.first) c->scratch_retired.push_back({c->dev[li.part_index], s.first});
    s = {p, bytes};
    return p;
}

// the one registry of builtin kernels (kernels/*.cu)
static const Builtin* const kAllBuiltins[] = {
    &kBuiltinJacobi2d,     &kBuiltinJacobi2dTb,   &kBuiltinHotspot2dTma, &kBuiltinHotspot2d, &kBuiltinHotspot2dTb2, &kBuiltinHotspot2dTbk,
    &kBuiltinHeat3dTma,    &kBuiltinHeat3d,       &kBuiltinHeat3dTb2, &kBuiltinHeat3dTb3,    &kBuiltinNbody,
    &kBuiltinSgemm};

const Builtin* find_builtin_by_fn(const void* fn) {
    if (!fn) return nullptr;
    for (const Builtin* b : kAllBuiltins)
        if (b->fn == fn) return b;
    return nullptr;
}
int32_t find_builtin_push_arg(const void* fn) {
    const Builtin* b = find_builtin_by_fn(fn);
    return b ? b->push_arg : -1;
}
LauncherFn find_builtin_launcher(const void* fn) {
    const Builtin* b = find_builtin_by_fn(fn);
    return b ? b->launcher : nullptr;
}
const Builtin* find_builtin(const char* name) {
    if (!name) return nullptr;
    for (const Builtin* b : kAllBuiltins)
        if (std::strcmp(b->name, name) == 0) return b;
    return nullptr;
}
}  // namespace pk
