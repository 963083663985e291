/*
 * pk_api.h -- C-ABI of the B200-native partitioned-kernel runtime ("pk").
 *
 * Hot path of Matz, Doerfert, Fröning, "Automated Partitioning of Data-Parallel
 * Kernels using Polyhedral Compilation" (ICPP Workshops 2020).  Citations
 * "P:Lnnn" are lines of /root/reference/PAPER.md (the paper's text) plus the
 * section / equation / figure they fall in.
 *
 * One regular, affine-access CUDA kernel has its grid split along thread-block
 * boundaries into P partitions (§5 task (1), §7 Eq. 8-10).
 * Before each launch the read/write regions of every partition are computed
 * from declared affine access descriptors (replacing the paper's polyhedral
 * analysis, §4, and its generated enumerators, §6), a
 * per-buffer validity map finds the stale ranges (§8.1,
 * P:L914-936 §8.3) and only those move between device instances before the
 * sub-grids launch (Fig. 4).
 *
 * Conventions
 *  - Every entry point returns an int status: PK_OK (0) or a negative PK_ERR_*.
 *    No C++ exception crosses the ABI.  A thread-local message describing the
 *    last failure is returned by pk_last_error().
 *  - Plain pointers and sizes only; no torch or CUDA types in the signatures.
 *    "device pointer" = a CUDA global-memory address valid on the partition's
 *    device; "host pointer" = ordinary process memory (pinned or pageable).
 *  - A context is used from one host thread at a time, like the paper's single
 *    rewritten host program (§8.4).
 *  - Integer parameters of descriptors and enumerators are int64 arrays, as in
 *    the paper's enumerator interface (§6.2).
 *  - Grid/block triples are ordered (x, y, z) like CUDA's dim3; partition
 *    6-tuples are ordered (zmin, zmax, ymin, ymax, xmin, xmax) like the paper's
 *    (§7, §6.2), half-open, in thread blocks.
 */
#ifndef PK_API_H
#define PK_API_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ------------------------------------------------------------------ status */
enum {
    PK_OK = 0,
    PK_ERR_INVALID = -1,        /* bad argument / handle / descriptor */
    PK_ERR_CUDA = -2,           /* a CUDA runtime call failed (message has the cudaError name) */
    PK_ERR_NCCL = -3,           /* reserved: NCCL transport */
    PK_ERR_OOM = -4,            /* device or host allocation failed */
    PK_ERR_OUT_OF_BOUNDS = -5,  /* an unclamped access leaves [0, shape) */
    PK_ERR_WRITE_OVERLAP = -6,  /* two partitions write the same byte: WAW, §4.1 */
    PK_ERR_OVERFLOW = -7,       /* int64 overflow in region arithmetic (P:L405-407 ignores it; we check) */
    PK_ERR_STATE = -8           /* call not valid in the context's current state/mode */
};

/* ------------------------------------------------------------------ handles */
typedef struct pk_ctx_s* pk_ctx;
typedef int64_t pk_buf;     /* virtual buffer id (§8.1) */
typedef int64_t pk_kernel;  /* kernel model record id (§4.1) */

#define PK_MAX_PARTS 64     /* validity masks are 64-bit */
#define PK_MAX_DIMS 4       /* array dimensions per descriptor */
#define PK_MAX_SCALARS 8    /* int64 scalar arguments visible to descriptors */
#define PK_MAX_ARGS 16      /* kernel arguments */

/* ---------------------------------------------------------------- init */
enum {
    PK_INIT_HOST_ONLY = 1u << 0  /* no CUDA call at all: partitioning, regions, tracker and
                                    transfer planning run, nothing is allocated, copied or
                                    launched.  For host-side tests and planning. */
};

typedef struct {
    int32_t nparts;              /* P, 1..PK_MAX_PARTS: partitions = virtual devices (§8.3:
                                    "each partition corresponds to exactly one GPU", P:L919-920;
                                    here several partitions may share one physical GPU) */
    int32_t my_rank;             /* SPMD process rank (0 for the single-process model) */
    int32_t world_size;          /* number of processes (1 = one host process drives every GPU) */
    uint32_t flags;              /* PK_INIT_* */
    const int32_t* part_device;  /* [nparts] CUDA ordinal of each partition's device on its rank;
                                    NULL = partition p on device p % cudaGetDeviceCount() */
    const int32_t* part_rank;    /* [nparts] owning rank; NULL = all partitions on rank 0 */
} pk_init_params;

/* Create a context: per-partition streams and events, peer access between every
 * pair of distinct devices (P:L927-929 copies "from its most recently written to
 * GPU").  Ownership: the context owns its streams/events; *out is released by
 * pk_finalize.  Errors: PK_ERR_INVALID (bad params), PK_ERR_CUDA. */
int pk_init(const pk_init_params* params, pk_ctx* out);
int pk_finalize(pk_ctx ctx);

/* ---- multi-process SPMD (one process per GPU) ----
 * Every rank runs the same host program and calls the same pk_* sequence, so the
 * partitioning, regions, tracker and transfer plan are computed identically
 * (replicated, deterministic) on every rank; a rank executes only the kernels of
 * the partitions it owns (part_rank[p] == my_rank) and its side of each copy.
 * Copies between partitions of different ranks are NCCL send/recv pairs on the
 * owning partitions' streams (NCCL is loaded at run time from libnccl.so.2); when
 * a launch's plan for a buffer is exactly "every partition reads the whole buffer
 * and partition q holds the q-th of P equal linear slabs" (N-body positions every
 * step, GEMM B), that buffer moves as ONE in-place ncclAllGather instead
 * (pk_stats.collectives; NVLS multicast on NVSwitch).
 * Execution requires exactly one partition per rank; host-only contexts accept
 * any mapping (planning / tests).
 * pk_nccl_unique_id writes the 128-byte ncclUniqueId (rank 0 creates it, the
 * caller broadcasts it, e.g. with torch.distributed); pk_init_spmd is pk_init
 * plus that id (ignored for host-only contexts; may be NULL then).
 * pk_sync_to_host is collective in SPMD mode: rank 0 receives every segment it
 * does not hold and writes `host`; other ranks may pass host = NULL.
 * Errors: PK_ERR_NCCL (library missing or an NCCL call failed), PK_ERR_STATE. */
int pk_nccl_unique_id(void* out, size_t bytes);
int pk_init_spmd(const pk_init_params* params, const void* nccl_unique_id, pk_ctx* out);

/* ---- multi-process SPMD over peer memory (CUDA IPC; no NCCL on the data path) ----
 * Same replicated model as pk_init_spmd, but every rank maps every other rank's
 * buffer instances into its own address space (cudaIpcGetMemHandle /
 * cudaIpcOpenMemHandle, exchanged at pk_register_buffer) and PULLS its stale
 * ranges itself, straight out of the holder's instance over NVLink/NVSwitch
 * (copy engine, or the SM halo-copy kernel for narrow strided runs) -- the
 * paper's "copy from the GPU it was most recently written to",
 * one process per GPU.  Ordering across processes replaces the global barrier
 * of Fig. 4 l. 8 by device-side epoch flags in peer memory: every rank
 * owns two monotone 64-bit words (incoming copies of launch E done / kernel of
 * launch E done) written by cuStreamWriteValue64 on its stream; a reader waits
 * (cuStreamWaitValue64, GEQ) for the holder's word before copying (RAW), a
 * writer waits for the readers' words before overwriting what they read (WAR).
 * The host thread never blocks on another rank inside pk_launch_partitioned.
 *
 * `allgather` is the caller's host all-gather (e.g. torch.distributed over gloo):
 * every rank passes `bytes` bytes at `send`; on return `recv` holds world_size *
 * bytes, rank r's contribution at offset r * bytes; it returns 0 on success.  The
 * library calls it (identically on every rank) inside pk_init_spmd_ipc,
 * pk_register_buffer, pk_unregister_buffer, pk_copy_from_host(_for),
 * pk_sync_to_host and pk_finalize, which are therefore collective in this mode.
 * `user` is passed back unchanged; callback and user must outlive the context.
 * Execution requires exactly one partition per rank; ranks may share a GPU
 * (functional testing on one device).  Caller-owned instances must come from
 * cudaMalloc'd allocations (IPC handles cover whole allocations; the offset is
 * exchanged too).  Errors: PK_ERR_STATE, PK_ERR_CUDA, PK_ERR_INVALID (callback
 * failed or missing). */
typedef int (*pk_host_allgather_fn)(void* user, const void* send, void* recv, size_t bytes);
int pk_init_spmd_ipc(const pk_init_params* params, pk_host_allgather_fn allgather, void* user, pk_ctx* out);

/* ---------------------------------------------------------------- buffers */
/* Virtual buffer = one full-size device instance per partition + a tracker
 * (§8.1; full-size instances keep the kernels' global indices, reading
 * Q13).  Row-major array of `ndim` (1..4) dims `shape[0..ndim)` (slowest first) of
 * `elem_bytes`-byte elements.
 *   dev_ptrs  == NULL: the library cudaMallocs and owns every instance.
 *   dev_ptrs  != NULL: [nparts] caller-owned device pointers (e.g. torch tensors),
 *                      16-byte aligned, which must outlive the registration.
 *   host_init == NULL: contents undefined -> valid on every partition (reading Q3).
 *   host_init != NULL: H2D 1:n linear distribution of the host array (P:L881-895
 *                      §8.2, reading Q2); blocking with respect to host memory.
 * Errors: PK_ERR_INVALID, PK_ERR_OOM, PK_ERR_CUDA. */
int pk_register_buffer(pk_ctx ctx, int ndim, const int64_t* shape, int elem_bytes,
                       void* const* dev_ptrs, const void* host_init, pk_buf* out);
/* cudaMemcpy(HostToDevice) replacement: 1:n linear distribution.
 * `bytes` must equal the buffer size.  Returns after the copies completed. */
int pk_copy_from_host(pk_ctx ctx, pk_buf buf, const void* host, size_t bytes);
/* cudaMemcpy(DeviceToHost) replacement: n:1 gather, one copy per tracker segment
 * from a partition holding it (§8.2).  Blocking. */
int pk_sync_to_host(pk_ctx ctx, pk_buf buf, void* host, size_t bytes);
/* Asynchronous variants (cudaMemcpyAsync replacements, same distribution and tracker
 * effect): the copies are enqueued on the partition streams, ordered by the same
 * stream/event hazards as the transfers of pk_launch_partitioned, and the call returns
 * without waiting.  The host buffer must stay valid (and, for overlap, pinned) until
 * pk_synchronize; a D2H result is complete only then.  Lets a caller pipeline steps:
 * the H2D of step i+1 (one context) overlaps the kernels and the D2H of step i (another
 * context), the host link being full duplex.  In SPMD contexts (and, for the D2H, with
 * PK_MODE_PUSH) they behave like the blocking calls.  Host-only contexts: tracker
 * effect only, like pk_copy_from_host. */
int pk_copy_from_host_async(pk_ctx ctx, pk_buf buf, const void* host, size_t bytes);
int pk_sync_to_host_async(pk_ctx ctx, pk_buf buf, void* host, size_t bytes);
/* Read-pattern-aware H2D (the paper's linear distribution is
 * "hoping that this pattern matches the read pattern of the following kernels",
 * P:L888-895, and its mismatch limits Matmul scaling): every
 * partition receives, straight from the host, the bytes its partition of the
 * given launch (kernel, grid, block, scalars) reads through argument `arg_index`;
 * bytes nobody reads go linearly as in pk_copy_from_host.  Partitions that
 * receive the same bytes all become holders.  Blocking w.r.t. host memory. */
int pk_copy_from_host_for(pk_ctx ctx, pk_buf buf, const void* host, size_t bytes, pk_kernel k, int arg_index,
                          const int32_t grid[3], const int32_t block[3], const int64_t* scalars, int nscalars);
/* cudaFree replacement.  Library-owned instances are freed after pending work. */
int pk_unregister_buffer(pk_ctx ctx, pk_buf buf);
/* Device pointer of partition `part`'s instance (tests / caller-side kernels). */
int pk_buffer_instance(pk_ctx ctx, pk_buf buf, int part, void** dev_ptr);

/* ---------------------------------------------------------------- descriptors */
/* Affine expression in the kernel's int64 scalar arguments and the launch's
 * blockDim (the paper's blockOff = blockIdx * blockDim trick, §4.1
 * Eq. 5-7, keeps descriptors affine in blockIdx):
 *   value = c0 + sum_s c_scalar[s] * scalars[s] + sum_w c_blockdim[w] * blockDim[w] */
typedef struct {
    int64_t c0;
    int64_t c_scalar[PK_MAX_SCALARS];
    int64_t c_blockdim[3];
} pk_expr;

enum { PK_DIM_CLAMP = 1u << 0, PK_DIM_GUARD = 1u << 1 };

/* One array dimension of one access "tap".  For a partition whose block range
 * along grid dimension `grid_dim` (0=x 1=y 2=z) is [m, M):
 *   Pos = U_{b in [m,M)} [b*scale, b*scale + extent)      (grid_dim >= 0)
 *   Pos = [0, extent)                                      (grid_dim == -1: all blocks
 *                                                           touch the same positions)
 *   if PK_DIM_GUARD: Pos = Pos n [guard_lo, guard_hi)      (the kernel's bounds test)
 *   Idx = { p + offset : p in Pos }, then
 *   if PK_DIM_CLAMP: each index clamped to [0, shape-1]    (replicate borders)
 *   else: every index must lie in [0, shape) or the call fails PK_ERR_OUT_OF_BOUNDS.
 * This is the paper's block-granular access map (threadId projected out under
 * 0 <= threadId < blockDim, §4.1) restricted to separable boxes. */
typedef struct {
    int32_t grid_dim;
    uint32_t flags;              /* PK_DIM_* */
    pk_expr scale, extent, guard_lo, guard_hi, offset;
} pk_dim_map;

/* One tap = the product of its per-dimension index sets (exact because a grid
 * dimension may drive at most one array dimension of a tap; otherwise
 * PK_ERR_INVALID).  Several taps of one (arg, mode) are unioned exactly, which is
 * the per-convex-piece enumeration of P:L773-775 §6.1 (no union over-approximation). */
typedef struct {
    int32_t ndim;                /* must equal the bound buffer's ndim */
    int32_t reserved;
    pk_dim_map dim[PK_MAX_DIMS]; /* dim[0] = slowest (row-major) */
} pk_affine_access;

enum { PK_READ = 1, PK_WRITE = 2, PK_MAY_WRITE = 3 };   /* PK_MAY_WRITE = read + write (reading Q6) */

/* ---------------------------------------------------------------- kernels */
enum { PK_ARG_BUFFER = 1, PK_ARG_SCALAR = 2 };

/* Passed BY VALUE as the kernel's last argument (§7): the kernel
 * computes blockIdx' = min + blockIdx (Eq. 8) and must read the full grid from
 * `grid` instead of gridDim (Eq. 9, reading Q10).  Index 0=x, 1=y, 2=z. */
typedef struct {
    int32_t min[3];
    int32_t max[3];
    int32_t grid[3];
} pk_partition;

/* Kernel model record (name, suggested partitioning strategy,
 * per-argument maps).  `fn` is a __global__ function of this library's CUDA
 * runtime (see pk_builtin_fn) launched with cudaLaunchKernel; arguments are the
 * kernel's own followed by a pk_partition.  arg_kind[nargs] = PK_ARG_*.
 * partition_dim: 0/1/2 forces x/y/z, -1 = slowest grid dim > 1 (reading Q1). */
int pk_register_kernel(pk_ctx ctx, const char* name, const void* fn, int nargs,
                       const int32_t* arg_kind, int32_t partition_dim, pk_kernel* out);
/* Add one access tap for argument `arg_index` with `mode` (PK_READ / PK_WRITE /
 * PK_MAY_WRITE).  Taps accumulate (union).  Write taps must be exact and
 * injective; read taps may over-approximate. */
int pk_declare_affine_access(pk_ctx ctx, pk_kernel k, int arg_index, int mode,
                             const pk_affine_access* tap);
/* Register one of the library's sm_100a kernels with its descriptors already declared:
 * "jacobi2d", "jacobi2d_tb" (K sweeps per launch, scalar 2), "hotspot2d",
 * "hotspot2d_regs", "hotspot2d_tb2", "hotspot2d_tbk" (K sweeps, scalar 3), "heat3d",
 * "heat3d_regs", "heat3d_tb2", "heat3d_tb3" (two / three sweeps per launch), "nbody",
 * "sgemm_tf32x3".  Launch geometry per kernel: DESIGN.md §4 and kernels.py. */
int pk_builtin_kernel(pk_ctx ctx, const char* name, pk_kernel* out);
/* __global__ entry of a builtin kernel, for pk_register_kernel + user-declared
 * descriptors.  NULL if unknown. */
const void* pk_builtin_fn(const char* name);

/* The kernel-launch replacement of Fig. 4:
 *   (1) partition the grid,  (2) synchronise every read buffer: stale
 *   ranges of each partition's read set are copied from a holder,
 *   (3) launch every partition with grid' = max - min (Eq. 10) on its device,
 *   (4) update the trackers with the write sets, on the host while
 *   the kernels run.
 * grid/block: the ORIGINAL single-device launch (x, y, z).  args[nargs]: for a
 * buffer argument a pointer to its pk_buf, for a scalar a pointer to its value
 * (copied at launch).  scalars[nscalars]: int64 scalar values the descriptors
 * use.  Asynchronous like <<<>>>: faults surface at pk_synchronize.
 * Errors: PK_ERR_INVALID, PK_ERR_OUT_OF_BOUNDS, PK_ERR_WRITE_OVERLAP (nothing is
 * launched), PK_ERR_OVERFLOW, PK_ERR_CUDA. */
int pk_launch_partitioned(pk_ctx ctx, pk_kernel k, const int32_t grid[3],
                          const int32_t block[3], size_t smem_bytes,
                          const void* const* args, const int64_t* scalars, int nscalars);
/* A sequence of partitioned launches (an inner loop of a host program: the C1
 * Jacobi sweeps, the Hotspot time steps), issued as ONE unit.  The result is
 * exactly that of n pk_launch_partitioned calls in order -- every launch still
 * partitions, resolves its stale ranges and updates the trackers (Fig. 4,
 * P:L616-666) -- but in steady state the whole sequence is memoised as one
 * multi-stream CUDA graph: the first call with a given (launch list, pre-launch
 * tracker state) runs eagerly, the second is captured, later ones replay it with
 * a single graph launch and restore the recorded tracker states.  For launch-bound
 * loops (microsecond kernels) this removes the per-launch host and launch
 * latency; it does not change what moves.  Each descriptor is one
 * pk_launch_partitioned argument list (args / scalars are read during the call).
 * n <= PK_MAX_SEQUENCE.  Errors: those of pk_launch_partitioned; launches before a
 * failing one stay issued. */
#define PK_MAX_SEQUENCE 1024
typedef struct pk_launch_desc {
    pk_kernel kernel;
    int32_t grid[3];
    int32_t block[3];
    size_t smem_bytes;
    const void* const* args;
    const int64_t* scalars;
    int nscalars;
} pk_launch_desc;
int pk_launch_sequence(pk_ctx ctx, const pk_launch_desc* launches, int n);
/* The ORIGINAL single-GPU launch, for the paper's E3 measurement (§9.2:
 * "slowdown of the partitioned binary on a single GPU"): the kernel's full grid is
 * launched once on partition 0's stream with partition 0's instances -- no partition
 * boxes, regions, tracker, transfers or graph replay.  It neither reads nor updates the
 * validity map, so it is a measurement baseline, not a way to run the method: only for
 * single-partition contexts (PK_ERR_STATE otherwise).  Same arguments and errors as
 * pk_launch_partitioned (PK_ERR_INVALID, PK_ERR_CUDA). */
int pk_launch_direct(pk_ctx ctx, pk_kernel k, const int32_t grid[3], const int32_t block[3], size_t smem_bytes,
                     const void* const* args, const int64_t* scalars, int nscalars);
/* cudaDeviceSynchronize replacement: all partitions' streams (§8.4). */
int pk_synchronize(pk_ctx ctx);
/* Device-side timer over everything the context enqueues between the two calls:
 * begin records an event on partition 0's stream and makes every other stream
 * wait for it; end makes partition 0's stream wait for every stream's tail and
 * records the stop event there, then blocks and returns the elapsed ms (CUDA
 * events, both on partition 0's device).  Not nestable.  PK_ERR_STATE in a
 * host-only context or when end is called without begin. */
int pk_timer_begin(pk_ctx ctx);
int pk_timer_end(pk_ctx ctx, double* elapsed_ms);

/* Tile partitions ("suggested partitioning
 * strategy"): split the grid into tiles[0] x tiles[1] x tiles[2] (x, y, z) block
 * boxes instead of P slabs of one dimension.  Partition p is tile
 * (p % tx, (p / tx) % ty, p / (tx*ty)); each grid dimension d is split like the
 * 1-D rule, [floor(i*G_d/t_d), floor((i+1)*G_d/t_d)).  tx*ty*tz must equal the
 * context's P (PK_ERR_INVALID otherwise); tiles == NULL or {0,0,0} restores the
 * 1-D split.  Halo columns become equal-length byte ranges at a constant pitch:
 * the transfer engine issues each such run (and equal runs repeated at a
 * constant slice stride, 3-D) as ONE copy: pieces up to 256 B by the
 * destination's SMs (halo-copy kernel reading the source through its peer
 * pointer), wider ones by cudaMemcpy2D/3D(Peer)Async (pk_stats.strided_copies,
 * pk_stats.copy_kernels).
 * Applies to later launches (bumps the kernel's descriptor version). */
int pk_set_partition_shape(pk_ctx ctx, pk_kernel k, const int32_t tiles[3]);

/* ---------------------------------------------------------------- introspection */
/* Grid partition p of the kernel's launch (a1), as (zmin,zmax,ymin,ymax,xmin,xmax). */
int pk_partition_grid(pk_ctx ctx, pk_kernel k, const int32_t grid[3], int part,
                      int64_t part_out[6]);
typedef void (*pk_range_cb)(void* user, uint64_t begin_byte, uint64_t end_byte);
/* Enumerator of §6.2: canonical (sorted, disjoint, coalesced) byte
 * ranges of the image of (arg, mode) over the 6-tuple block box `part`, for
 * buffer `buf`'s shape; one callback per range, no allocation visible to the
 * caller.  mode PK_READ includes PK_MAY_WRITE taps, PK_WRITE includes them too. */
int pk_enumerate(pk_ctx ctx, pk_kernel k, int arg_index, int mode, pk_buf buf,
                 const int64_t part[6], const int32_t block[3],
                 const int64_t* scalars, int nscalars, pk_range_cb cb, void* user);
typedef void (*pk_segment_cb)(void* user, uint64_t begin_byte, uint64_t end_byte,
                              uint64_t valid_mask);
/* Tracker state: canonical segments covering the buffer, each with the mask of
 * partitions holding its latest value (paper: owner). */
int pk_tracker_dump(pk_ctx ctx, pk_buf buf, pk_segment_cb cb, void* user);
typedef void (*pk_copy_cb)(void* user, pk_buf buf, int src_part, int dst_part,
                           uint64_t begin_byte, uint64_t end_byte);
/* Copies planned by the most recent pk_launch_partitioned (coalesced, in issue order; after a
 * pk_launch_sequence: those of its last launch). */
int pk_last_plan(pk_ctx ctx, pk_copy_cb cb, void* user);

typedef struct {
    uint64_t launches;           /* pk_launch_partitioned calls */
    uint64_t kernel_launches;    /* partition kernels actually launched */
    uint64_t copies;             /* device-to-device copy operations issued */
    uint64_t stale_bytes;        /* bytes of read sets not valid on the reader */
    uint64_t moved_bytes;        /* bytes actually copied between instances */
    uint64_t h2d_bytes, d2h_bytes;
    uint64_t pair_bytes[16][16]; /* [src][dst] moved bytes, partitions < 16 */
    uint64_t host_ns_partition;  /* host time per phase (a1, a2, a3, issue, a7) */
    uint64_t host_ns_regions;
    uint64_t host_ns_plan;
    uint64_t host_ns_issue;
    uint64_t host_ns_update;
    double kernel_ms;            /* sum over partition kernels (PK_MODE_TIME_KERNELS) */
    double kernel_ms_max_launch; /* per launch: max over partitions, summed */
    uint64_t timed_kernels;      /* kernels included in kernel_ms */
    uint64_t graph_replays;      /* launches served by steady-state graph replay (a replayed sequence counts
                                    each of its launches) */
    uint64_t graph_captures;     /* launches captured into a replay graph */
    uint64_t strided_copies;     /* of `copies`: equal pieces at a constant pitch (2-D / 3-D) */
    uint64_t copy_kernels;       /* of `strided_copies`: narrow runs moved by the SM halo-copy kernel */
    uint64_t pushed_bytes;       /* bytes stored into other partitions' instances by producing kernels (PK_MODE_PUSH) */
    uint64_t collectives;        /* NCCL SPMD: whole-buffer reads moved as one in-place all-gather */
    uint64_t graph_fallbacks;    /* a graph capture / instantiation failed: the launch ran eagerly and the
                                    context stays eager (pk_last_error() keeps the reason) */
    double graph_launch_ms;      /* PK_MODE_TIME_KERNELS with graph replay: CUDA events around each replayed
                                    graph on its stream (copies + partition kernels of its launches) */
    uint64_t timed_graph_launches; /* partitioned launches inside those graphs */
    uint64_t host_cpu_ns;        /* thread CPU time spent inside pk_launch_partitioned / _sequence (excludes time the
                                    thread is descheduled; a driver spinning on a full launch queue still counts) */
    uint64_t streamed_bytes;     /* of moved_bytes: copied on a side stream while the consuming kernel ran */
    uint64_t timed_eager_launches; /* launches whose partition kernels were timed (kernel_ms_max_launch) */
} pk_stats;
int pk_get_stats(pk_ctx ctx, pk_stats* out);   /* drains pending kernel timings */
int pk_reset_stats(pk_ctx ctx);

/* ---------------------------------------------------------------- modes */
enum {
    PK_MODE_SINGLE_OWNER = 1u << 0,  /* paper tracker: one owner, no shared copies */
    PK_MODE_NO_TRANSFERS = 1u << 1,  /* beta of §9.2: resolve + track, do not copy */
    PK_MODE_NO_TRACKING = 1u << 2,   /* gamma of §9.2: no resolution, no tracker, no copies */
    PK_MODE_GLOBAL_BARRIER = 1u << 3,/* literal all_devs_synchronize() between sync and launch (Fig. 4 l. 8) */
    PK_MODE_TIME_KERNELS = 1u << 4,  /* CUDA events around every eagerly launched partition kernel ->
                                        pk_stats.kernel_ms, and around every replayed graph launch ->
                                        pk_stats.graph_launch_ms (graph replay stays on) */
    PK_MODE_NO_GRAPHS = 1u << 5,     /* disable steady-state graph replay (see pk_launch_partitioned) */
    PK_MODE_PUSH = 1u << 6,          /* fused halo push, see below */
    PK_MODE_NO_OVERLAP = 1u << 7,    /* streamed operands are copied before the kernel instead (see below) */
    PK_MODE_NO_COLLECTIVES = 1u << 8 /* one process, P distinct GPUs: whole-buffer reads as peer copies
                                        instead of one ncclAllGather (see below) */
};
/* Whole-buffer reads, one process ("copy the data from its most
 * recently written GPU", P:L999-1004 Matmul's redistribution).  When a launch's plan for a
 * buffer is exactly "linear slab q -> every partition p != q" (N-body positions every step,
 * the GEMM's B operand when it is not streamed) and the P partitions sit on P distinct GPUs,
 * the P(P-1) copies are ONE in-place ncclAllGather over communicators from ncclCommInitAll
 * (created at the first such launch, destroyed by pk_finalize; NVLS multicast on NVSwitch
 * where NCCL picks it), issued on the partitions' streams after the launch's hazard waits.
 * pk_stats.collectives counts them, moved_bytes/copies as the copies they replace.  Not with
 * partitions sharing a GPU (NCCL refuses two ranks on one device) or without libnccl: peer
 * copies.  A context that used a collective launches eagerly from then on (no graph replay). */
/* Streamed operands -- the transfer overlapped with the kernel it feeds (B200 design; the
 * paper synchronises every read before the launch, Fig. 4 l. 2-8).  A builtin may name one
 * input argument it can consume while its copies are in flight (sgemm_tf32x3: B, the
 * operand every row partition reads whole).  Its stale ranges for partition p
 * are then copied on a side stream of p, granule by granule (copy engine: no SM), starting
 * after p's own linear slab, each granule followed by a stream-front-end store of an
 * arrival flag; p's kernel starts right away and its TMA producer polls the flag of a
 * granule before loading it.  The side stream forks from p's stream after every hazard
 * wait (so the copies only wait for data that is ready) and rejoins it behind the kernel.
 * Counted in pk_stats.streamed_bytes (also in moved_bytes).  Single-process contexts;
 * off with PK_MODE_GLOBAL_BARRIER and PK_MODE_NO_OVERLAP.  Only pieces pulled from ANOTHER
 * GPU are streamed (a same-device D2D copy needs SMs the consuming kernel is holding;
 * measured on a B200 it crawls); PK_STREAM_SAME_DEVICE=1 in the environment at pk_init
 * streams virtual partitions' copies too (functional tests on one GPU). */
/* PK_MODE_PUSH -- the transfer fused into the producing kernel (B200 design; the paper
 * only pulls).  For a kernel whose builtin can push its output (jacobi2d,
 * jacobi2d_tb, hotspot2d, hotspot2d_tbk, heat3d, heat3d_tb2, heat3d_tb3), the library
 * predicts that the next reader of the written buffer reads what its last reader read:
 * the bytes partition q writes that partition p read last time (W_q n R_p, at most 16
 * ranges per writer, 4-byte aligned)
 * are stored by q's kernel ALSO into p's instance (peer stores over NVLink/NVSwitch, or
 * an IPC mapping in peer-memory SPMD), and the tracker marks p as a holder, so the next
 * launch finds nothing stale and issues no copy.  A wrong prediction only costs bytes:
 * whatever is still stale is pulled as usual.  Ordering: q's kernel first waits for p's
 * previous kernel and the copies that read (b,p) (WAR); p's kernel and copies out of
 * (b,p) wait for q's kernel (RAW).  Not applied when the buffer is also read by the
 * same launch, in PK_MODE_SINGLE_OWNER (no shared copies), with NO_TRANSFERS/NO_TRACKING,
 * or in NCCL SPMD contexts.  pk_stats.pushed_bytes counts what was pushed; stale_bytes
 * keeps counting what a launch still finds stale. */
/* Steady-state replay: when a launch repeats with the same kernel, bindings, geometry,
 * scalars, mode and pre-launch tracker states of its buffers (e.g. the second sweep of
 * a ping-pong pair), the library captures its copies + partition kernels once into a
 * multi-stream (multi-device) CUDA graph and afterwards replays the graph and restores
 * the memoised post-launch tracker states instead of re-planning and re-issuing every
 * CUDA call -- the host overhead the paper measures as "patterns".
 * Active for single-process contexts (any number of local partitions, P = 1 included), unless
 * PK_MODE_GLOBAL_BARRIER or PK_MODE_NO_GRAPHS is set.  If a capture or instantiation
 * fails, that launch runs eagerly (its bookkeeping rolled back first) and the context
 * stays eager (pk_stats.graph_fallbacks). */
int pk_set_mode(pk_ctx ctx, uint32_t flags);
uint32_t pk_get_mode(pk_ctx ctx);

/* ---------------------------------------------------------------- access recording
 * The paper requires write maps to be exact and lets read maps over-approximate
 * (P:L568-571); tools of the VAST kind clone the kernel to mark the memory it touches
 * (P:L1231-1236).  libpk_trace.so (the same sources built with -DPK_TRACE_ACCESS, see
 * paper_conf_icppw_matzdf20_b200/build.py) records, at 4-byte granularity, every global
 * address each builtin kernel FETCHES (plain loads, and the in-bounds part of every TMA
 * copy -- halo over-fetch included) and every address it STORES, into one bitmap per
 * (instance, kind); bit w of word w/32 stands for bytes [4w, 4w+4) of the instance.
 * Single device; tests only.  In libpk.so these calls fail with PK_ERR_STATE. */
int pk_trace_available(void);                 /* 1 in libpk_trace.so, 0 in libpk.so */
int pk_trace_reset(pk_ctx ctx);               /* synchronise, clear every bitmap and the stray count */
/* kind 0 = fetched, 1 = stored; words[ceil(bytes/4/32)] receives the bitmap of instance
 * `part` of `buf` (synchronises first); PK_ERR_INVALID if nwords is too small. */
int pk_trace_fetch(pk_ctx ctx, pk_buf buf, int part, int kind, uint32_t* words, uint64_t nwords);
/* accesses that hit no registered instance or ran past its end (must be 0) */
int pk_trace_stray(pk_ctx ctx, uint64_t* out);

const char* pk_last_error(void);
const char* pk_version(void);

#ifdef __cplusplus
}
#endif
#endif /* PK_API_H */
