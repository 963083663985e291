"""Thin ctypes binding of include/pk_api.h -- same names, argument marshalling only.

Every step of the hot path runs inside libpk.so (host C++ + sm_100a kernels).
If the library is missing this module raises at import of ``lib()``: there is no
Python or CPU fallback.  Build it with ``python -m paper_conf_icppw_matzdf20_b200.build``.
"""
from __future__ import annotations

import ctypes as C
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
# PK_TRACE_ACCESS=1 selects the access-recording build libpk_trace.so (tests of the
# declared descriptors against what the kernels touch; pk_trace_* below)
LIB_PATH = os.path.join(_HERE, "libpk_trace.so" if os.environ.get("PK_TRACE_ACCESS") == "1" else "libpk.so")
LIB_PATH = os.environ.get("PK_LIB_OVERRIDE") or LIB_PATH   # A/B measurements of an older build only

PK_OK = 0
PK_ERR = {-1: "PK_ERR_INVALID", -2: "PK_ERR_CUDA", -3: "PK_ERR_NCCL", -4: "PK_ERR_OOM",
          -5: "PK_ERR_OUT_OF_BOUNDS", -6: "PK_ERR_WRITE_OVERLAP", -7: "PK_ERR_OVERFLOW",
          -8: "PK_ERR_STATE"}
PK_INIT_HOST_ONLY = 1
PK_MAX_PARTS, PK_MAX_DIMS, PK_MAX_SCALARS, PK_MAX_ARGS = 64, 4, 8, 16
PK_DIM_CLAMP, PK_DIM_GUARD = 1, 2
PK_READ, PK_WRITE, PK_MAY_WRITE = 1, 2, 3
PK_ARG_BUFFER, PK_ARG_SCALAR = 1, 2
PK_MODE_SINGLE_OWNER = 1 << 0
PK_MODE_NO_TRANSFERS = 1 << 1
PK_MODE_NO_TRACKING = 1 << 2
PK_MODE_GLOBAL_BARRIER = 1 << 3
PK_MODE_TIME_KERNELS = 1 << 4
PK_MODE_NO_GRAPHS = 1 << 5
PK_MODE_PUSH = 1 << 6
PK_MODE_NO_OVERLAP = 1 << 7
PK_MODE_NO_COLLECTIVES = 1 << 8


class PkError(RuntimeError):
    def __init__(self, code, where, msg):
        self.code = code
        self.name = PK_ERR.get(code, str(code))
        super().__init__(f"{where}: {self.name}: {msg}")


# ------------------------------------------------------------------ structs
class pk_init_params(C.Structure):
    _fields_ = [("nparts", C.c_int32), ("my_rank", C.c_int32), ("world_size", C.c_int32),
                ("flags", C.c_uint32), ("part_device", C.POINTER(C.c_int32)),
                ("part_rank", C.POINTER(C.c_int32))]


class pk_expr(C.Structure):
    _fields_ = [("c0", C.c_int64), ("c_scalar", C.c_int64 * PK_MAX_SCALARS),
                ("c_blockdim", C.c_int64 * 3)]


class pk_dim_map(C.Structure):
    _fields_ = [("grid_dim", C.c_int32), ("flags", C.c_uint32), ("scale", pk_expr),
                ("extent", pk_expr), ("guard_lo", pk_expr), ("guard_hi", pk_expr),
                ("offset", pk_expr)]


class pk_affine_access(C.Structure):
    _fields_ = [("ndim", C.c_int32), ("reserved", C.c_int32), ("dim", pk_dim_map * PK_MAX_DIMS)]


class pk_partition(C.Structure):
    _fields_ = [("min", C.c_int32 * 3), ("max", C.c_int32 * 3), ("grid", C.c_int32 * 3)]


class pk_stats(C.Structure):
    _fields_ = [("launches", C.c_uint64), ("kernel_launches", C.c_uint64), ("copies", C.c_uint64),
                ("stale_bytes", C.c_uint64), ("moved_bytes", C.c_uint64), ("h2d_bytes", C.c_uint64),
                ("d2h_bytes", C.c_uint64), ("pair_bytes", (C.c_uint64 * 16) * 16),
                ("host_ns_partition", C.c_uint64), ("host_ns_regions", C.c_uint64),
                ("host_ns_plan", C.c_uint64), ("host_ns_issue", C.c_uint64),
                ("host_ns_update", C.c_uint64), ("kernel_ms", C.c_double),
                ("kernel_ms_max_launch", C.c_double), ("timed_kernels", C.c_uint64),
                ("graph_replays", C.c_uint64), ("graph_captures", C.c_uint64),
                ("strided_copies", C.c_uint64), ("copy_kernels", C.c_uint64), ("pushed_bytes", C.c_uint64),
                ("collectives", C.c_uint64), ("graph_fallbacks", C.c_uint64),
                ("graph_launch_ms", C.c_double), ("timed_graph_launches", C.c_uint64), ("host_cpu_ns", C.c_uint64),
                ("streamed_bytes", C.c_uint64), ("timed_eager_launches", C.c_uint64)]


RANGE_CB = C.CFUNCTYPE(None, C.c_void_p, C.c_uint64, C.c_uint64)
SEGMENT_CB = C.CFUNCTYPE(None, C.c_void_p, C.c_uint64, C.c_uint64, C.c_uint64)
COPY_CB = C.CFUNCTYPE(None, C.c_void_p, C.c_int64, C.c_int, C.c_int, C.c_uint64, C.c_uint64)
ALLGATHER_CB = C.CFUNCTYPE(C.c_int, C.c_void_p, C.c_void_p, C.c_void_p, C.c_size_t)
_keepalive = {}   # ctx address -> ctypes callback of pk_init_spmd_ipc (must outlive the context)

_lib = None
_I64P = C.POINTER(C.c_int64)
_I32P = C.POINTER(C.c_int32)


def lib():
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(f"{LIB_PATH} is missing: build the CUDA extension first "
                           "(python -m paper_conf_icppw_matzdf20_b200.build); there is no fallback")
    if "PK_NCCL_LIB" not in os.environ:      # NCCL is dlopen'ed only by SPMD contexts
        try:
            import importlib.util
            spec = importlib.util.find_spec("nvidia")
            for base in (spec.submodule_search_locations or []) if spec else []:
                cand = os.path.join(base, "nccl", "lib", "libnccl.so.2")
                if os.path.exists(cand):
                    os.environ["PK_NCCL_LIB"] = cand
                    break
        except Exception:
            pass
    L = C.CDLL(LIB_PATH)
    sig = {
        "pk_init": [C.POINTER(pk_init_params), C.POINTER(C.c_void_p)],
        "pk_init_spmd": [C.POINTER(pk_init_params), C.c_void_p, C.POINTER(C.c_void_p)],
        "pk_nccl_unique_id": [C.c_void_p, C.c_size_t],
        "pk_init_spmd_ipc": [C.POINTER(pk_init_params), ALLGATHER_CB, C.c_void_p, C.POINTER(C.c_void_p)],
        "pk_finalize": [C.c_void_p],
        "pk_register_buffer": [C.c_void_p, C.c_int, _I64P, C.c_int, C.POINTER(C.c_void_p), C.c_void_p, _I64P],
        "pk_copy_from_host": [C.c_void_p, C.c_int64, C.c_void_p, C.c_size_t],
        "pk_sync_to_host": [C.c_void_p, C.c_int64, C.c_void_p, C.c_size_t],
        "pk_copy_from_host_async": [C.c_void_p, C.c_int64, C.c_void_p, C.c_size_t],
        "pk_sync_to_host_async": [C.c_void_p, C.c_int64, C.c_void_p, C.c_size_t],
        "pk_copy_from_host_for": [C.c_void_p, C.c_int64, C.c_void_p, C.c_size_t, C.c_int64, C.c_int, _I32P, _I32P,
                                  _I64P, C.c_int],
        "pk_unregister_buffer": [C.c_void_p, C.c_int64],
        "pk_buffer_instance": [C.c_void_p, C.c_int64, C.c_int, C.POINTER(C.c_void_p)],
        "pk_register_kernel": [C.c_void_p, C.c_char_p, C.c_void_p, C.c_int, _I32P, C.c_int32, _I64P],
        "pk_declare_affine_access": [C.c_void_p, C.c_int64, C.c_int, C.c_int, C.POINTER(pk_affine_access)],
        "pk_builtin_kernel": [C.c_void_p, C.c_char_p, _I64P],
        "pk_launch_partitioned": [C.c_void_p, C.c_int64, _I32P, _I32P, C.c_size_t,
                                  C.POINTER(C.c_void_p), _I64P, C.c_int],
        "pk_launch_direct": [C.c_void_p, C.c_int64, _I32P, _I32P, C.c_size_t,
                             C.POINTER(C.c_void_p), _I64P, C.c_int],
        "pk_launch_sequence": [C.c_void_p, C.c_void_p, C.c_int],
        "pk_synchronize": [C.c_void_p],
        "pk_timer_begin": [C.c_void_p],
        "pk_timer_end": [C.c_void_p, C.POINTER(C.c_double)],
        "pk_partition_grid": [C.c_void_p, C.c_int64, _I32P, C.c_int, _I64P],
        "pk_set_partition_shape": [C.c_void_p, C.c_int64, _I32P],
        "pk_enumerate": [C.c_void_p, C.c_int64, C.c_int, C.c_int, C.c_int64, _I64P, _I32P, _I64P,
                         C.c_int, RANGE_CB, C.c_void_p],
        "pk_tracker_dump": [C.c_void_p, C.c_int64, SEGMENT_CB, C.c_void_p],
        "pk_last_plan": [C.c_void_p, COPY_CB, C.c_void_p],
        "pk_get_stats": [C.c_void_p, C.POINTER(pk_stats)],
        "pk_reset_stats": [C.c_void_p],
        "pk_set_mode": [C.c_void_p, C.c_uint32],
        "pk_trace_reset": [C.c_void_p],
        "pk_trace_fetch": [C.c_void_p, C.c_int64, C.c_int, C.c_int, C.POINTER(C.c_uint32), C.c_uint64],
        "pk_trace_stray": [C.c_void_p, C.POINTER(C.c_uint64)],
    }
    for name, args in sig.items():
        f = getattr(L, name)
        f.argtypes = args
        f.restype = C.c_int
    L.pk_trace_available.argtypes = []
    L.pk_trace_available.restype = C.c_int
    L.pk_builtin_fn.argtypes = [C.c_char_p]
    L.pk_builtin_fn.restype = C.c_void_p
    L.pk_get_mode.argtypes = [C.c_void_p]
    L.pk_get_mode.restype = C.c_uint32
    L.pk_last_error.restype = C.c_char_p
    L.pk_version.restype = C.c_char_p
    _lib = L
    return L


def _check(rc, where):
    if rc != PK_OK:
        raise PkError(rc, where, lib().pk_last_error().decode())


def _addr(x):
    """Host or device address of a numpy array, torch tensor or int."""
    if x is None:
        return None
    if isinstance(x, int):
        return x
    if hasattr(x, "data_ptr"):
        return x.data_ptr()
    if hasattr(x, "ctypes"):
        return x.ctypes.data
    raise TypeError(f"cannot take the address of {type(x)}")


def _nbytes(x):
    if hasattr(x, "nbytes"):
        return int(x.nbytes)
    return int(x.numel() * x.element_size())


def _i32(v):
    return (C.c_int32 * len(v))(*v)


def _i64(v):
    return (C.c_int64 * max(1, len(v)))(*v)


# ------------------------------------------------------------------ same names as the C-ABI
def pk_version() -> str:
    return lib().pk_version().decode()


def pk_last_error() -> str:
    return lib().pk_last_error().decode()


def pk_init(nparts, part_device=None, part_rank=None, my_rank=0, world_size=1, flags=0):
    p = pk_init_params(nparts, my_rank, world_size, flags,
                       _i32(part_device) if part_device is not None else None,
                       _i32(part_rank) if part_rank is not None else None)
    ctx = C.c_void_p()
    _check(lib().pk_init(C.byref(p), C.byref(ctx)), "pk_init")
    return ctx


def pk_nccl_unique_id() -> bytes:
    buf = C.create_string_buffer(128)
    _check(lib().pk_nccl_unique_id(buf, 128), "pk_nccl_unique_id")
    return buf.raw


def pk_init_spmd(nparts, my_rank, world_size, part_rank, part_device=None, nccl_id=None, flags=0):
    """Multi-process SPMD context: this rank owns the partitions p with part_rank[p] == my_rank."""
    p = pk_init_params(nparts, my_rank, world_size, flags,
                       _i32(part_device) if part_device is not None else None, _i32(part_rank))
    ctx = C.c_void_p()
    idbuf = C.create_string_buffer(nccl_id, 128) if nccl_id is not None else None
    _check(lib().pk_init_spmd(C.byref(p), idbuf, C.byref(ctx)), "pk_init_spmd")
    return ctx


def pk_init_spmd_ipc(nparts, my_rank, world_size, part_rank, allgather, part_device=None, flags=0):
    """Multi-process SPMD context over peer memory (CUDA IPC, device epoch flags).
    `allgather(data: bytes) -> bytes` must return the concatenation of every rank's
    `data` in rank order (e.g. ``spmd.dist_allgather()``); it is called collectively."""
    def _cb(_user, send, recv, n):
        try:
            out = allgather(C.string_at(send, n))
            if len(out) != n * world_size:
                return -1
            C.memmove(recv, out, len(out))
            return 0
        except Exception:
            return -1
    cb = ALLGATHER_CB(_cb)
    p = pk_init_params(nparts, my_rank, world_size, flags,
                       _i32(part_device) if part_device is not None else None, _i32(part_rank))
    ctx = C.c_void_p()
    _check(lib().pk_init_spmd_ipc(C.byref(p), cb, None, C.byref(ctx)), "pk_init_spmd_ipc")
    _keepalive[ctx.value] = cb
    return ctx


def pk_finalize(ctx):
    try:
        _check(lib().pk_finalize(ctx), "pk_finalize")
    finally:
        _keepalive.pop(ctx.value, None)


def pk_register_buffer(ctx, shape, elem_bytes, dev_ptrs=None, host_init=None, nparts=None):
    shape = list(shape)
    out = C.c_int64()
    dp = None
    if dev_ptrs is not None:
        dp = (C.c_void_p * len(dev_ptrs))(*[_addr(d) for d in dev_ptrs])
    _check(lib().pk_register_buffer(ctx, len(shape), _i64(shape), elem_bytes, dp, _addr(host_init),
                                    C.byref(out)), "pk_register_buffer")
    return out.value


def pk_copy_from_host(ctx, buf, host, nbytes=None):
    _check(lib().pk_copy_from_host(ctx, buf, _addr(host), nbytes if nbytes is not None else _nbytes(host)),
           "pk_copy_from_host")


def pk_copy_from_host_for(ctx, buf, host, kernel, arg_index, grid, block, scalars=(), nbytes=None):
    """Read-pattern-aware H2D: each partition receives what `kernel`'s launch reads via `arg_index`."""
    sc = list(scalars)
    _check(lib().pk_copy_from_host_for(ctx, buf, _addr(host), nbytes if nbytes is not None else _nbytes(host),
                                       kernel, arg_index, _i32(grid), _i32(block), _i64(sc), len(sc)),
           "pk_copy_from_host_for")


def pk_sync_to_host(ctx, buf, host, nbytes=None):
    """host may be None on SPMD ranks other than 0 (then pass nbytes)."""
    _check(lib().pk_sync_to_host(ctx, buf, _addr(host), nbytes if nbytes is not None else _nbytes(host)),
           "pk_sync_to_host")


def pk_copy_from_host_async(ctx, buf, host, nbytes=None):
    """Enqueued H2D; `host` (pinned for overlap) must stay alive until pk_synchronize."""
    _check(lib().pk_copy_from_host_async(ctx, buf, _addr(host), nbytes if nbytes is not None else _nbytes(host)),
           "pk_copy_from_host_async")


def pk_sync_to_host_async(ctx, buf, host, nbytes=None):
    """Enqueued D2H gather; `host` is complete after pk_synchronize."""
    _check(lib().pk_sync_to_host_async(ctx, buf, _addr(host), nbytes if nbytes is not None else _nbytes(host)),
           "pk_sync_to_host_async")


def pk_unregister_buffer(ctx, buf):
    _check(lib().pk_unregister_buffer(ctx, buf), "pk_unregister_buffer")


def pk_buffer_instance(ctx, buf, part) -> int:
    p = C.c_void_p()
    _check(lib().pk_buffer_instance(ctx, buf, part, C.byref(p)), "pk_buffer_instance")
    return p.value or 0


def pk_builtin_fn(name) -> int:
    return lib().pk_builtin_fn(name.encode()) or 0


def pk_register_kernel(ctx, name, fn, arg_kinds, partition_dim=-1) -> int:
    out = C.c_int64()
    _check(lib().pk_register_kernel(ctx, name.encode(), fn, len(arg_kinds), _i32(arg_kinds), partition_dim,
                                    C.byref(out)), "pk_register_kernel")
    return out.value


def pk_declare_affine_access(ctx, kernel, arg_index, mode, tap: pk_affine_access):
    _check(lib().pk_declare_affine_access(ctx, kernel, arg_index, mode, C.byref(tap)),
           "pk_declare_affine_access")


def pk_builtin_kernel(ctx, name) -> int:
    out = C.c_int64()
    _check(lib().pk_builtin_kernel(ctx, name.encode(), C.byref(out)), "pk_builtin_kernel")
    return out.value


_LAUNCH_ARGS = {}   # marshalled ctypes arguments of recent launches (steady-state loops repeat them)


def _launch_args(kernel, grid, block, args, scalars):
    key = (kernel, tuple(grid), tuple(block), tuple(args), tuple(scalars))
    m = _LAUNCH_ARGS.get(key)
    if m is None:
        vals = [C.c_int64(a) if a is not None else None for a in args]
        argv = (C.c_void_p * max(1, len(vals)))(*[C.addressof(v) if v is not None else None for v in vals])
        sc = list(scalars)
        m = (_i32(grid), _i32(block), argv, _i64(sc), len(sc), vals)
        if len(_LAUNCH_ARGS) > 1024:
            _LAUNCH_ARGS.clear()
        _LAUNCH_ARGS[key] = m
    return m


def pk_launch_partitioned(ctx, kernel, grid, block, args, scalars=(), smem=0):
    """args: one int per kernel argument -- the pk_buf id for a buffer, the
    (int64) value for a scalar; None passes a NULL pointer."""
    m = _launch_args(kernel, grid, block, args, scalars)
    _check(lib().pk_launch_partitioned(ctx, kernel, m[0], m[1], smem, m[2], m[3], m[4]), "pk_launch_partitioned")


class pk_launch_desc(C.Structure):
    _fields_ = [("kernel", C.c_int64), ("grid", C.c_int32 * 3), ("block", C.c_int32 * 3), ("smem_bytes", C.c_size_t),
                ("args", C.POINTER(C.c_void_p)), ("scalars", _I64P), ("nscalars", C.c_int)]


_SEQUENCES = {}


def pk_launch_sequence(ctx, launches):
    """launches: [(kernel, grid, block, args, scalars), ...] -- one pk_launch_partitioned
    argument list each (args as there), issued as one unit (memoised as one graph)."""
    key = tuple((k, tuple(g), tuple(b), tuple(a), tuple(sc)) for k, g, b, a, sc in launches)
    m = _SEQUENCES.get(key)
    if m is None:
        descs = (pk_launch_desc * max(1, len(key)))()
        keep = []
        for i, (k, g, b, a, sc) in enumerate(key):
            la = _launch_args(k, g, b, a, sc)
            keep.append(la)
            d = descs[i]
            d.kernel, d.smem_bytes = k, 0
            d.grid[:] = list(g)
            d.block[:] = list(b)
            d.args = la[2]
            d.scalars = la[3]
            d.nscalars = la[4]
        m = (descs, len(key), keep)
        if len(_SEQUENCES) > 64:
            _SEQUENCES.clear()
        _SEQUENCES[key] = m
    _check(lib().pk_launch_sequence(ctx, C.cast(m[0], C.c_void_p), m[1]), "pk_launch_sequence")


def pk_launch_direct(ctx, kernel, grid, block, args, scalars=(), smem=0):
    """The original single-GPU launch (E3 baseline; single-partition contexts only)."""
    m = _launch_args(kernel, grid, block, args, scalars)
    _check(lib().pk_launch_direct(ctx, kernel, m[0], m[1], smem, m[2], m[3], m[4]), "pk_launch_direct")


def pk_synchronize(ctx):
    _check(lib().pk_synchronize(ctx), "pk_synchronize")


def pk_timer_begin(ctx):
    _check(lib().pk_timer_begin(ctx), "pk_timer_begin")


def pk_timer_end(ctx) -> float:
    ms = C.c_double()
    _check(lib().pk_timer_end(ctx, C.byref(ms)), "pk_timer_end")
    return ms.value


def pk_set_partition_shape(ctx, kernel, tiles=None):
    """tiles = (tx, ty, tz) with tx*ty*tz == P, or None for the 1-D split (NEXT-2)."""
    t = None if tiles is None else _i32(list(tiles))
    _check(lib().pk_set_partition_shape(ctx, kernel, t), "pk_set_partition_shape")


def pk_partition_grid(ctx, kernel, grid, part):
    out = (C.c_int64 * 6)()
    _check(lib().pk_partition_grid(ctx, kernel, _i32(grid), part, out), "pk_partition_grid")
    return tuple(out)


def pk_enumerate(ctx, kernel, arg_index, mode, buf, part6, block, scalars=()):
    ranges = []
    cb = RANGE_CB(lambda _u, b, e: ranges.append((b, e)))
    sc = list(scalars)
    _check(lib().pk_enumerate(ctx, kernel, arg_index, mode, buf, _i64(list(part6)), _i32(block), _i64(sc),
                              len(sc), cb, None), "pk_enumerate")
    return ranges


def pk_tracker_dump(ctx, buf):
    segs = []
    cb = SEGMENT_CB(lambda _u, b, e, m: segs.append((b, e, m)))
    _check(lib().pk_tracker_dump(ctx, buf, cb, None), "pk_tracker_dump")
    return segs


def pk_last_plan(ctx):
    ops = []
    cb = COPY_CB(lambda _u, buf, s, d, b, e: ops.append((buf, s, d, b, e)))
    _check(lib().pk_last_plan(ctx, cb, None), "pk_last_plan")
    return ops


def pk_get_stats(ctx) -> dict:
    s = pk_stats()
    _check(lib().pk_get_stats(ctx, C.byref(s)), "pk_get_stats")
    d = {name: getattr(s, name) for name, _ in pk_stats._fields_ if name != "pair_bytes"}
    d["pair_bytes"] = [[s.pair_bytes[i][j] for j in range(16)] for i in range(16)]
    return d


def pk_reset_stats(ctx):
    _check(lib().pk_reset_stats(ctx), "pk_reset_stats")


def pk_set_mode(ctx, flags):
    _check(lib().pk_set_mode(ctx, flags), "pk_set_mode")


def pk_get_mode(ctx) -> int:
    return int(lib().pk_get_mode(ctx))


# ------------------------------------------------------------------ descriptor builders
def expr(c0=0, scalars=None, blockdim=None) -> pk_expr:
    """c0 + sum scalars[s] * coef + sum blockdim[w] * coef (dicts index -> coef)."""
    e = pk_expr()
    e.c0 = c0
    for s, v in (scalars or {}).items():
        e.c_scalar[s] = v
    for w, v in (blockdim or {}).items():
        e.c_blockdim[w] = v
    return e


def dim_map(grid_dim, scale, extent, offset=0, clamp=False, guard=None) -> pk_dim_map:
    """scale/extent/offset: int or pk_expr; guard: (lo, hi) of ints/pk_expr or None."""
    def ex(v):
        return v if isinstance(v, pk_expr) else expr(int(v))
    d = pk_dim_map()
    d.grid_dim = grid_dim
    d.flags = (PK_DIM_CLAMP if clamp else 0) | (PK_DIM_GUARD if guard is not None else 0)
    d.scale, d.extent, d.offset = ex(scale), ex(extent), ex(offset)
    if guard is not None:
        d.guard_lo, d.guard_hi = ex(guard[0]), ex(guard[1])
    return d


def affine_access(dims) -> pk_affine_access:
    a = pk_affine_access()
    a.ndim = len(dims)
    for i, d in enumerate(dims):
        a.dim[i] = d
    return a


# ---------------------------------------------------------------- access recording (libpk_trace.so)
def pk_trace_available() -> bool:
    return bool(lib().pk_trace_available())


def pk_trace_reset(ctx):
    _check(lib().pk_trace_reset(ctx), "pk_trace_reset")


def pk_trace_fetch(ctx, buf, part, kind, nbytes):
    """Bitmap of instance `part` of `buf` (kind 0 fetched, 1 stored) as a bool array with
    one entry per 4-byte word of the instance."""
    import numpy as np
    nw = nbytes // 4
    words = np.zeros((nw + 31) // 32, dtype=np.uint32)
    _check(lib().pk_trace_fetch(ctx, buf, part, kind, words.ctypes.data_as(C.POINTER(C.c_uint32)), words.size),
           "pk_trace_fetch")
    bits = np.unpackbits(words.view(np.uint8), bitorder="little")
    return bits[:nw].astype(bool)


def pk_trace_stray(ctx) -> int:
    v = C.c_uint64(0)
    _check(lib().pk_trace_stray(ctx, C.byref(v)), "pk_trace_stray")
    return int(v.value)
