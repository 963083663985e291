"""Launch sequences of every builtin kernel on small ragged grids, shared by the
access-recording test (tests/trace_worker.py, libpk_trace.so) and the poison test
(tests/test_gpu_access.py) -- test infrastructure.

A case builds its buffers through a caller-supplied `make(shape, elem_bytes, host)`
(so the poison test can hand in caller-owned torch instances) and returns
  (kernel id, [launch, ...], {buffer id: (shape, elem_bytes)})
with launch = (grid, block, args, scalars) in the order the program issues them.

`overfetch[(case, arg)] = (dz, dy, dx)` states, per input argument, how far beyond its
DECLARED read set the kernel may FETCH (in elements of the last three dimensions) --
the halo a TMA copy brings in but no computation uses ("what the kernels
touch"): 16-byte aligned bulk-copy segments (4 or 8 columns each side), tensor-TMA boxes
whose width is a multiple of 16 bytes, and tb2/tbK fetching power over temp's halo rows.
"""
from __future__ import annotations

import numpy as np

import synth
from paper_conf_icppw_matzdf20_b200 import abi
from paper_conf_icppw_matzdf20_b200 import kernels as K


def _pingpong(geom, a, b, extra, n):
    grid, blk, sc = geom
    out = []
    for t in range(n):
        x, y = (a, b) if t % 2 == 0 else (b, a)
        out.append((grid, blk, [x, *extra[0], y, *extra[1]], sc))
    return out


def jacobi2d(ctx, make, h=72, w=100):
    u = synth.jacobi_grid(h, w)
    kid = abi.pk_builtin_kernel(ctx, "jacobi2d")
    u0, u1 = make((h, w), 4, u), make((h, w), 4, u)
    geom = K.jacobi2d_launch(h, w)
    return kid, _pingpong(geom, u0, u1, ([], [h, w]), 2), {u0: ((h, w), 4), u1: ((h, w), 4)}


def jacobi2d_tb(ctx, make, h=72, w=100, k=3):
    u = synth.jacobi_grid(h, w)
    kid = abi.pk_builtin_kernel(ctx, "jacobi2d_tb")
    u0, u1 = make((h, w), 4, u), make((h, w), 4, u)
    geom = K.jacobi2d_tb_launch(h, w, k)
    return kid, _pingpong(geom, u0, u1, ([], [h, w, k]), 2), {u0: ((h, w), 4), u1: ((h, w), 4)}


def _hotspot(name, ctx, make, h, w, ty, k=4, bdx=K.HOTSPOT_BDX):
    t, p = synth.hotspot_grids(h, w)
    kid = abi.pk_builtin_kernel(ctx, name)
    t0, t1, pw = make((h, w), 4, t), make((h, w), 4, None), make((h, w), 4, p)
    geom = K.hotspot2d_tbk_launch(h, w, ty, k) if name == "hotspot2d_tbk" else K.hotspot2d_launch(h, w, ty, bdx)
    grid, blk, sc = geom
    launches = [(grid, blk, [t0, pw, t1, h, w, sc[2]], sc), (grid, blk, [t1, pw, t0, h, w, sc[2]], sc)]
    return kid, launches, {t0: ((h, w), 4), t1: ((h, w), 4), pw: ((h, w), 4)}


def hotspot2d(ctx, make):
    return _hotspot("hotspot2d", ctx, make, 70, 1100, 16)


def hotspot2d_regs(ctx, make):
    return _hotspot("hotspot2d_regs", ctx, make, 70, 600, 8, bdx=32)


def hotspot2d_tb2(ctx, make):
    return _hotspot("hotspot2d_tb2", ctx, make, 70, 1100, 16)


def hotspot2d_tbk(k):
    def case(ctx, make):
        return _hotspot("hotspot2d_tbk", ctx, make, 70, 1000, 16, k=k)
    case.__name__ = f"hotspot2d_tbk{k}"
    return case


def _heat(name, ctx, make, d, h, w, zc, bdy=K.HEAT_BDY):
    u = synth.heat_grid(d, h, w)
    kid = abi.pk_builtin_kernel(ctx, name)
    u0, u1 = make((d, h, w), 4, u), make((d, h, w), 4, None)
    geom = (K.heat3d_tb2_launch(d, h, w, zc) if name == "heat3d_tb2" else
            K.heat3d_tb3_launch(d, h, w, zc) if name == "heat3d_tb3" else K.heat3d_launch(d, h, w, zc, bdy))
    grid, blk, sc = geom
    launches = [(grid, blk, [u0, u1, d, h, w, sc[3]], sc), (grid, blk, [u1, u0, d, h, w, sc[3]], sc)]
    return kid, launches, {u0: ((d, h, w), 4), u1: ((d, h, w), 4)}


def heat3d(ctx, make):
    return _heat("heat3d", ctx, make, 21, 70, 260, 4, bdy=30)


def heat3d_regs(ctx, make):
    return _heat("heat3d_regs", ctx, make, 21, 70, 260, 4, bdy=8)


def heat3d_tb2(ctx, make):
    return _heat("heat3d_tb2", ctx, make, 21, 40, 252, 4)


def heat3d_tb3(ctx, make):
    return _heat("heat3d_tb3", ctx, make, 21, 40, 252, 4)


def nbody(ctx, make, n=3000):
    pos, vel = synth.nbody_bodies(n)
    kid = abi.pk_builtin_kernel(ctx, "nbody")
    p0, p1, v = make((n,), 16, pos), make((n,), 16, None), make((n,), 16, vel)
    grid, blk, sc = K.nbody_launch(n)
    launches = [(grid, blk, [p0, v, p1, n], sc), (grid, blk, [p1, v, p0, n], sc)]
    return kid, launches, {p0: ((n,), 16), p1: ((n,), 16), v: ((n,), 16)}


def sgemm(ctx, make, m=300, n=520, k=200):
    a, b = synth.gemm_operands(m, n, k)
    kid = abi.pk_builtin_kernel(ctx, "sgemm_tf32x3")
    ab, bb, cb = make((m, k), 4, a), make((k, n), 4, b), make((m, n), 4, None)
    grid, blk, sc = K.sgemm_launch(m, n, k)
    launches = [(grid, blk, [ab, bb, cb, m, n, k], sc)] * 2
    return kid, launches, {ab: ((m, k), 4), bb: ((k, n), 4), cb: ((m, n), 4)}


def tiled(case, tiles):
    """The same case on a tile partition (NEXT-2, reading Q24): column cuts expose the
    horizontal TMA over-fetch that row slabs hide (full rows are read there anyway)."""
    def fn(ctx, make):
        kid, launches, buffers = case(ctx, make)
        abi.pk_set_partition_shape(ctx, kid, tiles)
        return kid, launches, buffers
    fn.__name__ = case.__name__ + "_t" + "x".join(str(t) for t in tiles)
    fn.tiles = tiles
    return fn


_BASE = (jacobi2d, jacobi2d_tb, hotspot2d, hotspot2d_regs, hotspot2d_tb2, hotspot2d_tbk(2), hotspot2d_tbk(3), hotspot2d_tbk(4),
         hotspot2d_tbk(6), hotspot2d_tbk(8), heat3d, heat3d_regs, heat3d_tb2, heat3d_tb3, nbody, sgemm)
_B = {f.__name__: f for f in _BASE}
_TILED = (tiled(_B["jacobi2d"], (2, 2, 1)), tiled(_B["jacobi2d_tb"], (2, 2, 1)), tiled(_B["hotspot2d"], (3, 1, 1)), tiled(_B["hotspot2d_regs"], (2, 2, 1)),
          tiled(_B["hotspot2d_tb2"], (3, 1, 1)), tiled(_B["hotspot2d_tbk2"], (3, 1, 1)),
          tiled(_B["hotspot2d_tbk3"], (2, 2, 1)), tiled(_B["hotspot2d_tbk4"], (3, 1, 1)),
          tiled(_B["hotspot2d_tbk8"], (3, 1, 1)), tiled(_B["heat3d"], (2, 1, 2)), tiled(_B["heat3d_tb2"], (2, 1, 2)),
          tiled(_B["heat3d_tb3"], (2, 1, 2)),
          tiled(_B["sgemm"], (2, 2, 1)))
CASES = {f.__name__: f for f in _BASE + _TILED}


def parts(name):
    """Partition counts a case runs at: slabs at 1 and 3, tiles at their tile count."""
    t = getattr(CASES[name], "tiles", None)
    return (t[0] * t[1] * t[2],) if t else (1, 3)


def _tbk_halo(k):
    return 4 if k <= 4 else 8      # fetched temp halo columns: 4 (K <= 4) or 8 (K = 5..8) per side


OVERFETCH = {
    ("hotspot2d", 0): (0, 0, 3),                  # 16-B aligned temp segments: 4 halo columns, 1 used
    ("hotspot2d_tb2", 0): (0, 0, 2),              # 4 halo columns fetched, 2 used
    ("hotspot2d_tb2", 1): (0, 1, 3),              # power rides with temp: 2 halo rows / 4 columns, 1 used
    # one TMA box per streamed plane, the z-halo planes included (where only the block's own
    # rows and columns are declared): 136 x (bdy + 2) box = 4 columns / 1 row around the block
    ("heat3d", 0): (0, 1, 4),
    ("heat3d_tb2", 0): (0, 0, 2),                 # 128 x 20 box for 120 x 16 owned: 4 columns, 2 used
    ("heat3d_tb3", 0): (0, 0, 1),                 # 128 x 22 box for 120 x 16 owned: 4 columns, 3 used
}
for _k in (2, 3, 4, 6, 8):
    OVERFETCH[(f"hotspot2d_tbk{_k}", 0)] = (0, 0, _tbk_halo(_k) - _k)
    OVERFETCH[(f"hotspot2d_tbk{_k}", 1)] = (0, 1, _tbk_halo(_k) - _k + 1)
for (_n, _a), _v in list(OVERFETCH.items()):
    for _t in _TILED:
        if _t.__name__.rsplit("_t", 1)[0] == _n:
            OVERFETCH[(_t.__name__, _a)] = _v


def ranges_to_mask(ranges, nbytes):
    m = np.zeros(nbytes // 4, dtype=bool)
    for b, e in ranges:
        assert b % 4 == 0 and e % 4 == 0
        m[b // 4:e // 4] = True
    return m


def declared(ctx, kid, launch, buffers, P):
    """{(buf, part): (read mask, write mask)} of one launch, per 4-byte word, from pk_enumerate
    over every argument bound to the buffer (the library's own region analysis)."""
    grid, blk, args, sc = launch
    nbuf = 0                       # buffer arguments lead every builtin's argument list
    while nbuf < len(args) and args[nbuf] in buffers:
        nbuf += 1
    out = {}
    for p in range(P):
        box = abi.pk_partition_grid(ctx, kid, grid, p)
        for a, x in enumerate(args[:nbuf]):
            shape, eb = buffers[x]
            nbytes = int(np.prod(shape)) * eb
            r, w = out.get((x, p), (np.zeros(nbytes // 4, bool), np.zeros(nbytes // 4, bool)))
            r = r | ranges_to_mask(abi.pk_enumerate(ctx, kid, a, abi.PK_READ, x, box, blk, sc), nbytes)
            w = w | ranges_to_mask(abi.pk_enumerate(ctx, kid, a, abi.PK_WRITE, x, box, blk, sc), nbytes)
            out[(x, p)] = (r, w)
    return out


def dilate(mask, shape, eb, dz, dy, dx):
    """Dilate a per-word mask of an array of `shape` (elements of eb bytes) by (dz, dy, dx)
    elements along its last three dimensions, clipped to the array."""
    wpe = eb // 4
    sh = tuple(shape) + (wpe,)
    m = mask.reshape(sh).any(axis=-1)
    full3 = (1,) * (3 - m.ndim) + m.shape
    m3 = m.reshape(full3)
    out = m3.copy()
    for axis, d in zip(range(3), (dz, dy, dx)):
        for s in range(1, d + 1):
            n = m3.shape[axis]
            if s >= n:
                break
            sl_a = [slice(None)] * 3
            sl_b = [slice(None)] * 3
            sl_a[axis], sl_b[axis] = slice(s, None), slice(None, n - s)
            out[tuple(sl_a)] |= m3[tuple(sl_b)]
            out[tuple(sl_b)] |= m3[tuple(sl_a)]
        m3 = out.copy()
    return np.repeat(out.reshape(m.shape)[..., None], wpe, axis=-1).reshape(-1)
