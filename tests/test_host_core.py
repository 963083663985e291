"""Host core of libpk.so (region analyzer, validity tracker, transfer planner) vs the
oracle, bit-exact, on CPU (contexts created with PK_INIT_HOST_ONLY: no CUDA call).

  - pk_enumerate == brute-force thread programs (oracle/regions.py) for every
    builtin kernel, ragged shapes, several block geometries and P
  - pk_enumerate == brute-force descriptor evaluation (oracle/descriptors.py) for
    random descriptors (hypothesis)
  - Eq. 1-4: the library's union of taps is the exact 27-point U,
    not the 28-point row-wise first/last over-approximation
  - launch sequences: stale bytes, copy plans and tracker dumps == shadow oracle
    (c3), and == the closed forms (c5)
  - error paths: WAW overlap, out of bounds, overflow, non-separable
"""
import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

from oracle import closed_forms as cf
from oracle import descriptors as od
from oracle import grid as og
from oracle import polyhedral as poly
from oracle import regions, shadow
from paper_conf_icppw_matzdf20_b200 import abi
from paper_conf_icppw_matzdf20_b200 import kernels as K

HO = abi.PK_INIT_HOST_ONLY


def host_ctx(P, mode=0):
    ctx = abi.pk_init(P, flags=HO)
    if mode:
        abi.pk_set_mode(ctx, mode)
    return ctx


def _lib_sets(ctx, k, nargs, bufs, box, block, sc):
    out = {}
    for a in range(nargs):
        if bufs[a] is None:
            continue
        for mode, tag in ((abi.PK_READ, "r"), (abi.PK_WRITE, "w")):
            r = abi.pk_enumerate(ctx, k, a, mode, bufs[a], box, block, sc)
            if r:
                out[(a, tag)] = r
    return out


def _oracle_sets(acc, ebs):
    return {key: regions.to_byte_ranges(v, ebs[key[0]]) for key, v in acc.items() if len(v)}


# ------------------------------------------------------------ regions vs brute force
@pytest.mark.parametrize("h,w,block", [(64, 64, (32, 8)), (37, 50, (32, 8)), (9, 70, (16, 4)), (3, 3, (32, 8))])
@pytest.mark.parametrize("P", [1, 2, 3, 5, 8])
def test_jacobi_regions(h, w, block, P):
    ctx = host_ctx(P)
    k = abi.pk_builtin_kernel(ctx, "jacobi2d")
    b0 = abi.pk_register_buffer(ctx, (h, w), 4)
    b1 = abi.pk_register_buffer(ctx, (h, w), 4)
    grid, blk, sc = K.jacobi2d_launch(h, w, block + (1,))
    for p in range(P):
        box = abi.pk_partition_grid(ctx, k, grid, p)
        assert box == og.partition_box(grid, P, p)
        lib = _lib_sets(ctx, k, 4, [b0, b1, None, None], box, blk, sc)
        ora = _oracle_sets(regions.jacobi2d(box, blk, h, w), {0: 4, 1: 4})
        assert lib == ora
    abi.pk_finalize(ctx)


@pytest.mark.parametrize("kernel,h,w,ty,bdx", [("hotspot2d_regs", 64, 64, 4, 32), ("hotspot2d_regs", 100, 36, 16, 32),
                                               ("hotspot2d_regs", 33, 520, 4, 128), ("hotspot2d", 33, 1100, 4, 128),
                                               ("hotspot2d", 5, 4, 64, 128), ("hotspot2d", 200, 1028, 16, 128)])
@pytest.mark.parametrize("P", [1, 2, 3, 4, 7])
def test_hotspot_regions(kernel, h, w, ty, bdx, P):
    ctx = host_ctx(P)
    k = abi.pk_builtin_kernel(ctx, kernel)
    bufs = [abi.pk_register_buffer(ctx, (h, w), 4) for _ in range(3)]
    grid, blk, sc = K.hotspot2d_launch(h, w, ty, bdx)
    for p in range(P):
        box = abi.pk_partition_grid(ctx, k, grid, p)
        lib = _lib_sets(ctx, k, 6, bufs + [None] * 3, box, blk, sc)
        ora = _oracle_sets(regions.hotspot2d(box, blk, h, w, ty), {0: 4, 1: 4, 2: 4})
        assert lib == ora
    abi.pk_finalize(ctx)


@pytest.mark.parametrize("d,h,w,zc,bdy", [(16, 8, 32, 3, 4), (10, 9, 132, 8, 8), (1, 1, 4, 64, 8)])
@pytest.mark.parametrize("P", [1, 2, 3, 6])
def test_heat_regions(d, h, w, zc, bdy, P):
    ctx = host_ctx(P)
    k = abi.pk_builtin_kernel(ctx, "heat3d")
    bufs = [abi.pk_register_buffer(ctx, (d, h, w), 4) for _ in range(2)]
    grid, blk, sc = K.heat3d_launch(d, h, w, zc, bdy)
    for p in range(P):
        box = abi.pk_partition_grid(ctx, k, grid, p)
        lib = _lib_sets(ctx, k, 6, bufs + [None] * 4, box, blk, sc)
        ora = _oracle_sets(regions.heat3d(box, blk, d, h, w, zc), {0: 4, 1: 4})
        assert lib == ora
    abi.pk_finalize(ctx)


@pytest.mark.parametrize("n,bdx", [(300, 64), (1024, 256), (1, 32), (5000, 128)])
@pytest.mark.parametrize("P", [1, 2, 3, 8])
def test_nbody_regions(n, bdx, P):
    ctx = host_ctx(P)
    k = abi.pk_builtin_kernel(ctx, "nbody")
    bufs = [abi.pk_register_buffer(ctx, (n,), 16) for _ in range(3)]
    grid, blk, sc = K.nbody_launch(n, bdx)
    for p in range(P):
        box = abi.pk_partition_grid(ctx, k, grid, p)
        lib = _lib_sets(ctx, k, 4, bufs + [None], box, blk, sc)
        ora = _oracle_sets(regions.nbody(box, blk, n, K.NBODY_PER_THREAD), {0: 16, 1: 16, 2: 16})
        assert lib == ora
    abi.pk_finalize(ctx)


# ------------------------------------------------------------ Eq. 1-4 through the library
def _point_taps():
    """S1 as one tap per row y: {y} x [y, 4]; S2 = M(S1)."""
    s1, s2 = [], []
    for y in range(5):
        for (dy, dx), out in (((0, 0), s1), ((1, 3), s2)):
            out.append([{"grid_dim": -1, "scale": 0, "extent": 1, "offset": y + dy, "clamp": False, "guard": None},
                        {"grid_dim": -1, "scale": 0, "extent": 5 - y, "offset": y + dx, "clamp": False, "guard": None}])
    return s1, s2


def _to_abi(tap):
    return abi.affine_access([abi.dim_map(d["grid_dim"], d["scale"], d["extent"], d["offset"], d["clamp"],
                                          d["guard"]) for d in tap])


def test_eq1_4_union_is_exact_through_library():
    ctx = host_ctx(1)
    k = abi.pk_register_kernel(ctx, "eq1_4", None, [abi.PK_ARG_BUFFER])
    buf = abi.pk_register_buffer(ctx, (8, 8), 1)
    s1, s2 = _point_taps()
    for t in s1 + s2:
        abi.pk_declare_affine_access(ctx, k, 0, abi.PK_READ, _to_abi(t))
    rng = abi.pk_enumerate(ctx, k, 0, abi.PK_READ, buf, (0, 1, 0, 1, 0, 1), (1, 1, 1))
    pts = {(b // 8, b % 8) for (lo, hi) in rng for b in range(lo, hi)}
    assert pts == poly.U()
    assert len(pts) == 27                                   # not 28: row y = 4 is [4,4] u [6,7]
    assert (4, 5) not in pts
    # the descriptor brute force agrees (pins oracle/descriptors.py by Eq. 1-4)
    el = od.union_elements(s1 + s2, (0, 1, 0, 1, 0, 1), (8, 8))
    assert {(e // 8, e % 8) for e in el} == poly.U()
    abi.pk_finalize(ctx)


# ------------------------------------------------------------ random descriptors
@st.composite
def _descr(draw):
    ndim = draw(st.integers(1, 3))
    shape = tuple(draw(st.integers(1, 9)) for _ in range(ndim))
    grid_dims = draw(st.permutations([0, 1, 2]))
    taps = []
    for _ in range(draw(st.integers(1, 3))):
        tap = []
        for k in range(ndim):
            use = draw(st.booleans())
            g = grid_dims[k] if use else -1
            scale = draw(st.integers(0, 4))
            extent = draw(st.integers(0, 5))
            clamp = draw(st.booleans())
            guard = None
            if draw(st.booleans()):
                lo = draw(st.integers(-2, 6))
                guard = (lo, lo + draw(st.integers(0, 8)))
            off = draw(st.integers(-3, 3)) if clamp else 0
            tap.append({"grid_dim": g, "scale": scale, "extent": extent, "offset": off, "clamp": clamp,
                        "guard": guard if clamp else None})
        taps.append(tap)
    gridv = tuple(draw(st.integers(1, 4)) for _ in range(3))
    P = draw(st.integers(1, 4))
    eb = draw(st.sampled_from([1, 4, 16]))
    return shape, taps, gridv, P, eb


@settings(max_examples=150, deadline=None)
@given(_descr())
def test_random_descriptors_match_brute_force(case):
    shape, taps, gridv, P, eb = case
    ctx = host_ctx(P)
    k = abi.pk_register_kernel(ctx, "rand", None, [abi.PK_ARG_BUFFER])
    buf = abi.pk_register_buffer(ctx, shape, eb)
    for t in taps:
        abi.pk_declare_affine_access(ctx, k, 0, abi.PK_READ, _to_abi(t))
    for p in range(P):
        box = abi.pk_partition_grid(ctx, k, gridv, p)
        try:
            exp = regions.to_byte_ranges(od.union_elements(taps, box, shape), eb)
        except od.OutOfBounds:
            with pytest.raises(abi.PkError) as ei:
                abi.pk_enumerate(ctx, k, 0, abi.PK_READ, buf, box, (1, 1, 1))
            assert ei.value.name == "PK_ERR_OUT_OF_BOUNDS"
            continue
        assert abi.pk_enumerate(ctx, k, 0, abi.PK_READ, buf, box, (1, 1, 1)) == exp
    abi.pk_finalize(ctx)


# ------------------------------------------------------------ launch sequences vs shadow
def _norm_plan(plan, names):
    out = {}
    for (b, s, d, lo, hi) in plan:
        out.setdefault((names[b], s, d), []).append((lo, hi))
    res = {}
    for key, rs in out.items():
        rs.sort()
        m = []
        for lo, hi in rs:
            if m and lo <= m[-1][1]:
                m[-1] = (m[-1][0], max(hi, m[-1][1]))
            else:
                m.append((lo, hi))
        res[key] = m
    return res


def _run_pair(P, kernel, specs, launches, geom, thread_prog, mode=0, tiles=None, push_arg=None):
    """specs: {name: (shape, eb, uploaded)}; launches: list of [arg binding names or None];
    thread_prog(box) -> oracle access dict keyed by (arg, 'r'/'w'); tiles: NEXT-2 tile shape."""
    ctx = host_ctx(P, mode)
    sh = shadow.Shadow(P, single_owner=bool(mode & abi.PK_MODE_SINGLE_OWNER))
    k = abi.pk_builtin_kernel(ctx, kernel)
    if tiles:
        abi.pk_set_partition_shape(ctx, k, tiles)
    ids, names = {}, {}
    for name, (shape, eb, up) in specs.items():
        host = np.zeros(int(np.prod(shape)) * eb // 4, dtype=np.float32) if up else None
        ids[name] = abi.pk_register_buffer(ctx, shape, eb, host_init=host)
        names[ids[name]] = name
        sh.register(name, int(np.prod(shape)), eb, up)
    grid, blk, sc = geom
    stale_prev = 0
    for binding in launches:
        args = [ids[n] if isinstance(n, str) else n for n in binding]
        abi.pk_launch_partitioned(ctx, k, grid, blk, args, sc)
        per = []
        for p in range(P):
            box = og.tile_box(grid, tiles, p) if tiles else og.partition_box(grid, P, p)
            assert abi.pk_partition_grid(ctx, k, grid, p) == box
            if og.box_empty(box):
                per.append(None)
                continue
            acc = thread_prog(box)
            d = {}
            for (a, tag), el in acc.items():
                name = binding[a]
                r, w = d.get(name, (np.zeros(0, np.int64), np.zeros(0, np.int64)))
                if tag == "r":
                    r = np.union1d(r, el)
                else:
                    w = np.union1d(w, el)
                d[name] = (r, w)
            per.append(d)
        res = sh.launch(per, push=(binding[push_arg],) if (mode & abi.PK_MODE_PUSH) and push_arg is not None else ())
        st_ = abi.pk_get_stats(ctx)
        assert st_["pushed_bytes"] == sh.pushed_bytes
        assert st_["stale_bytes"] - stale_prev == sum(res["stale"])
        stale_prev = st_["stale_bytes"]
        exp_plan = {key: regions.to_byte_ranges(el, specs[key[0]][1]) for key, el in res["copies"].items()}
        assert _norm_plan(abi.pk_last_plan(ctx), names) == exp_plan
        for name, bid in ids.items():
            assert abi.pk_tracker_dump(ctx, bid) == sh.buffers[name].rle()
    st_ = abi.pk_get_stats(ctx)
    abi.pk_finalize(ctx)
    return st_, sh


def _jacobi_case(n, P, iters, mode=0):
    geom = K.jacobi2d_launch(n, n)
    launches = [[("u0" if t % 2 == 0 else "u1"), ("u1" if t % 2 == 0 else "u0"), n, n] for t in range(iters)]
    return _run_pair(P, "jacobi2d", {"u0": ((n, n), 4, True), "u1": ((n, n), 4, True)}, launches, geom,
                     lambda box: regions.jacobi2d(box, geom[1], n, n), mode)


def test_c1_sequence_40800_bytes():
    st_, _ = _jacobi_case(512, 2, 10)
    assert st_["stale_bytes"] == 40800 == 10 * cf.jacobi2d_stale_per_iter(512, 2)
    assert st_["launches"] == 10 and st_["kernel_launches"] == 20


@pytest.mark.parametrize("P,chunks", [(2, [10]), (3, [3, 3]), (3, [1, 5]), (4, [2, 4])])
@pytest.mark.parametrize("mode", [0, abi.PK_MODE_SINGLE_OWNER])
def test_launch_sequence_equals_single_launches(P, chunks, mode):
    """pk_launch_sequence = the same launches one by one (pk_api.h): after every chunk the
    trackers equal the shadow oracle's after that many launches, and the stale bytes and
    launch counts add up (Jacobi 64², misaligned linear upload at P = 3)."""
    n = 64
    geom = K.jacobi2d_launch(n, n)
    iters = sum(chunks)
    sh = shadow.Shadow(P, single_owner=bool(mode & abi.PK_MODE_SINGLE_OWNER))
    for name in ("u0", "u1"):
        sh.register(name, n * n, 4, True)
    rle_after, stale_after = [], []
    for t in range(iters):
        a, b = ("u0", "u1") if t % 2 == 0 else ("u1", "u0")
        per = []
        for p in range(P):
            acc = regions.jacobi2d(og.partition_box(geom[0], P, p), geom[1], n, n)
            d = {}
            for (arg, tag), el in acc.items():
                name = (a, b)[arg]
                r, w = d.get(name, (np.zeros(0, np.int64), np.zeros(0, np.int64)))
                d[name] = (np.union1d(r, el), w) if tag == "r" else (r, np.union1d(w, el))
            per.append(d)
        res = sh.launch(per)
        stale_after.append((stale_after[-1] if stale_after else 0) + sum(res["stale"]))
        rle_after.append({nm: sh.buffers[nm].rle() for nm in ("u0", "u1")})
    ctx = host_ctx(P, mode)
    k = abi.pk_builtin_kernel(ctx, "jacobi2d")
    ids = {nm: abi.pk_register_buffer(ctx, (n, n), 4, host_init=np.zeros(n * n, np.float32)) for nm in ("u0", "u1")}
    t = 0
    for c in chunks:
        seq = []
        for i in range(t, t + c):
            a, b = (ids["u0"], ids["u1"]) if i % 2 == 0 else (ids["u1"], ids["u0"])
            seq.append((k, geom[0], geom[1], [a, b, n, n], geom[2]))
        abi.pk_launch_sequence(ctx, seq)
        t += c
        st_ = abi.pk_get_stats(ctx)
        assert st_["launches"] == t and st_["kernel_launches"] == t * P
        assert st_["stale_bytes"] == stale_after[t - 1]
        for nm, bid in ids.items():
            assert abi.pk_tracker_dump(ctx, bid) == rle_after[t - 1][nm]
    abi.pk_launch_sequence(ctx, [])                              # empty: nothing happens
    assert abi.pk_get_stats(ctx)["launches"] == iters
    with pytest.raises(abi.PkError) as ei:                       # a bad descriptor: PK_ERR_INVALID
        abi.pk_launch_sequence(ctx, [(k + 99, geom[0], geom[1], [ids["u0"], ids["u1"], n, n], geom[2])])
    assert ei.value.name == "PK_ERR_INVALID"
    abi.pk_finalize(ctx)


@pytest.mark.parametrize("mode", [0, abi.PK_MODE_SINGLE_OWNER])
def test_c1_misaligned_p3_both_tracker_modes(mode):
    _jacobi_case(64, 3, 6, mode)


@pytest.mark.parametrize("P", [2, 3, 4, 8])
def test_hotspot_sequence(P):
    h = w = 64
    geom = K.hotspot2d_launch(h, w, 4, 32)
    launches = [[("t0" if t % 2 == 0 else "t1"), "pw", ("t1" if t % 2 == 0 else "t0"), h, w, 4] for t in range(5)]
    st_, sh = _run_pair(P, "hotspot2d_regs", {"t0": ((h, w), 4, True), "t1": ((h, w), 4, False),
                                         "pw": ((h, w), 4, True)}, launches, geom,
                        lambda box: regions.hotspot2d(box, geom[1], h, w, 4))
    # every iteration moves exactly the halo rows when the linear upload of t0 is
    # row-aligned with the partitions (P | 16 blocks); otherwise launch 1 also redistributes
    if 16 % P == 0:
        assert st_["stale_bytes"] == 5 * cf.hotspot2d_stale_per_iter(w, P)
    else:
        assert st_["stale_bytes"] > 5 * cf.hotspot2d_stale_per_iter(w, P)
    assert len(sh.buffers["t0"].rle()) <= 2 * P - 1


@pytest.mark.parametrize("P", [2, 5])
def test_hotspot_tma_sequence(P):
    h, w = 40, 1100
    geom = K.hotspot2d_launch(h, w, 4, 128)
    launches = [[("t0" if t % 2 == 0 else "t1"), "pw", ("t1" if t % 2 == 0 else "t0"), h, w, 4] for t in range(4)]
    _run_pair(P, "hotspot2d", {"t0": ((h, w), 4, True), "t1": ((h, w), 4, False), "pw": ((h, w), 4, True)},
              launches, geom, lambda box: regions.hotspot2d(box, geom[1], h, w, 4))


@pytest.mark.parametrize("P", [2, 3])
def test_heat_sequence(P):
    d, h, w = 12, 8, 64
    geom = K.heat3d_launch(d, h, w, 2, 4)
    launches = [[("u0" if t % 2 == 0 else "u1"), ("u1" if t % 2 == 0 else "u0"), d, h, w, 2] for t in range(4)]
    _run_pair(P, "heat3d", {"u0": ((d, h, w), 4, True), "u1": ((d, h, w), 4, False)}, launches, geom,
              lambda box: regions.heat3d(box, geom[1], d, h, w, 2))


@pytest.mark.parametrize("mode", [0, abi.PK_MODE_SINGLE_OWNER])
def test_nbody_sequence(mode):
    n, P = 1024, 8
    geom = K.nbody_launch(n, 32)            # 8 blocks of 128 bodies: one per partition
    launches = [[("p0" if s % 2 == 0 else "p1"), "v", ("p1" if s % 2 == 0 else "p0"), n] for s in range(3)]
    st_, _ = _run_pair(P, "nbody", {"p0": ((n,), 16, True), "p1": ((n,), 16, False), "v": ((n,), 16, True)},
                       launches, geom, lambda box: regions.nbody(box, geom[1], n, K.NBODY_PER_THREAD), mode)
    assert st_["stale_bytes"] == 3 * cf.nbody_stale_per_step(n, P)


# ------------------------------------------------------------ tile partitions (NEXT-2)
@pytest.mark.parametrize("tiles", [(2, 2, 1), (4, 2, 1), (3, 1, 1), (1, 1, 1)])
def test_jacobi_tile_sequence(tiles):
    n = 64
    P = tiles[0] * tiles[1] * tiles[2]
    geom = K.jacobi2d_launch(n, n)
    launches = [[("u0" if t % 2 == 0 else "u1"), ("u1" if t % 2 == 0 else "u0"), n, n] for t in range(5)]
    st_, _ = _run_pair(P, "jacobi2d", {"u0": ((n, n), 4, True), "u1": ((n, n), 4, True)}, launches, geom,
                       lambda box: regions.jacobi2d(box, geom[1], n, n), tiles=tiles)
    assert st_["launches"] == 5


@pytest.mark.parametrize("kernel,tiles", [("hotspot2d", (2, 2, 1)), ("hotspot2d_regs", (4, 2, 1)),
                                          ("hotspot2d_tb2", (2, 3, 1)), ("hotspot2d_tb2", (3, 2, 1))])
def test_hotspot_tile_sequence(kernel, tiles):
    h, w = 48, 1600
    P = tiles[0] * tiles[1]
    prog = regions.hotspot2d_tb2 if kernel == "hotspot2d_tb2" else regions.hotspot2d
    bdx = 32 if kernel == "hotspot2d_regs" else 128
    geom = K.hotspot2d_launch(h, w, 4, bdx)
    launches = [[("t0" if t % 2 == 0 else "t1"), "pw", ("t1" if t % 2 == 0 else "t0"), h, w, 4] for t in range(4)]
    _run_pair(P, kernel, {"t0": ((h, w), 4, True), "t1": ((h, w), 4, False), "pw": ((h, w), 4, True)},
              launches, geom, lambda box: prog(box, geom[1], h, w, 4), tiles=tiles)


def test_heat_tile_sequence():
    d, h, w = 12, 16, 64
    tiles = (1, 2, 2)
    geom = K.heat3d_launch(d, h, w, 2, 4)
    launches = [[("u0" if t % 2 == 0 else "u1"), ("u1" if t % 2 == 0 else "u0"), d, h, w, 2] for t in range(4)]
    _run_pair(4, "heat3d", {"u0": ((d, h, w), 4, True), "u1": ((d, h, w), 4, False)}, launches, geom,
              lambda box: regions.heat3d(box, geom[1], d, h, w, 2), tiles=tiles)


def test_tile_shape_validation_and_reset():
    ctx = host_ctx(4)
    k = abi.pk_builtin_kernel(ctx, "jacobi2d")
    for bad in ((2, 1, 1), (0, 4, 1), (2, 2, 2), (-2, -2, 1)):
        with pytest.raises(abi.PkError):
            abi.pk_set_partition_shape(ctx, k, bad)
    abi.pk_set_partition_shape(ctx, k, (2, 2, 1))
    assert abi.pk_partition_grid(ctx, k, (16, 64, 1), 3) == (0, 1, 32, 64, 8, 16)
    abi.pk_set_partition_shape(ctx, k, None)
    assert abi.pk_partition_grid(ctx, k, (16, 64, 1), 3) == og.partition_box((16, 64, 1), 4, 3)
    abi.pk_finalize(ctx)


def test_hotspot_tile_closed_form_through_library():
    h, w = 64, 2048
    tiles = (4, 2, 1)
    geom = K.hotspot2d_launch(h, w, 4, 128)
    ctx = host_ctx(8)
    k = abi.pk_builtin_kernel(ctx, "hotspot2d")
    abi.pk_set_partition_shape(ctx, k, tiles)
    t0 = abi.pk_register_buffer(ctx, (h, w), 4, host_init=np.zeros(h * w, np.float32))
    t1 = abi.pk_register_buffer(ctx, (h, w), 4)
    pw = abi.pk_register_buffer(ctx, (h, w), 4, host_init=np.zeros(h * w, np.float32))
    per = []
    for t in range(6):
        a, b = (t0, t1) if t % 2 == 0 else (t1, t0)
        s0 = abi.pk_get_stats(ctx)["stale_bytes"]
        abi.pk_launch_partitioned(ctx, k, geom[0], geom[1], [a, pw, b, h, w, 4], geom[2])
        per.append(abi.pk_get_stats(ctx)["stale_bytes"] - s0)
    assert per[2:] == [cf.hotspot2d_tile_stale_per_iter(h, w, 4, 2)] * 4
    abi.pk_finalize(ctx)


# ------------------------------------------------------------ error paths / modes
def test_write_overlap_rejected_before_anything():
    ctx = host_ctx(2)
    k = abi.pk_register_kernel(ctx, "bad", None, [abi.PK_ARG_BUFFER])
    buf = abi.pk_register_buffer(ctx, (64,), 4)
    # every block writes [b*8, b*8+12): blocks overlap -> partitions overlap
    abi.pk_declare_affine_access(ctx, k, 0, abi.PK_WRITE, abi.affine_access([abi.dim_map(0, 8, 12, guard=(0, 64))]))
    before = abi.pk_tracker_dump(ctx, buf)
    with pytest.raises(abi.PkError) as ei:
        abi.pk_launch_partitioned(ctx, k, (8, 1, 1), (1, 1, 1), [buf])
    assert ei.value.name == "PK_ERR_WRITE_OVERLAP"
    assert abi.pk_tracker_dump(ctx, buf) == before
    assert abi.pk_get_stats(ctx)["launches"] == 0
    abi.pk_finalize(ctx)


def test_out_of_bounds_overflow_and_non_separable():
    ctx = host_ctx(1)
    k = abi.pk_register_kernel(ctx, "oob", None, [abi.PK_ARG_BUFFER])
    buf = abi.pk_register_buffer(ctx, (10,), 4)
    abi.pk_declare_affine_access(ctx, k, 0, abi.PK_READ, abi.affine_access([abi.dim_map(0, 4, 4, offset=1)]))
    with pytest.raises(abi.PkError) as ei:
        abi.pk_launch_partitioned(ctx, k, (3, 1, 1), (1, 1, 1), [buf])
    assert ei.value.name == "PK_ERR_OUT_OF_BOUNDS"
    k2 = abi.pk_register_kernel(ctx, "ovf", None, [abi.PK_ARG_BUFFER])
    abi.pk_declare_affine_access(ctx, k2, 0, abi.PK_READ,
                                 abi.affine_access([abi.dim_map(0, abi.expr(1 << 62), 4, clamp=True)]))
    with pytest.raises(abi.PkError) as ei:
        abi.pk_launch_partitioned(ctx, k2, (3, 1, 1), (1, 1, 1), [buf])
    assert ei.value.name == "PK_ERR_OVERFLOW"
    k3 = abi.pk_register_kernel(ctx, "nonsep", None, [abi.PK_ARG_BUFFER])
    b2 = abi.pk_register_buffer(ctx, (4, 4), 4)
    with pytest.raises(abi.PkError) as ei:
        abi.pk_declare_affine_access(ctx, k3, 0, abi.PK_READ,
                                     abi.affine_access([abi.dim_map(0, 1, 1), abi.dim_map(0, 1, 1)]))
    assert ei.value.name == "PK_ERR_INVALID"
    del b2
    abi.pk_finalize(ctx)


def test_no_tracking_and_no_transfers_modes():
    # gamma: no resolution, no tracker -> no stale bytes counted, tracker untouched
    n = 64
    ctx = host_ctx(2, abi.PK_MODE_NO_TRACKING)
    pr, _ = K.jacobi2d_program(ctx, np.zeros((n, n), np.float32), 4)
    s = abi.pk_get_stats(ctx)
    assert s["stale_bytes"] == 0 and s["launches"] == 4
    abi.pk_finalize(ctx)
    # beta: resolution + tracking still run
    ctx = host_ctx(2, abi.PK_MODE_NO_TRANSFERS)
    K.jacobi2d_program(ctx, np.zeros((n, n), np.float32), 4)
    s = abi.pk_get_stats(ctx)
    assert s["stale_bytes"] == 4 * cf.jacobi2d_stale_per_iter(n, 2) and s["moved_bytes"] == 0
    abi.pk_finalize(ctx)


def test_h2d_linear_distribution_tracker():
    ctx = host_ctx(3)
    b = abi.pk_register_buffer(ctx, (10,), 4, host_init=np.zeros(10, np.float32))
    sb = shadow.ShadowBuffer(10, 4, 3)
    sb.h2d_linear()
    assert abi.pk_tracker_dump(ctx, b) == sb.rle()
    b2 = abi.pk_register_buffer(ctx, (7, 3), 4)
    assert abi.pk_tracker_dump(ctx, b2) == [(0, 84, 7)]           # reading Q3
    abi.pk_finalize(ctx)


@pytest.mark.parametrize("P", [1, 3, 5])
def test_h2d_async_same_tracker_effect(P):
    """pk_copy_from_host_async distributes like pk_copy_from_host (shadow oracle's linear H2D)."""
    ctx = host_ctx(P)
    b = abi.pk_register_buffer(ctx, (23, 3), 4)
    abi.pk_copy_from_host_async(ctx, b, np.zeros((23, 3), np.float32))
    sb = shadow.ShadowBuffer(69, 4, P)
    sb.h2d_linear()
    assert abi.pk_tracker_dump(ctx, b) == sb.rle()
    with pytest.raises(abi.PkError):
        abi.pk_sync_to_host_async(ctx, b, np.zeros((23, 3), np.float32))   # a host-only context holds no data
    abi.pk_finalize(ctx)


@pytest.mark.parametrize("m,n,k", [(300, 520, 200), (1024, 512, 64)])
@pytest.mark.parametrize("P", [1, 2, 3])
def test_gemm_regions(m, n, k, P):
    ctx = host_ctx(P)
    kern = abi.pk_builtin_kernel(ctx, "sgemm_tf32x3")
    bufs = [abi.pk_register_buffer(ctx, s, 4) for s in ((m, k), (k, n), (m, n))]
    grid, blk, sc = K.sgemm_launch(m, n, k)
    for p in range(P):
        box = abi.pk_partition_grid(ctx, kern, grid, p)
        lib = _lib_sets(ctx, kern, 6, bufs + [None] * 3, box, blk, sc)
        ora = _oracle_sets(regions.gemm(box, m, n, k, K.GEMM_BM, K.GEMM_BN), {0: 4, 1: 4, 2: 4})
        assert lib == ora
    abi.pk_finalize(ctx)


def test_gemm_b_broadcast_stale_bytes():
    m = n = k = 512
    P = 4
    ctx = host_ctx(P)
    K.sgemm_program(ctx, np.zeros((m, k), np.float32), np.zeros((k, n), np.float32), launches=2)
    s = abi.pk_get_stats(ctx)
    # first launch: every partition pulls the (P-1)/P of B it lacks; A's linear upload
    # matches the row partition; the second launch moves nothing (validity map, Q4)
    assert s["stale_bytes"] == cf.gemm_stale(k, n, P)
    abi.pk_finalize(ctx)


# ------------------------------------------------------------ read-pattern-aware placement (NEXT-1)
@pytest.mark.parametrize("P", [2, 3, 4])
def test_placement_for_gemm_b_and_hotspot_halo(P):
    # GEMM: B placed where the launch reads it -> the launch moves nothing
    m, n, k = 768, 256, 256                  # 6 row tiles: no empty partition for P <= 4
    ctx = host_ctx(P)
    pr = K.Problem(ctx, "sgemm_tf32x3")
    a = pr.buffer((m, k), 4)
    b = pr.buffer((k, n), 4)
    c = pr.buffer((m, n), 4)
    grid, blk, sc = K.sgemm_launch(m, n, k)
    abi.pk_copy_from_host_for(ctx, a, np.zeros((m, k), np.float32), pr.k, 0, grid, blk, sc)
    abi.pk_copy_from_host_for(ctx, b, np.zeros((k, n), np.float32), pr.k, 1, grid, blk, sc)
    assert abi.pk_tracker_dump(ctx, b) == [(0, k * n * 4, (1 << P) - 1)]
    pr.launch(grid, blk, [a, b, c, m, n, k], sc)
    assert abi.pk_get_stats(ctx)["stale_bytes"] == 0
    abi.pk_finalize(ctx)
    # Hotspot: halo rows land on both neighbours; tracker == shadow oracle; first launch moves nothing
    h, w = 40, 1100
    ctx = host_ctx(P)
    geom = K.hotspot2d_launch(h, w, 4, 128)
    pr = K.Problem(ctx, "hotspot2d")
    t0 = pr.buffer((h, w), 4)
    t1 = pr.buffer((h, w), 4)
    pw = pr.buffer((h, w), 4)
    abi.pk_copy_from_host_for(ctx, t0, np.zeros((h, w), np.float32), pr.k, 0, *geom)
    sb = shadow.ShadowBuffer(h * w, 4, P)
    sb.h2d_for([regions.hotspot2d(og.partition_box(geom[0], P, p), geom[1], h, w, 4)[(0, "r")]
                for p in range(P)])
    assert abi.pk_tracker_dump(ctx, t0) == sb.rle()
    pr.launch(geom[0], geom[1], [t0, pw, t1, h, w, 4], geom[2])
    assert abi.pk_get_stats(ctx)["stale_bytes"] == 0
    abi.pk_finalize(ctx)


# ------------------------------------------------------------ temporally blocked Hotspot (NEXT-3)
@pytest.mark.parametrize("h,w,ty", [(33, 1100, 4), (200, 1028, 16), (5, 8, 64)])
@pytest.mark.parametrize("P", [1, 2, 3, 7])
def test_hotspot_tb2_regions(h, w, ty, P):
    ctx = host_ctx(P)
    k = abi.pk_builtin_kernel(ctx, "hotspot2d_tb2")
    bufs = [abi.pk_register_buffer(ctx, (h, w), 4) for _ in range(3)]
    grid, blk, sc = K.hotspot2d_launch(h, w, ty, 128)
    for p in range(P):
        box = abi.pk_partition_grid(ctx, k, grid, p)
        lib = _lib_sets(ctx, k, 6, bufs + [None] * 3, box, blk, sc)
        ora = _oracle_sets(regions.hotspot2d_tb2(box, blk, h, w, ty), {0: 4, 1: 4, 2: 4})
        assert lib == ora
    abi.pk_finalize(ctx)


@pytest.mark.parametrize("h,w,ty,k", [(33, 1100, 4, 4), (200, 1028, 16, 3), (5, 8, 64, 2), (40, 960, 7, 4),
                                      (41, 1000, 9, 6), (70, 900, 16, 8), (20, 452, 5, 5)])
@pytest.mark.parametrize("P", [1, 2, 3, 7])
def test_hotspot_tbk_regions(h, w, ty, k, P):
    """K-sweep Hotspot: one dilated tap per argument == brute-force (2K+1)^2 / (2K-1)^2 squares
    (logical blocks 480 columns wide for K <= 4, 448 for K = 5..8)."""
    ctx = host_ctx(P)
    kk = abi.pk_builtin_kernel(ctx, "hotspot2d_tbk")
    bufs = [abi.pk_register_buffer(ctx, (h, w), 4) for _ in range(3)]
    grid, blk, sc = K.hotspot2d_tbk_launch(h, w, ty, k)
    for p in range(P):
        box = abi.pk_partition_grid(ctx, kk, grid, p)
        lib = _lib_sets(ctx, kk, 6, bufs + [None] * 3, box, blk, sc)
        ora = _oracle_sets(regions.hotspot2d_tbk(box, blk, h, w, ty, k, cols=480 if k <= 4 else 448),
                           {0: 4, 1: 4, 2: 4})
        assert lib == ora
    abi.pk_finalize(ctx)


@pytest.mark.parametrize("P", [2, 4])
def test_hotspot_tb2_sequence(P):
    h, w = 64, 1024
    geom = K.hotspot2d_launch(h, w, 4, 128)
    launches = [[("t0" if t % 2 == 0 else "t1"), "pw", ("t1" if t % 2 == 0 else "t0"), h, w, 4] for t in range(4)]
    st_, _ = _run_pair(P, "hotspot2d_tb2", {"t0": ((h, w), 4, True), "t1": ((h, w), 4, False),
                                            "pw": ((h, w), 4, True)}, launches, geom,
                       lambda box: regions.hotspot2d_tb2(box, geom[1], h, w, 4))
    # 2 halo rows of temp each way per boundary per launch, + the 1-row power halo once
    assert st_["stale_bytes"] == 4 * 2 * cf.hotspot2d_stale_per_iter(w, P) + cf.hotspot2d_stale_per_iter(w, P)


# ------------------------------------------------------------ fused halo push (PK_MODE_PUSH, reading Q25)
@pytest.mark.parametrize("P", [2, 3, 4])
def test_push_jacobi_sequence_vs_shadow(P):
    """Tracker, plans, stale and pushed bytes with the predictive push == shadow oracle;
    after the first two launches nothing is stale any more."""
    n, iters = 64, 8
    geom = K.jacobi2d_launch(n, n)
    launches = [[("u0" if t % 2 == 0 else "u1"), ("u1" if t % 2 == 0 else "u0"), n, n] for t in range(iters)]
    st_, sh = _run_pair(P, "jacobi2d", {"u0": ((n, n), 4, True), "u1": ((n, n), 4, True)}, launches, geom,
                        lambda box: regions.jacobi2d(box, geom[1], n, n), mode=abi.PK_MODE_PUSH, push_arg=1)
    per_iter = cf.jacobi2d_stale_per_iter(n, P)
    pull2, _ = _jacobi_case(n, P, 2)                      # launches 1 and 2 pull, then everything is pushed
    assert st_["stale_bytes"] == pull2["stale_bytes"]
    if P == 2:                                            # (P = 3 also repairs the linear H2D split, reading Q2)
        assert st_["stale_bytes"] == 2 * per_iter
    assert st_["pushed_bytes"] == (iters - 1) * per_iter


@pytest.mark.parametrize("kernel,P", [("hotspot2d", 2), ("hotspot2d", 4), ("hotspot2d_tbk", 3)])
def test_push_hotspot_sequence_vs_shadow(kernel, P):
    h, w = 64, 1024
    if kernel == "hotspot2d_tbk":
        geom = K.hotspot2d_tbk_launch(h, w, 8, 4)
        prog = lambda box: regions.hotspot2d_tbk(box, geom[1], h, w, 8, 4)
    else:
        geom = K.hotspot2d_launch(h, w, 4, 128)
        prog = lambda box: regions.hotspot2d(box, geom[1], h, w, 4)
    launches = [[("t0" if t % 2 == 0 else "t1"), "pw", ("t1" if t % 2 == 0 else "t0"), h, w, geom[2][2]]
                for t in range(6)]
    st_, _ = _run_pair(P, kernel, {"t0": ((h, w), 4, True), "t1": ((h, w), 4, False), "pw": ((h, w), 4, True)},
                       launches, geom, prog, mode=abi.PK_MODE_PUSH, push_arg=2)
    assert st_["pushed_bytes"] > 0


def test_push_heat_sequence_vs_shadow():
    d, h, w = 16, 8, 64
    geom = K.heat3d_launch(d, h, w, 4, 8)
    launches = [[("u0" if t % 2 == 0 else "u1"), ("u1" if t % 2 == 0 else "u0"), d, h, w, 4] for t in range(5)]
    st_, _ = _run_pair(2, "heat3d", {"u0": ((d, h, w), 4, True), "u1": ((d, h, w), 4, False)}, launches, geom,
                       lambda box: regions.heat3d(box, geom[1], d, h, w, 4), mode=abi.PK_MODE_PUSH, push_arg=1)
    assert st_["pushed_bytes"] == 4 * cf.heat3d_stale_per_iter(h, w, 2)   # launches 2..5 push


def test_push_tiles_fall_back_to_pull():
    """A 2x2 tile split makes W_q n R_p per-row pieces (> 4 runs): no push, everything pulled."""
    n = 64
    geom = K.jacobi2d_launch(n, n)
    launches = [[("u0" if t % 2 == 0 else "u1"), ("u1" if t % 2 == 0 else "u0"), n, n] for t in range(4)]
    st_, _ = _run_pair(4, "jacobi2d", {"u0": ((n, n), 4, True), "u1": ((n, n), 4, True)}, launches, geom,
                       lambda box: regions.jacobi2d(box, geom[1], n, n), mode=abi.PK_MODE_PUSH, push_arg=1,
                       tiles=(2, 2, 1))
    assert st_["pushed_bytes"] == 0


# ------------------------------------------------------------ two-sweep heat (NEXT-3, 3-D)
@pytest.mark.parametrize("d,h,w,zc", [(10, 30, 260, 4), (7, 50, 124, 128), (3, 5, 8, 2)])
@pytest.mark.parametrize("P", [1, 2, 3, 5])
def test_heat3d_tb2_regions(d, h, w, zc, P):
    """One dilated tap == brute-force clamped 5x5x5 cubes of every owned cell."""
    ctx = host_ctx(P)
    kk = abi.pk_builtin_kernel(ctx, "heat3d_tb2")
    bufs = [abi.pk_register_buffer(ctx, (d, h, w), 4) for _ in range(2)]
    grid, blk, sc = K.heat3d_tb2_launch(d, h, w, zc)
    for p in range(P):
        box = abi.pk_partition_grid(ctx, kk, grid, p)
        lib = _lib_sets(ctx, kk, 6, bufs + [None] * 4, box, blk, sc)
        ora = _oracle_sets(regions.heat3d_tb2(box, d, h, w, zc, rows=16), {0: 4, 1: 4})   # 120 x 16 x zc blocks
        assert lib == ora
    abi.pk_finalize(ctx)


@pytest.mark.parametrize("d,h,w,zc", [(10, 30, 260, 4), (7, 50, 124, 128), (3, 5, 8, 2)])
@pytest.mark.parametrize("P", [1, 2, 3, 5])
def test_heat3d_tb3_regions(d, h, w, zc, P):
    """Three sweeps per launch: one tap dilated by 3 == brute-force clamped 7x7x7 cubes."""
    ctx = host_ctx(P)
    kk = abi.pk_builtin_kernel(ctx, "heat3d_tb3")
    bufs = [abi.pk_register_buffer(ctx, (d, h, w), 4) for _ in range(2)]
    grid, blk, sc = K.heat3d_tb3_launch(d, h, w, zc)
    for p in range(P):
        box = abi.pk_partition_grid(ctx, kk, grid, p)
        lib = _lib_sets(ctx, kk, 6, bufs + [None] * 4, box, blk, sc)
        ora = _oracle_sets(regions.heat3d_tb2(box, d, h, w, zc, rows=16, sweeps=3), {0: 4, 1: 4})
        assert lib == ora
    abi.pk_finalize(ctx)


@pytest.mark.parametrize("h,w,k", [(64, 64, 1), (64, 64, 5), (70, 100, 10), (33, 31, 16), (3, 3, 2)])
@pytest.mark.parametrize("P", [1, 2, 3])
def test_jacobi2d_tb_regions(h, w, k, P):
    """K sweeps per launch: the dilated, clamped window and the interior writes == brute force."""
    ctx = host_ctx(P)
    kk = abi.pk_builtin_kernel(ctx, "jacobi2d_tb")
    bufs = [abi.pk_register_buffer(ctx, (h, w), 4) for _ in range(2)]
    grid, blk, sc = K.jacobi2d_tb_launch(h, w, k)
    for p in range(P):
        box = abi.pk_partition_grid(ctx, kk, grid, p)
        lib = _lib_sets(ctx, kk, 5, bufs + [None] * 3, box, blk, sc)
        ora = _oracle_sets(regions.jacobi2d_tb(box, h, w, k), {0: 4, 1: 4})
        assert lib == ora
    abi.pk_finalize(ctx)


# ------------------------------------------------------------------ degenerate cases
def test_degenerate_buffers_and_grids():
    """A zero-element buffer holds no segments; an empty grid launches nothing and moves
    nothing; a one-block grid at P = 3 leaves two empty partitions (reading Q1), which are
    not launched, and its stale bytes equal the shadow oracle's."""
    ctx = host_ctx(3)
    z = abi.pk_register_buffer(ctx, (0, 16), 4)
    assert abi.pk_tracker_dump(ctx, z) == []
    k = abi.pk_builtin_kernel(ctx, "jacobi2d")
    u = np.arange(16, dtype=np.float32).reshape(4, 4)
    b0 = abi.pk_register_buffer(ctx, (4, 4), 4, host_init=u)
    b1 = abi.pk_register_buffer(ctx, (4, 4), 4, host_init=u)
    abi.pk_launch_partitioned(ctx, k, (0, 1, 1), (32, 8, 1), [b0, b1, 4, 4], [4, 4])
    st = abi.pk_get_stats(ctx)
    assert st["kernel_launches"] == 0 and st["stale_bytes"] == 0 and st["moved_bytes"] == 0
    abi.pk_finalize(ctx)
    geom = ((1, 1, 1), (32, 8, 1), [4, 4])
    st_, _ = _run_pair(3, "jacobi2d", {"u0": ((4, 4), 4, True), "u1": ((4, 4), 4, True)},
                       [["u0", "u1", 4, 4], ["u1", "u0", 4, 4]], geom,
                       lambda box: regions.jacobi2d(box, (32, 8), 4, 4))
    assert st_["kernel_launches"] == 2                      # one partition launched per launch


def test_no_collectives_mode_flag_and_allgather_plan_shape():
    """PK_MODE_NO_COLLECTIVES (one process, distinct GPUs: whole-buffer reads as peer copies
    instead of one ncclAllGather) is a known flag; the flag after it is not.  The
    N-body position plan at P = 4 is the all-gather pattern the one-process path detects:
    every partition pulls every other partition's linear slab, P(P-1) copies of |pos|/P."""
    ctx = host_ctx(4, abi.PK_MODE_NO_COLLECTIVES)
    assert abi.pk_get_mode(ctx) == abi.PK_MODE_NO_COLLECTIVES
    with pytest.raises(RuntimeError):
        abi.pk_set_mode(ctx, 1 << 9)
    abi.pk_finalize(ctx)
    n, P = 1024, 4
    ctx = host_ctx(P)
    k = abi.pk_builtin_kernel(ctx, "nbody")
    p0 = abi.pk_register_buffer(ctx, (n,), 16, host_init=np.zeros((n, 4), np.float32))
    p1 = abi.pk_register_buffer(ctx, (n,), 16)
    v = abi.pk_register_buffer(ctx, (n,), 16, host_init=np.zeros((n, 4), np.float32))
    grid, blk, sc = K.nbody_launch(n, 32)
    abi.pk_launch_partitioned(ctx, k, grid, blk, [p0, v, p1, n], sc)
    plan = abi.pk_last_plan(ctx)
    slab = n * 16 // P
    assert sorted((s, d, b, e) for buf, s, d, b, e in plan if buf == p0) == sorted(
        (q, p, q * slab, (q + 1) * slab) for p in range(P) for q in range(P) if q != p)
    assert abi.pk_get_stats(ctx)["collectives"] == 0     # host-only: plans, no transport
    abi.pk_finalize(ctx)
