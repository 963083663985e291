"""Pins of the oracle's brute-force regions, grid split and shadow tracker (no GPU).

Checked against hand derivations from the kernel definitions,
closed-form stale-byte minima (oracle/closed_forms.py) and the
paper's qualitative statements (Fig. 3 text P:L561-566; fragmentation P:L860-870;
redundant transfers without shared copies P:L929-931).
"""
import numpy as np
import pytest

from oracle import closed_forms as cf
from oracle import grid, regions, shadow


def _rng(a, b):
    return list(range(a, b))


# ------------------------------ grid split (Q1) ------------------------------
def test_partition_rule():
    assert grid.split_dim((16, 64, 1)) == grid.Y
    assert grid.split_dim((8, 128, 16)) == grid.Z
    assert grid.split_dim((4096, 1, 1)) == grid.X
    assert grid.split_dim((1, 1, 1)) == grid.X
    boxes = [grid.partition_box((16, 64, 1), 2, p) for p in range(2)]
    assert boxes == [(0, 1, 0, 32, 0, 16), (0, 1, 32, 64, 0, 16)]
    # balanced floor split, empty partitions when P > G
    assert [grid.partition_box((1, 3, 1), 5, p)[2:4] for p in range(5)] == \
        [(0, 0), (0, 1), (1, 1), (1, 2), (2, 3)]
    covered = []
    for p in range(7):
        b = grid.partition_box((5, 100, 1), 7, p)
        covered += _rng(b[2], b[3])
    assert covered == _rng(0, 100)


def test_tile_rule():
    # NEXT-2 tile partitions (reading Q24): x fastest, each dim split by the floor rule
    assert [grid.tile_box((16, 64, 1), (2, 2, 1), p) for p in range(4)] == [
        (0, 1, 0, 32, 0, 8), (0, 1, 0, 32, 8, 16), (0, 1, 32, 64, 0, 8), (0, 1, 32, 64, 8, 16)]
    # (1, P, 1) tiles of a 2-D grid are the 1-D row slabs
    for p in range(3):
        assert grid.tile_box((5, 100, 1), (1, 3, 1), p) == grid.partition_box((5, 100, 1), 3, p)
    # every block of the grid lies in exactly one tile (brute force, ragged sizes)
    for g, t in (((7, 5, 3), (2, 2, 2)), ((3, 9, 1), (3, 2, 1)), ((1, 4, 6), (1, 2, 3)), ((2, 2, 2), (3, 1, 1))):
        seen = {}
        for p in range(t[0] * t[1] * t[2]):
            z0, z1, y0, y1, x0, x1 = grid.tile_box(g, t, p)
            for z in range(z0, z1):
                for y in range(y0, y1):
                    for x in range(x0, x1):
                        assert (x, y, z) not in seen
                        seen[(x, y, z)] = p
        assert len(seen) == g[0] * g[1] * g[2]


# ----------------------- C1 worked example (hand derived) -----------------------
def test_c1_partition0_read_and_write_sets():
    n = 512
    acc = regions.jacobi2d(grid.partition_box((16, 64, 1), 2, 0), (32, 8), n, n)
    # Partition 0 = rows [0, 256).  Threads on rows 1..255, cols 1..510 (Dirichlet).
    # Row 0: only the 'up' tap of row 1 -> interior cols 1..510.
    # Rows 1..255: left tap of col 1 reaches col 0, right tap of col 510 reaches 511.
    # Row 256: only the 'down' tap of row 255 -> interior.
    r = regions.to_byte_ranges(acc[(0, "r")], 1)
    assert r == [(1, 511), (512, 131072), (131073, 131583)]
    w = regions.to_byte_ranges(acc[(1, "w")], 1)
    assert len(w) == 255 and w[0] == (513, 1023) and w[-1] == (255 * 512 + 1, 255 * 512 + 511)
    assert sum(e - s for s, e in w) == 130050
    acc1 = regions.jacobi2d(grid.partition_box((16, 64, 1), 2, 1), (32, 8), n, n)
    assert regions.to_byte_ranges(acc1[(0, "r")], 1) == [(130561, 131071), (131072, 261632), (261633, 262143)]


def test_hotspot_heat_nbody_gemm_sets_shape():
    # hotspot: clamped 5-point -> one contiguous range rows [r0-1, r1+1) clamped
    acc = regions.hotspot2d((0, 1, 2, 5, 0, 1), (16,), 40, 64, 4)   # rows 8..19
    assert regions.to_byte_ranges(acc[(0, "r")], 1) == [(7 * 64, 21 * 64)]
    assert regions.to_byte_ranges(acc[(1, "r")], 1) == [(8 * 64, 20 * 64)]
    assert regions.to_byte_ranges(acc[(2, "w")], 1) == [(8 * 64, 20 * 64)]
    # ragged tail: last block row clipped to H; the top partition clamps at row 0
    acc = regions.hotspot2d((0, 1, 0, 1, 0, 1), (16,), 3, 64, 4)
    assert regions.to_byte_ranges(acc[(0, "r")], 1) == [(0, 3 * 64)]
    # heat: planes
    acc = regions.heat3d((1, 2, 0, 2, 0, 1), (8, 4), 10, 8, 32, 3)   # planes 3..5
    assert regions.to_byte_ranges(acc[(0, "r")], 1) == [(2 * 256, 7 * 256)]
    assert regions.to_byte_ranges(acc[(1, "w")], 1) == [(3 * 256, 6 * 256)]
    # nbody: everything read, own slab written
    acc = regions.nbody((0, 1, 0, 1, 1, 2), (64,), 300)      # 2 bodies per thread
    assert regions.to_byte_ranges(acc[(0, "r")], 16) == [(0, 300 * 16)]
    assert regions.to_byte_ranges(acc[(2, "w")], 16) == [(128 * 16, 256 * 16)]
    acc = regions.nbody((0, 1, 0, 1, 2, 3), (64,), 300)      # ragged last block
    assert regions.to_byte_ranges(acc[(1, "w")], 16) == [(256 * 16, 300 * 16)]
    # gemm: A row band, B whole, C tile rows
    acc = regions.gemm((0, 1, 1, 2, 0, 2), 10, 12, 5, 4, 8)
    assert regions.to_byte_ranges(acc[(0, "r")], 1) == [(20, 40)]
    assert regions.to_byte_ranges(acc[(1, "r")], 1) == [(0, 60)]
    assert regions.to_byte_ranges(acc[(2, "w")], 1) == [(48, 96)]


# ------------------------------ shadow tracker ------------------------------
def _jacobi_run(n, nparts, iters, single=False, block=(32, 8)):
    sh = shadow.Shadow(nparts, single)
    sh.register("u0", n * n, 4, True)
    sh.register("u1", n * n, 4, True)
    g = ((n + block[0] - 1) // block[0], (n + block[1] - 1) // block[1], 1)
    per_iter = []
    for t in range(iters):
        a, b = ("u0", "u1") if t % 2 == 0 else ("u1", "u0")
        per = []
        for p in range(nparts):
            box = grid.partition_box(g, nparts, p)
            if grid.box_empty(box):
                per.append(None)
                continue
            acc = regions.jacobi2d(box, block, n, n)
            per.append({a: (acc[(0, "r")], None), b: (None, acc[(1, "w")])})
        per_iter.append(sum(sh.launch(per)["stale"]))
    return sh, per_iter


def test_c1_stale_bytes_40800():
    sh, per = _jacobi_run(512, 2, 10)
    assert per == [cf.jacobi2d_stale_per_iter(512, 2)] * 10
    assert sh.stale_bytes == 40800


@pytest.mark.parametrize("k", [1, 3, 5])
def test_jacobi2d_tb_stale_hand_derived(k):
    """K sweeps per launch (jacobi2d_tb), 64^2, P = 2 (row slabs [0, 32), [32, 64), aligned
    with the linear H2D split).  Hand count: each partition's window reaches K full rows
    into the other (all 64 columns, boundary columns included).  Launch 1 reads u0 and
    launch 2 reads u1 as uploaded: both directions lack K full rows, 2 K 64 4 B.  From
    launch 3 on, the boundary columns of those rows were copied once (validity mode: the
    reader became a co-holder, and they are never rewritten), so only the K interior row
    segments rewritten by the owner move: 2 K 62 4 B."""
    n, P = 64, 2
    sh = shadow.Shadow(P)
    sh.register("u0", n * n, 4, True)
    sh.register("u1", n * n, 4, True)
    g = (2, 2, 1)                       # 32 x 32 logical blocks
    per_launch = []
    for t in range(5):
        a, b = ("u0", "u1") if t % 2 == 0 else ("u1", "u0")
        per = []
        for p in range(P):
            acc = regions.jacobi2d_tb(grid.partition_box(g, P, p), n, n, k)
            per.append({a: (acc[(0, "r")], None), b: (None, acc[(1, "w")])})
        per_launch.append(sum(sh.launch(per)["stale"]))
    full, inner = 2 * k * 64 * 4, 2 * k * 62 * 4
    assert per_launch == [full, full, inner, inner, inner]


def test_misaligned_h2d_redistribution_and_paper_mode_redundancy():
    """Jacobi 64^2, P = 3 (SURVEY §8(c) Q2 / paper-vs-validity pin).

    Hand derivation.  Grid (2, 8) blocks of 32x8 -> row slabs [0,16), [16,40), [40,64);
    the linear H2D split of 4096 elements is [0,1365), [1365,2730), [2730,4096), i.e. the
    slab boundaries fall at (row 21, col 21) and (row 42, col 42).  A partition on rows
    [r0, r1) reads row r0-1 and row r1 interior (62 cells) and rows r0..r1-1 in full,
    clipped to interior thread rows 1..62.
      launch 1 (reads u0 as uploaded): p0 holds all it reads; p1 lacks row 15 interior (62),
        rows 16-20 (5 x 64) and row 21 cols 0-20 (21) = 403; p2 lacks row 39 interior
        (62), rows 40-41 (128), row 42 cols 0-41 (42) = 232.  635 cells = 2,540 B.
      launch 2 (reads u1: interior written by launch 1's slabs, border cells still
        linear): p0 lacks row 16 interior (62); p1 row 15 and row 40 interior (124) plus
        the border cells (col 0 / 63) of rows 16-20 and (21, 0), held by p0 (11); p2 row
        39 interior (62) plus (40, 0), (40, 63), (41, 0), (41, 63), (42, 0) held by p1 (5).
        264 cells = 1,056 B.
      launch 3+ (reads the buffer read in launch 1, whose border cells the readers now
        co-hold): only the 4 interior halo rows cross: 248 cells = 992 B.  Without shared
        copies (the paper's tracker) those 16 border cells are fetched again every time:
        1,056 B per launch.
    """
    _, per = _jacobi_run(64, 3, 6)
    assert per == [2540, 1056, 992, 992, 992, 992]
    _, per_so = _jacobi_run(64, 3, 6, single=True)
    assert per_so == [2540, 1056, 1056, 1056, 1056, 1056]


def test_gemm_launched_twice_single_owner_vs_validity():
    """Paper-vs-validity pin: the same GEMM launched twice on unchanged
    operands.  Every partition reads all of B (k x n), of which it holds its 1/P linear
    slab: launch 1 moves (P-1) |B|.  With shared copies the readers keep B and launch 2
    moves nothing (1x); the paper's single-owner tracker fetches it again (2x).  A's row
    band equals the linear slab when the tile rows divide M."""
    m, n, k, bm, bn, P = 32, 24, 20, 4, 8, 4
    g = ((n + bn - 1) // bn, m // bm, 1)
    res = {}
    for single in (False, True):
        sh = shadow.Shadow(P, single)
        sh.register("A", m * k, 4, True)
        sh.register("B", k * n, 4, True)
        sh.register("C", m * n, 4, False)
        per_launch = []
        for _ in range(2):
            per = []
            for p in range(P):
                acc = regions.gemm(grid.partition_box(g, P, p), m, n, k, bm, bn)
                per.append({"A": (acc[(0, "r")], None), "B": (acc[(1, "r")], None), "C": (None, acc[(2, "w")])})
            per_launch.append(sum(sh.launch(per)["stale"]))
        res[single] = per_launch
    one = (P - 1) * k * n * 4
    assert one == cf.gemm_stale(k, n, P) == 5760
    assert res[False] == [one, 0]
    assert res[True] == [one, one]


def test_nbody_soa_with_mass_single_owner_vs_validity():
    """Paper-vs-validity pin: N-body on structure-of-arrays fp32 positions
    x, y, z (ping-pong), a separate read-only mass array and in-place velocities;
    1,024 bodies, P = 8, 3 steps.  Hand derivation: every step each partition reads all
    of x, y, z and m and holds 1/8 of each, so each step moves 7 x 1,024 x 4 = 28,672 B per
    array.  Positions are rewritten every step (3 x 3 x 28,672 = 258,048 B in both modes);
    velocities are read and written on the own slab only (0 B).  Masses are never written:
    with shared copies they move once (28,672 B) -> 286,720 B; the paper's tracker moves
    them every step (3 x 28,672) -> 344,064 B."""
    n, P, steps = 1024, 8, 3
    g = (n // 128, 1, 1)
    totals = {}
    for single in (False, True):
        sh = shadow.Shadow(P, single)
        for name in ("x0", "y0", "z0", "m", "vx", "vy", "vz"):
            sh.register(name, n, 4, True)
        for name in ("x1", "y1", "z1"):
            sh.register(name, n, 4, False)
        tot = 0
        for s in range(steps):
            src = ("x0", "y0", "z0") if s % 2 == 0 else ("x1", "y1", "z1")
            dst = ("x1", "y1", "z1") if s % 2 == 0 else ("x0", "y0", "z0")
            names = src + ("m", "vx", "vy", "vz") + dst
            per = []
            for p in range(P):
                acc = regions.nbody_soa(grid.partition_box(g, P, p), (128,), n)
                per.append({nm: (acc.get((a, "r")), acc.get((a, "w"))) for a, nm in enumerate(names)})
            tot += sum(sh.launch(per)["stale"])
        totals[single] = tot
    assert totals[False] == 286720
    assert totals[True] == 344064


@pytest.mark.parametrize("k", [2, 3, 4])
@pytest.mark.parametrize("nparts", [2, 4])
def test_hotspot_tbk_stale_matches_closed_form(nparts, k):
    """K fused sweeps per launch (hotspot2d_tb2 = K 2, hotspot2d_tbk): temperature is
    dilated by K rows per cut, power by K - 1 rows (once in validity mode, every launch
    in single-owner mode) -- closed forms derived from the dependency cone, so an
    over- or under-declared brute-force region fails here."""
    h, w, ty = 64, 64, 8
    for single in (False, True):
        sh = shadow.Shadow(nparts, single)
        sh.register("t0", h * w, 4, True)
        sh.register("t1", h * w, 4, False)
        sh.register("pw", h * w, 4, True)
        stale = []
        for it in range(4):
            a, b = ("t0", "t1") if it % 2 == 0 else ("t1", "t0")
            per = []
            for p in range(nparts):
                if k == 2:
                    g = (w // 32 + (w % 32 > 0), (h + ty - 1) // ty, 1)
                    acc = regions.hotspot2d_tb2(grid.partition_box(g, nparts, p), (8,), h, w, ty)
                else:
                    g = (1, (h + ty - 1) // ty, 1)
                    acc = regions.hotspot2d_tbk(grid.partition_box(g, nparts, p), None, h, w, ty, k)
                per.append({a: (acc[(0, "r")], None), "pw": (acc[(1, "r")], None), b: (None, acc[(2, "w")])})
            stale.append(sum(sh.launch(per)["stale"]))
        t = cf.hotspot2d_tbk_stale_per_launch(w, nparts, k)
        pw = cf.hotspot2d_tbk_power_once(w, nparts, k)
        if single:
            assert stale == [t + pw] * 4
        else:
            assert stale == [t + pw, t, t, t]


@pytest.mark.parametrize("nparts", [2, 4])
def test_heat3d_tb2_stale_matches_closed_form(nparts):
    d, h, w, zc = 16, 6, 8, 2
    g = (1, 1, d // zc)
    sh = shadow.Shadow(nparts)
    sh.register("u0", d * h * w, 4, True)
    sh.register("u1", d * h * w, 4, False)
    stale = []
    for it in range(3):
        a, b = ("u0", "u1") if it % 2 == 0 else ("u1", "u0")
        per = []
        for p in range(nparts):
            acc = regions.heat3d_tb2(grid.partition_box(g, nparts, p), d, h, w, zc)
            per.append({a: (acc[(0, "r")], None), b: (None, acc[(1, "w")])})
        stale.append(sum(sh.launch(per)["stale"]))
    assert stale == [cf.heat3d_tb2_stale_per_launch(h, w, nparts)] * 3


@pytest.mark.parametrize("nparts", [2, 4])
def test_heat3d_tb3_stale_matches_closed_form(nparts):
    """Three sweeps: the thread program's 7x7x7 cones cross each z-cut by 3 planes (hand
    count: 3 planes x h x w x 4 B each way), not 2 (two sweeps) or 4."""
    d, h, w, zc = 24, 6, 8, 3
    g = (1, 1, d // zc)
    sh = shadow.Shadow(nparts)
    sh.register("u0", d * h * w, 4, True)
    sh.register("u1", d * h * w, 4, False)
    stale = []
    for it in range(3):
        a, b = ("u0", "u1") if it % 2 == 0 else ("u1", "u0")
        per = []
        for p in range(nparts):
            acc = regions.heat3d_tb2(grid.partition_box(g, nparts, p), d, h, w, zc, sweeps=3)
            per.append({a: (acc[(0, "r")], None), b: (None, acc[(1, "w")])})
        stale.append(sum(sh.launch(per)["stale"]))
    assert stale == [cf.heat3d_tb3_stale_per_launch(h, w, nparts)] * 3 == [(nparts - 1) * 6 * 6 * 8 * 4] * 3


@pytest.mark.parametrize("nparts", [2, 3, 4, 8])
def test_hotspot_steady_state_matches_closed_form(nparts):
    h = w = 64
    ty, bdx = 4, 8                                      # block = 32 columns x 4 rows
    g = ((w + 4 * bdx - 1) // (4 * bdx), (h + ty - 1) // ty, 1)
    sh = shadow.Shadow(nparts)
    sh.register("t0", h * w, 4, True)
    sh.register("t1", h * w, 4, False)
    sh.register("pw", h * w, 4, True)
    stale = []
    for it in range(5):
        a, b = ("t0", "t1") if it % 2 == 0 else ("t1", "t0")
        per = []
        for p in range(nparts):
            box = grid.partition_box(g, nparts, p)
            acc = regions.hotspot2d(box, (bdx,), h, w, ty)
            per.append({a: (acc[(0, "r")], None), "pw": (acc[(1, "r")], None), b: (None, acc[(2, "w")])})
        stale.append(sum(sh.launch(per)["stale"]))
    assert stale[1:] == [cf.hotspot2d_stale_per_iter(w, nparts)] * 4
    # fragmentation: bounded segment count per buffer
    for name in ("t0", "t1"):
        assert len(sh.buffers[name].rle()) <= 2 * nparts - 1


@pytest.mark.parametrize("tiles", [(2, 2, 1), (4, 2, 1), (2, 3, 1)])
def test_tile_partition_steady_state_matches_closed_form(tiles):
    """NEXT-2: with tx x ty tiles every internal cut moves one row / column each way."""
    h, w = 48, 96
    ty, bdx = 4, 4                                      # block = 16 columns x 4 rows
    g = ((w + 4 * bdx - 1) // (4 * bdx), (h + ty - 1) // ty, 1)
    nparts = tiles[0] * tiles[1]
    sh = shadow.Shadow(nparts)
    for name, up in (("t0", True), ("t1", False), ("pw", True)):
        sh.register(name, h * w, 4, up)
    stale = []
    for it in range(4):
        a, b = ("t0", "t1") if it % 2 == 0 else ("t1", "t0")
        per = []
        for p in range(nparts):
            acc = regions.hotspot2d(grid.tile_box(g, tiles, p), (bdx,), h, w, ty)
            per.append({a: (acc[(0, "r")], None), "pw": (acc[(1, "r")], None), b: (None, acc[(2, "w")])})
        stale.append(sum(sh.launch(per)["stale"]))
    assert stale[2:] == [cf.hotspot2d_tile_stale_per_iter(h, w, tiles[0], tiles[1])] * 2
    # Jacobi (Dirichlet): interior cells only cross the cuts
    n = 64
    sj = shadow.Shadow(nparts)
    sj.register("u0", n * n, 4, True)
    sj.register("u1", n * n, 4, True)
    gj = (n // 32 + (n % 32 > 0), n // 8, 1)
    per_it = []
    for it in range(4):
        a, b = ("u0", "u1") if it % 2 == 0 else ("u1", "u0")
        per = []
        for p in range(nparts):
            acc = regions.jacobi2d(grid.tile_box(gj, tiles, p), (32, 8), n, n)
            per.append({a: (acc[(0, "r")], None), b: (None, acc[(1, "w")])})
        per_it.append(sum(sj.launch(per)["stale"]))
    if gj[0] % tiles[0] == 0:
        assert per_it[2:] == [cf.jacobi2d_tile_stale_per_iter(n, n, tiles[0], tiles[1])] * 2


def test_nbody_allgather_and_validity_vs_single_owner():
    n, P = 1024, 8
    sh = shadow.Shadow(P)
    sh.register("p0", n, 16, True)
    sh.register("p1", n, 16, False)
    sh.register("v", n, 16, True)
    g = (n // 128, 1, 1)
    tot = 0
    for s in range(3):
        a, b = ("p0", "p1") if s % 2 == 0 else ("p1", "p0")
        per = []
        for p in range(P):
            acc = regions.nbody(grid.partition_box(g, P, p), (64,), n)
            per.append({a: (acc[(0, "r")], None), "v": (acc[(1, "r")], acc[(1, "w")]),
                        b: (None, acc[(2, "w")])})
        tot += sum(sh.launch(per)["stale"])
    assert tot == 3 * cf.nbody_stale_per_step(n, P)


def test_write_overlap_is_rejected():
    sh = shadow.Shadow(2)
    sh.register("x", 10, 4, False)
    with pytest.raises(shadow.WriteOverlap):
        sh.launch([{"x": (None, np.arange(0, 6))}, {"x": (None, np.arange(5, 10))}])


def test_rle_and_source_choice():
    b = shadow.ShadowBuffer(10, 4, 3)
    b.h2d_linear()
    assert b.rle() == [(0, 12, 1), (12, 24, 2), (24, 40, 4)]
    assert shadow.choose_source(0b101, 1, 3) == 0          # tie -> lower
    assert shadow.choose_source(0b110, 0, 3) == 1
    assert shadow.choose_source(0b1001, 2, 4) == 3
