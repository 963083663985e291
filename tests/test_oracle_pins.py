"""Pins of the CPU oracle against what the paper and mathematics fix (no GPU).

Each test checks an oracle function against something other than itself: the
paper's printed worked example (tests/golden/eq1_4.json), closed forms,
invariants, brute force on tiny inputs, or a special case that reduces to a
library routine.  Chosen so that a dropped term, wrong sign/index or transposed
operand in oracle/ fails at least one of them.
"""
import json
import math
import os

import numpy as np
import pytest

from oracle import closed_forms as cf
from oracle import kernels as ok
from oracle import polyhedral as poly

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _golden_set(expr, lo=-2, hi=12):
    pts = set()
    for y in range(lo, hi):
        for x in range(lo, hi):
            if eval(expr, {}, {"x": x, "y": y}):
                pts.add((y, x))
    return pts


# --------------------------- Eq. 1-4 ---------------------------
def test_eq1_4_image_matches_printed_eq3():
    g = json.load(open(os.path.join(GOLDEN, "eq1_4.json")))
    s1 = _golden_set(g["S1"])
    assert s1 == poly.S1()
    # image of S1 under the printed map M (Eq. 2) equals the printed S2 (Eq. 3)
    img = set()
    for (y, x) in s1:
        for y2 in range(-2, 14):
            for x2 in range(-2, 14):
                if eval(g["M"], {}, {"x": x, "y": y, "x2": x2, "y2": y2}):
                    img.add((y2, x2))
    s2 = _golden_set(g["S2"])
    assert img == s2 == poly.M(poly.S1()) == poly.S2_printed()
    assert len(s1) == 15 and len(s2) == 15 and len(s1 & s2) == 3
    assert len(poly.U()) == 27


def test_rowwise_first_last_union_overapproximates_and_per_piece_is_exact():
    # row-wise min/max over the union over-approximates ...
    u = poly.U()
    over = poly.points_of_rows(poly.rowwise_first_last(u))
    assert u < over
    assert over - u == {(4, 5)}          # row y = 4: pieces [4,4] and [6,7]
    # ... and applying it per convex piece is exact.
    exact = poly.points_of_rows(poly.rowwise_per_piece([poly.S1(), poly.M(poly.S1())]))
    assert exact == u
    # convex piece alone: row-wise first/last is exact
    assert poly.points_of_rows(poly.rowwise_first_last(poly.S1())) == poly.S1()


# --------------------------- C1 Jacobi (reading Q15) ---------------------------
def test_jacobi_harmonic_fixed_point_exact():
    n = 64
    i = np.arange(n)[:, None].astype(np.float64)
    j = np.arange(n)[None, :].astype(np.float64)
    u = i * j                              # discrete-harmonic: sum of 4 neighbours = 4ij
    out = ok.jacobi2d(u, 10)
    assert np.array_equal(out, u)


def test_jacobi_sine_mode_decays_by_eigenvalue():
    n, iters = 48, 7
    u, lam = cf.jacobi_sine_mode(n, 3, 5)
    out = ok.jacobi2d(u, iters)
    np.testing.assert_allclose(out, lam ** iters * u, atol=1e-13)


def test_jacobi_boundary_untouched_and_asymmetric_input():
    rng = np.random.default_rng(7)
    u = rng.uniform(size=(9, 13))
    out = ok.jacobi2d(u, 1)
    # brute force on a tiny input, one cell at a time from the definition
    exp = u.copy()
    for a in range(1, 8):
        for b in range(1, 12):
            exp[a, b] = 0.25 * (u[a - 1, b] + u[a + 1, b] + u[a, b - 1] + u[a, b + 1])
    np.testing.assert_allclose(out, exp, rtol=1e-15, atol=0)
    assert np.array_equal(out[0], u[0]) and np.array_equal(out[:, -1], u[:, -1])


def test_jacobi_f32_mirror_brute_force_and_fp64():
    """The fp32 mirror (SURVEY §8(c) optional strong pin): equal bit for bit to a per-cell
    numpy float32 evaluation of the same expression in the same order (each operation rounded
    to fp32, no FMA) on a tiny ragged input over three ping-pong sweeps; within 1e-6 of the fp64
    definition after 10 sweeps on 64^2; the harmonic field i*j stays an exact fixed point."""
    rng = np.random.default_rng(8)
    u = rng.uniform(size=(9, 13)).astype(np.float32)
    a, b = u.copy(), u.copy()
    q = np.float32(0.25)
    for _ in range(3):
        for r in range(1, 8):
            for c in range(1, 12):
                b[r, c] = q * (((a[r - 1, c] + a[r + 1, c]) + a[r, c - 1]) + a[r, c + 1])
        a, b = b, a
    assert np.array_equal(ok.jacobi2d_f32(u, 3), a)
    v = np.random.default_rng(9).uniform(size=(64, 64)).astype(np.float32)
    np.testing.assert_allclose(ok.jacobi2d_f32(v, 10), ok.jacobi2d(v, 10), rtol=1e-6, atol=0)
    i = np.arange(64)[:, None].astype(np.float32)
    j = np.arange(64)[None, :].astype(np.float32)
    assert np.array_equal(ok.jacobi2d_f32(i * j, 10), i * j)


# --------------------------- C2 Hotspot (reading Q14) ---------------------------
def test_hotspot_uniform_recurrence():
    h, w, it = 17, 24, 9
    t = np.full((h, w), 323.0)
    p = np.full((h, w), 0.004)
    out = ok.hotspot2d(t, p, it)
    exp = cf.hotspot_uniform(323.0, 0.004, it, ok.HOTSPOT_CAP, ok.HOTSPOT_RZ1, ok.HOTSPOT_AMB)
    np.testing.assert_allclose(out, exp, rtol=1e-13)


@pytest.mark.parametrize("ky,kx", [(1, 0), (2, 3), (5, 1)])
def test_hotspot_cosine_mode(ky, kx):
    h, w, it = 20, 28, 6
    f, lam_terms = cf.cosine_mode((h, w), (ky, kx))
    t = ok.HOTSPOT_AMB + f            # zero power: T - amb evolves linearly
    p = np.zeros((h, w))
    out = ok.hotspot2d(t, p, it)
    g = 1.0 + ok.HOTSPOT_CAP * (ok.HOTSPOT_RY1 * lam_terms[0] + ok.HOTSPOT_RX1 * lam_terms[1]
                                - ok.HOTSPOT_RZ1)
    np.testing.assert_allclose(out - ok.HOTSPOT_AMB, g ** it * f, atol=1e-11)


def test_hotspot_rx_ry_not_swapped():
    # Rx1 == Ry1 in the frozen constants, so also check the x/y roles on a
    # non-square grid with a row-only and a column-only mode: both must decay
    # by their own 1-D factor (a transposed index would mix them).
    h, w = 10, 30
    f_rows, lt = cf.cosine_mode((h, w), (2, 0))
    f_cols, lt2 = cf.cosine_mode((h, w), (0, 2))
    for f, lam in ((f_rows, lt[0]), (f_cols, lt2[1])):
        out = ok.hotspot2d(ok.HOTSPOT_AMB + f, np.zeros((h, w)), 1)
        g = 1.0 + ok.HOTSPOT_CAP * (0.1 * lam - ok.HOTSPOT_RZ1)
        np.testing.assert_allclose(out - ok.HOTSPOT_AMB, g * f, atol=1e-12)


# --------------------------- C3 Heat (reading Q15) ---------------------------
@pytest.mark.parametrize("ks", [(1, 0, 0), (0, 2, 1), (3, 1, 2)])
def test_heat_cosine_eigenmode(ks):
    shape, it = (9, 12, 14), 4
    u, lam_terms = cf.cosine_mode(shape, ks)
    out = ok.heat3d(u, it)
    lam = 1.0 + ok.HEAT_ALPHA * sum(lam_terms)
    np.testing.assert_allclose(out, lam ** it * u, atol=1e-13)


def test_heat_conserves_sum_and_uniform_stays_uniform():
    rng = np.random.default_rng(3)
    u = rng.uniform(size=(7, 11, 13))
    out = ok.heat3d(u, 5)
    assert abs(out.sum() - u.sum()) < 1e-11 * u.size
    c = np.full((5, 6, 7), 0.375)
    assert np.array_equal(ok.heat3d(c, 3), c)


def test_heat_brute_force_tiny():
    rng = np.random.default_rng(11)
    u = rng.uniform(size=(3, 4, 5))
    out = ok.heat3d(u, 1)
    d, h, w = u.shape
    for k in range(d):
        for i in range(h):
            for j in range(w):
                nb = 0.0
                for dk, di, dj in ((-1, 0, 0), (1, 0, 0), (0, -1, 0), (0, 1, 0), (0, 0, -1), (0, 0, 1)):
                    nb += u[min(max(k + dk, 0), d - 1), min(max(i + di, 0), h - 1), min(max(j + dj, 0), w - 1)]
                assert abs(out[k, i, j] - (u[k, i, j] + 0.125 * (nb - 6 * u[k, i, j]))) < 1e-15


# --------------------------- C4 GEMM (reading Q17) ---------------------------
def test_gemm_identity_and_library_special_case():
    rng = np.random.default_rng(5)
    b = rng.uniform(-1, 1, size=(24, 40))
    assert np.array_equal(ok.gemm(np.eye(24), b), b)
    a = rng.uniform(-1, 1, size=(17, 24))
    np.testing.assert_allclose(ok.gemm(a, b), a @ b, rtol=1e-13, atol=1e-13)


def test_gemm_rank1_small_integers_exact():
    m, n, k = 13, 21, 37
    u = np.arange(1, m + 1, dtype=np.float64)
    v = np.arange(1, n + 1, dtype=np.float64) * 2
    a = np.repeat(u[:, None], k, axis=1)
    b = np.repeat(v[None, :], k, axis=0)
    assert np.array_equal(ok.gemm(a, b), k * np.outer(u, v))


def test_gemm_entries_match_full():
    rng = np.random.default_rng(9)
    a = rng.uniform(-1, 1, size=(33, 19)).astype(np.float32)
    b = rng.uniform(-1, 1, size=(19, 45)).astype(np.float32)
    full = ok.gemm(a, b)
    rows = np.array([0, 5, 32, 17], dtype=np.int64)
    cols = np.array([44, 0, 3, 20], dtype=np.int64)
    np.testing.assert_array_equal(ok.gemm_entries(a, b, rows, cols), full[rows, cols])


# --------------------------- C5 N-body (reading Q16) ---------------------------
def test_nbody_two_body_closed_form():
    pos = np.array([[0.1, -0.2, 0.3, 0.5], [0.4, 0.2, -0.1, 0.25]])
    acc = ok.nbody_accel(pos, np.array([0, 1]))
    np.testing.assert_allclose(acc[0], cf.nbody_two_body_accel(pos[0, :3], pos[1, :3], 0.25, ok.NBODY_EPS2), rtol=1e-14)
    np.testing.assert_allclose(acc[1], cf.nbody_two_body_accel(pos[1, :3], pos[0, :3], 0.5, ok.NBODY_EPS2), rtol=1e-14)


def test_nbody_cube_symmetry_and_momentum():
    verts = np.array([[sx, sy, sz] for sx in (-1, 1) for sy in (-1, 1) for sz in (-1, 1)], dtype=np.float64)
    pos = np.concatenate([verts, np.full((8, 1), 0.125)], axis=1)
    acc = ok.nbody_accel(pos, np.arange(8))
    mags = np.linalg.norm(acc, axis=1)
    np.testing.assert_allclose(mags, mags[0], rtol=1e-13)
    # pointing to the centre: a_i parallel to -x_i
    cos = np.sum(acc * -verts, axis=1) / (mags * np.linalg.norm(verts, axis=1))
    np.testing.assert_allclose(cos, 1.0, rtol=1e-13)
    rng = np.random.default_rng(2)
    p = np.concatenate([rng.uniform(-1, 1, size=(50, 3)), rng.uniform(0.1, 1, size=(50, 1))], axis=1)
    a = ok.nbody_accel(p, np.arange(50))
    mom = (p[:, 3:4] * a).sum(axis=0)
    assert np.max(np.abs(mom)) < 1e-12 * np.max(np.abs(p[:, 3:4] * a))


def test_nbody_step_is_kick_then_drift():
    rng = np.random.default_rng(4)
    pos = np.concatenate([rng.uniform(-1, 1, size=(6, 3)), np.full((6, 1), 1 / 6)], axis=1)
    vel = np.concatenate([rng.uniform(-1, 1, size=(6, 3)), np.zeros((6, 1))], axis=1)
    p1, v1 = ok.nbody(pos, vel, 1)
    a = ok.nbody_accel(pos, np.arange(6))
    np.testing.assert_allclose(v1[:, :3], vel[:, :3] + a * ok.NBODY_DT, rtol=1e-15)
    np.testing.assert_allclose(p1[:, :3], pos[:, :3] + v1[:, :3] * ok.NBODY_DT, rtol=1e-15)
    assert np.array_equal(p1[:, 3], pos[:, 3])
