"""Analytic minima of stale bytes and numeric closed forms -- TEST INFRASTRUCTURE ONLY.

Stale-byte minima (SURVEY.md §8(d) "Stale bytes: analytic minimum"; [derived]):
each internal partition boundary of a row/plane-slab decomposition exchanges one
halo row/plane per direction per iteration; whole-buffer reads (GEMM B, N-body
positions) move the (P-1)/P of the buffer each partition lacks.

The numeric closed forms are mathematical facts about the kernel definitions
(DESIGN.md §3 readings Q14-Q17), used to pin the oracle (tests/test_oracle_pins.py).
"""
from __future__ import annotations

import math

import numpy as np


# ------------------------- stale bytes (per launch) -------------------------
def jacobi2d_stale_per_iter(w: int, nparts: int, elem_bytes: int = 4) -> int:
    """Dirichlet: each boundary moves one interior row (w - 2 cells) each way."""
    return (nparts - 1) * 2 * (w - 2) * elem_bytes


def hotspot2d_stale_per_iter(w: int, nparts: int, elem_bytes: int = 4) -> int:
    """Clamped: each boundary moves one full row each way: 131,072 (P-1) B at w = 16384."""
    return (nparts - 1) * 2 * w * elem_bytes


def heat3d_stale_per_iter(h: int, w: int, nparts: int, elem_bytes: int = 4) -> int:
    """One full h x w plane each way per boundary: 8,388,608 (P-1) B at 1024^2."""
    return (nparts - 1) * 2 * h * w * elem_bytes


def hotspot2d_tile_stale_per_iter(h: int, w: int, tx: int, ty: int, elem_bytes: int = 4) -> int:
    """Tile partitions (NEXT-2), clamped 5-point: every internal horizontal cut moves
    one full row (w cells) each way, every internal vertical cut one full column
    (h cells) each way; the 5-point stencil reads no diagonal, so corners move nothing."""
    return 2 * ((ty - 1) * w + (tx - 1) * h) * elem_bytes


def jacobi2d_tile_stale_per_iter(h: int, w: int, tx: int, ty: int, elem_bytes: int = 4) -> int:
    """Tile partitions, Dirichlet 5-point: only interior cells are read through a cut,
    so a horizontal cut moves w - 2 cells and a vertical cut h - 2 cells each way."""
    return 2 * ((ty - 1) * (w - 2) + (tx - 1) * (h - 2)) * elem_bytes


def gemm_stale(k: int, n: int, nparts: int, elem_bytes: int = 4) -> int:
    """B (k x n) linearly distributed, read whole by every partition: (P-1) * |B|."""
    return (nparts - 1) * k * n * elem_bytes


def nbody_stale_per_step(n: int, nparts: int, elem_bytes: int = 16) -> int:
    """Positions read whole by every partition: (P-1) * |pos| per step."""
    return (nparts - 1) * n * elem_bytes


# ------------------------- numeric closed forms -------------------------
def jacobi_sine_mode(n: int, k: int, l: int):
    """u = sin(pi k i/(n-1)) sin(pi l j/(n-1)) vanishes on the boundary and is an
    eigenvector of the Dirichlet Jacobi sweep with eigenvalue
    (cos(pi k/(n-1)) + cos(pi l/(n-1))) / 2."""
    i = np.arange(n)[:, None]
    j = np.arange(n)[None, :]
    u = np.sin(math.pi * k * i / (n - 1)) * np.sin(math.pi * l * j / (n - 1))
    lam = 0.5 * (math.cos(math.pi * k / (n - 1)) + math.cos(math.pi * l / (n - 1)))
    return u, lam


def cosine_mode(shape, ks):
    """prod_d cos(pi k_d (i_d + 1/2) / N_d): eigenvector of the replicate-clamped
    second difference along each axis, with eigenvalue 2 cos(pi k_d / N_d) - 2."""
    u = np.ones(shape)
    lam_terms = []
    for axis, (nd, kd) in enumerate(zip(shape, ks)):
        idx = np.arange(nd).reshape([-1 if a == axis else 1 for a in range(len(shape))])
        u = u * np.cos(math.pi * kd * (idx + 0.5) / nd)
        lam_terms.append(2.0 * math.cos(math.pi * kd / nd) - 2.0)
    return u, lam_terms


def hotspot_uniform(t0: float, p0: float, iters: int, cap, rz1, amb) -> float:
    """Uniform T, uniform P: every neighbour difference vanishes, so
    T_{t+1} = T_t + cap (P0 + rz1 (amb - T_t)); closed form around T* = amb + P0/rz1."""
    tstar = amb + p0 / rz1
    return tstar + (t0 - tstar) * (1.0 - cap * rz1) ** iters


def nbody_two_body_accel(p1, p2, m2, eps2):
    d = np.asarray(p2, dtype=np.float64) - np.asarray(p1, dtype=np.float64)
    r2 = float(d @ d) + eps2
    return m2 * d / r2 ** 1.5


def hotspot2d_tbk_stale_per_launch(w: int, nparts: int, k: int, elem_bytes: int = 4) -> int:
    """K fused clamped 5-point sweeps per launch (NEXT-3; K = 2 is hotspot2d_tb2): the
    output at distance K from a cut depends on input rows up to K rows across it, so
    every cut moves K full rows of temperature each way per launch."""
    return (nparts - 1) * 2 * k * w * elem_bytes


def hotspot2d_tbk_power_once(w: int, nparts: int, k: int, elem_bytes: int = 4) -> int:
    """Power enters sweeps 1..K; the last sweep's power term is local, so the cone of
    one launch reaches K - 1 power rows across each cut.  Power is never rewritten:
    in validity mode these rows move once (first launch), in single-owner mode every launch."""
    return (nparts - 1) * 2 * (k - 1) * w * elem_bytes


def heat3d_tb2_stale_per_launch(h: int, w: int, nparts: int, elem_bytes: int = 4) -> int:
    """Two fused 7-point sweeps per launch: two h x w planes each way per z-cut."""
    return (nparts - 1) * 2 * 2 * h * w * elem_bytes


def heat3d_tb3_stale_per_launch(h: int, w: int, nparts: int, elem_bytes: int = 4) -> int:
    """Three fused 7-point sweeps per launch: three h x w planes each way per z-cut."""
    return (nparts - 1) * 2 * 3 * h * w * elem_bytes
