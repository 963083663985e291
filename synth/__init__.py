"""Seeded synthetic inputs shared by the CUDA path's tests/bench and by the oracle.

This module holds NO arithmetic of the method (no stencil, no region, no tracker
logic): it only draws random numbers with numpy's ``default_rng(seed)`` in the
shapes and value ranges DESIGN.md §"Input recipe" states (SURVEY.md §8(d),
"Synthetic inputs" table).  Both sides import it; neither side imports the other.

All arrays are C-contiguous, row-major, float32 (the storage type of every
benchmark buffer, BASELINE.json ``configs``).
"""
from __future__ import annotations

import numpy as np

# Seeds of SURVEY.md §8(d): one per buffer so that every config is reproducible.
SEED_JACOBI = 0
SEED_HOTSPOT_TEMP = 1
SEED_HOTSPOT_POWER = 2
SEED_HEAT = 3
SEED_GEMM_A = 4
SEED_GEMM_B = 5
SEED_NBODY = 6


def uniform(shape, lo: float, hi: float, seed: int) -> np.ndarray:
    """U[lo, hi) float32 array of ``shape`` drawn from default_rng(seed)."""
    rng = np.random.default_rng(seed)
    return rng.uniform(lo, hi, size=shape).astype(np.float32)


def jacobi_grid(h: int, w: int, seed: int = SEED_JACOBI) -> np.ndarray:
    """C1: U[0,1) everywhere, boundary included (Dirichlet boundary = these values)."""
    return uniform((h, w), 0.0, 1.0, seed)


def hotspot_grids(h: int, w: int, seed_t: int = SEED_HOTSPOT_TEMP,
                  seed_p: int = SEED_HOTSPOT_POWER):
    """C2: temperature U[300,350), power U[0,0.01) (Rodinia-like ranges)."""
    return uniform((h, w), 300.0, 350.0, seed_t), uniform((h, w), 0.0, 0.01, seed_p)


def heat_grid(d: int, h: int, w: int, seed: int = SEED_HEAT) -> np.ndarray:
    """C3: U[0,1) on a d x h x w (z, y, x) grid."""
    return uniform((d, h, w), 0.0, 1.0, seed)


def gemm_operands(m: int, n: int, k: int, seed_a: int = SEED_GEMM_A,
                  seed_b: int = SEED_GEMM_B):
    """C4: A (m x k) and B (k x n), both U[-1,1)."""
    return uniform((m, k), -1.0, 1.0, seed_a), uniform((k, n), -1.0, 1.0, seed_b)


def nbody_bodies(n: int, seed: int = SEED_NBODY):
    """C5: pos float4 (x, y, z, m) with xyz U[-1,1)^3 and m = 1/n; vel = 0.

    Returns (pos[n,4], vel[n,4]) float32.
    """
    rng = np.random.default_rng(seed)
    pos = np.empty((n, 4), dtype=np.float32)
    pos[:, :3] = rng.uniform(-1.0, 1.0, size=(n, 3)).astype(np.float32)
    pos[:, 3] = np.float32(1.0 / n)
    vel = np.zeros((n, 4), dtype=np.float32)
    return pos, vel


def sample_indices(n_total: int, n_sample: int, seed: int = 1234) -> np.ndarray:
    """Sorted distinct flat indices for sampled comparisons at full size."""
    rng = np.random.default_rng(seed)
    n_sample = min(n_sample, n_total)
    return np.sort(rng.choice(n_total, size=n_sample, replace=False)).astype(np.int64)
