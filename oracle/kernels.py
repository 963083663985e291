"""ctypes front-end of oracle/kernels.c -- TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

All functions take/return numpy arrays; computation is fp64 in plain C.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

from . import build as _build

# Reading Q14: Rodinia hotspot constants frozen at their N=1024
# values (step/Cap = 1e-3 / (3e6 * (0.016/1024)^2) = 4096/3000, Rx_1 = Ry_1 = 0.1,
# Rz_1 = 1/20480, ambient 80).  PAPER.md P:L977-984 names the benchmark only.
HOTSPOT_CAP = 4096.0 / 3000.0
HOTSPOT_RX1 = 0.1
HOTSPOT_RY1 = 0.1
HOTSPOT_RZ1 = 1.0 / 20480.0
HOTSPOT_AMB = 80.0
# Reading Q15: clamped 7-point heat, alpha = 1/8.
HEAT_ALPHA = 0.125
# Reading Q16: G = 1, softening eps^2 = 1e-4, dt = 1e-3.
NBODY_EPS2 = 1e-4
NBODY_DT = 1e-3

_lib = None
_D = ctypes.POINTER(ctypes.c_double)
_F = ctypes.POINTER(ctypes.c_float)
_I = ctypes.POINTER(ctypes.c_int64)
_i64 = ctypes.c_int64


def lib():
    global _lib
    if _lib is None:
        path = _build.build()
        _lib = ctypes.CDLL(path)
        L = _lib
        L.oracle_jacobi2d.argtypes = [_D, _D, _i64, _i64, ctypes.c_int]
        L.oracle_jacobi2d_f32.argtypes = [_F, _F, _i64, _i64, ctypes.c_int]
        L.oracle_hotspot2d.argtypes = [_D, _D, _D, _i64, _i64, ctypes.c_int] + [ctypes.c_double] * 5
        L.oracle_heat3d.argtypes = [_D, _D, _i64, _i64, _i64, ctypes.c_int, ctypes.c_double]
        L.oracle_gemm.argtypes = [_D, _D, _D, _i64, _i64, _i64]
        L.oracle_gemm_entries_f32.argtypes = [_F, _F, _i64, _i64, _I, _I, _i64, _D]
        L.oracle_nbody_accel.argtypes = [_D, _i64, _I, _i64, ctypes.c_double, _D]
        L.oracle_nbody_step.argtypes = [_D, _D, _D, _D, _i64, ctypes.c_double, ctypes.c_double]
        L.oracle_num_threads.restype = ctypes.c_int
    return _lib


def _dp(a):
    return a.ctypes.data_as(_D)


def num_threads() -> int:
    return int(lib().oracle_num_threads())


def jacobi2d(u: np.ndarray, iters: int) -> np.ndarray:
    """C1 result after ``iters`` Dirichlet sweeps (both buffers start equal to u)."""
    u0 = np.ascontiguousarray(u, dtype=np.float64).copy()
    u1 = u0.copy()
    h, w = u0.shape
    lib().oracle_jacobi2d(_dp(u0), _dp(u1), h, w, iters)
    return u0 if iters % 2 == 0 else u1


def jacobi2d_f32(u: np.ndarray, iters: int) -> np.ndarray:
    """C1 in fp32 storage and arithmetic, each operation rounded as written (no FMA): the
    bit-exact mirror of a kernel that evaluates the same expression in the same order."""
    u0 = np.ascontiguousarray(u, dtype=np.float32).copy()
    u1 = u0.copy()
    h, w = u0.shape
    lib().oracle_jacobi2d_f32(u0.ctypes.data_as(_F), u1.ctypes.data_as(_F), h, w, iters)
    return u0 if iters % 2 == 0 else u1


def hotspot2d(temp: np.ndarray, power: np.ndarray, iters: int) -> np.ndarray:
    t0 = np.ascontiguousarray(temp, dtype=np.float64).copy()
    t1 = np.zeros_like(t0)
    p = np.ascontiguousarray(power, dtype=np.float64)
    h, w = t0.shape
    lib().oracle_hotspot2d(_dp(t0), _dp(t1), _dp(p), h, w, iters, HOTSPOT_CAP,
                           HOTSPOT_RX1, HOTSPOT_RY1, HOTSPOT_RZ1, HOTSPOT_AMB)
    return t0 if iters % 2 == 0 else t1


def heat3d(u: np.ndarray, iters: int, alpha: float = HEAT_ALPHA) -> np.ndarray:
    u0 = np.ascontiguousarray(u, dtype=np.float64).copy()
    u1 = np.zeros_like(u0)
    d, h, w = u0.shape
    lib().oracle_heat3d(_dp(u0), _dp(u1), d, h, w, iters, alpha)
    return u0 if iters % 2 == 0 else u1


def gemm(a: np.ndarray, b: np.ndarray) -> np.ndarray:
    a64 = np.ascontiguousarray(a, dtype=np.float64)
    b64 = np.ascontiguousarray(b, dtype=np.float64)
    m, k = a64.shape
    k2, n = b64.shape
    assert k == k2
    c = np.empty((m, n), dtype=np.float64)
    lib().oracle_gemm(_dp(a64), _dp(b64), _dp(c), m, n, k)
    return c


def gemm_entries(a: np.ndarray, b: np.ndarray, rows: np.ndarray, cols: np.ndarray) -> np.ndarray:
    a32 = np.ascontiguousarray(a, dtype=np.float32)
    b32 = np.ascontiguousarray(b, dtype=np.float32)
    rows = np.ascontiguousarray(rows, dtype=np.int64)
    cols = np.ascontiguousarray(cols, dtype=np.int64)
    k, n = b32.shape
    out = np.empty(rows.shape[0], dtype=np.float64)
    lib().oracle_gemm_entries_f32(a32.ctypes.data_as(_F), b32.ctypes.data_as(_F), n, k,
                                  rows.ctypes.data_as(_I), cols.ctypes.data_as(_I),
                                  rows.shape[0], _dp(out))
    return out


def nbody_accel(pos: np.ndarray, targets: np.ndarray, eps2: float = NBODY_EPS2) -> np.ndarray:
    p = np.ascontiguousarray(pos, dtype=np.float64)
    t = np.ascontiguousarray(targets, dtype=np.int64)
    out = np.empty((t.shape[0], 3), dtype=np.float64)
    lib().oracle_nbody_accel(_dp(p), p.shape[0], t.ctypes.data_as(_I), t.shape[0], eps2, _dp(out))
    return out


def nbody(pos: np.ndarray, vel: np.ndarray, steps: int, dt: float = NBODY_DT,
          eps2: float = NBODY_EPS2):
    p0 = np.ascontiguousarray(pos, dtype=np.float64).copy()
    v0 = np.ascontiguousarray(vel, dtype=np.float64).copy()
    p1 = np.empty_like(p0)
    v1 = np.empty_like(v0)
    n = p0.shape[0]
    for _ in range(steps):
        lib().oracle_nbody_step(_dp(p0), _dp(v0), _dp(p1), _dp(v1), n, dt, eps2)
        p0, p1 = p1, p0
        v0, v1 = v1, v0
    return p0, v0
