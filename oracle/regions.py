"""Brute-force read/write sets per partition -- TEST INFRASTRUCTURE ONLY.

SURVEY.md §8(c) row c2 / PAPER.md P:L458-466 (§4.1: block-granular access maps,
threadId projected out under 0 <= threadId < blockDim), P:L561-571 (Fig. 3 text:
read set = partition + halo, write set 1:1) and P:L709-718 (§6: the image of an
access map constrained to one partition box).

Here nothing is analysed: every thread of every block inside the partition box
is enumerated, each access the thread performs (its "thread program", written
from the kernel's definition in DESIGN.md §4) is evaluated with its guard, and
the touched element indices are collected into a set.  The library's region
analyzer must produce exactly these sets as canonical byte ranges.

Thread programs take the launch geometry (block dims, tile sizes) as inputs;
those numbers are the kernels' published launch contract, not
shared code.
"""
from __future__ import annotations

import numpy as np

READ, WRITE = "r", "w"


def _block_ranges(box):
    z0, z1, y0, y1, x0, x1 = box
    return np.arange(z0, z1), np.arange(y0, y1), np.arange(x0, x1)


def _clamp(v, n):
    return np.clip(v, 0, n - 1)


def _ravel(*idx_and_shape):
    *idx, shape = idx_and_shape
    return np.ravel_multi_index(tuple(np.asarray(i, dtype=np.int64) for i in idx), shape)


def _uniq(parts):
    if not parts:
        return np.zeros(0, dtype=np.int64)
    return np.unique(np.concatenate([np.asarray(p, dtype=np.int64).ravel() for p in parts]))


# ---------------------------------------------------------------------------
# C1 jacobi2d(in, out; H, W): block (bdx, bdy); thread -> cell
#   i = by*bdy + ty, j = bx*bdx + tx; if 1 <= i <= H-2 and 1 <= j <= W-2:
#   reads in[i-1][j], in[i+1][j], in[i][j-1], in[i][j+1]; writes out[i][j].
# ---------------------------------------------------------------------------
def jacobi2d(box, block, h, w):
    bdx, bdy = block[0], block[1]
    _, bys, bxs = _block_ranges(box)
    i = (bys[:, None] * bdy + np.arange(bdy)[None, :]).ravel()
    j = (bxs[:, None] * bdx + np.arange(bdx)[None, :]).ravel()
    i = i[(i >= 1) & (i <= h - 2)]
    j = j[(j >= 1) & (j <= w - 2)]
    I, J = np.meshgrid(i, j, indexing="ij")
    reads = [_ravel(I - 1, J, (h, w)), _ravel(I + 1, J, (h, w)),
             _ravel(I, J - 1, (h, w)), _ravel(I, J + 1, (h, w))]
    return {(0, READ): _uniq(reads), (1, WRITE): _uniq([_ravel(I, J, (h, w))])}


def jacobi2d_tb(box, h, w, k, t=32):
    """K fused C1 sweeps per launch (jacobi2d_tb): logical block (bx, by) owns the t x t
    cells rows [t*by, +t) x cols [t*bx, +t); it loads every grid cell within K of its
    tile (the square window, corners included) and writes its interior cells."""
    _, bys, bxs = _block_ranges(box)
    reads, writes = [], []
    for by in bys:
        for bx in bxs:
            r = np.arange(by * t - k, by * t + t + k)
            c = np.arange(bx * t - k, bx * t + t + k)
            r, c = r[(r >= 0) & (r < h)], c[(c >= 0) & (c < w)]
            R, C = np.meshgrid(r, c, indexing="ij")
            reads.append(_ravel(R, C, (h, w)))
            ro = np.arange(by * t, by * t + t)
            co = np.arange(bx * t, bx * t + t)
            ro, co = ro[(ro >= 1) & (ro <= h - 2)], co[(co >= 1) & (co <= w - 2)]
            R, C = np.meshgrid(ro, co, indexing="ij")
            writes.append(_ravel(R, C, (h, w)))
    return {(0, READ): _uniq(reads), (1, WRITE): _uniq(writes)}


# ---------------------------------------------------------------------------
# C2 hotspot2d(temp_in, power, temp_out; H, W, TY): block (bdx) threads, each
#   thread owns VEC=4 consecutive columns j = bx*4*bdx + 4*tx + v and marches the
#   TY rows i = by*TY + r.  Guard i < H, j < W.  Reads temp_in at (i, j) and its
#   4 neighbours clamped to the grid, power at (i, j); writes temp_out (i, j).
# ---------------------------------------------------------------------------
def hotspot2d(box, block, h, w, ty, vec=4):
    bdx = block[0]
    _, bys, bxs = _block_ranges(box)
    i = (bys[:, None] * ty + np.arange(ty)[None, :]).ravel()
    j = (bxs[:, None] * (vec * bdx) + np.arange(vec * bdx)[None, :]).ravel()
    i = i[i < h]
    j = j[j < w]
    I, J = np.meshgrid(i, j, indexing="ij")
    c = _ravel(I, J, (h, w))
    reads_t = [c, _ravel(_clamp(I - 1, h), J, (h, w)), _ravel(_clamp(I + 1, h), J, (h, w)),
               _ravel(I, _clamp(J - 1, w), (h, w)), _ravel(I, _clamp(J + 1, w), (h, w))]
    return {(0, READ): _uniq(reads_t), (1, READ): _uniq([c]), (2, WRITE): _uniq([c])}


def hotspot2d_tb2(box, block, h, w, ty, vec=4):
    """Two fused sweeps per launch (hotspot2d_tb2): every owned cell (same tile
    contract as hotspot2d) reads the clamped 5x5 square of temp_in and the clamped
    3x3 square of power around it and writes temp_out at the cell."""
    bdx = block[0]
    _, bys, bxs = _block_ranges(box)
    i = (bys[:, None] * ty + np.arange(ty)[None, :]).ravel()
    j = (bxs[:, None] * (vec * bdx) + np.arange(vec * bdx)[None, :]).ravel()
    i = i[i < h]
    j = j[j < w]
    I, J = np.meshgrid(i, j, indexing="ij")
    rt = [_ravel(_clamp(I + di, h), _clamp(J + dj, w), (h, w)) for di in range(-2, 3) for dj in range(-2, 3)]
    rp = [_ravel(_clamp(I + di, h), _clamp(J + dj, w), (h, w)) for di in range(-1, 2) for dj in range(-1, 2)]
    return {(0, READ): _uniq(rt), (1, READ): _uniq(rp), (2, WRITE): _uniq([_ravel(I, J, (h, w))])}


def hotspot2d_tbk(box, block, h, w, ty, k, cols=480):
    """K fused sweeps per launch (hotspot2d_tbk): logical block (bx, by) owns rows
    [by*ty, +ty) x columns [cols*bx, +cols); every owned cell reads the clamped
    (2K+1)^2 square of temp_in and the clamped (2K-1)^2 square of power around it
    (sweep s at distance <= K-s from the output needs power), writes temp_out."""
    _, bys, bxs = _block_ranges(box)
    i = (bys[:, None] * ty + np.arange(ty)[None, :]).ravel()
    j = (bxs[:, None] * cols + np.arange(cols)[None, :]).ravel()
    i = i[i < h]
    j = j[j < w]
    I, J = np.meshgrid(i, j, indexing="ij")
    rt = [_ravel(_clamp(I + di, h), _clamp(J + dj, w), (h, w)) for di in range(-k, k + 1) for dj in range(-k, k + 1)]
    rp = [_ravel(_clamp(I + di, h), _clamp(J + dj, w), (h, w))
          for di in range(-k + 1, k) for dj in range(-k + 1, k)]
    return {(0, READ): _uniq(rt), (1, READ): _uniq(rp), (2, WRITE): _uniq([_ravel(I, J, (h, w))])}


# ---------------------------------------------------------------------------
# C3 heat3d(u_in, u_out; D, H, W, ZC): block (bdx, bdy); thread owns VEC=4
#   columns j = bx*4*bdx + 4*tx + v, row i = by*bdy + ty, and marches ZC planes
#   k = bz*ZC + q.  Guard k < D, i < H, j < W.  Reads the 7-point clamped
#   neighbourhood of u_in, writes u_out (k, i, j).
# ---------------------------------------------------------------------------
def heat3d(box, block, d, h, w, zc, vec=4):
    bdx, bdy = block[0], block[1]
    bzs, bys, bxs = _block_ranges(box)
    k = (bzs[:, None] * zc + np.arange(zc)[None, :]).ravel()
    i = (bys[:, None] * bdy + np.arange(bdy)[None, :]).ravel()
    j = (bxs[:, None] * (vec * bdx) + np.arange(vec * bdx)[None, :]).ravel()
    k, i, j = k[k < d], i[i < h], j[j < w]
    K, I, J = np.meshgrid(k, i, j, indexing="ij")
    s = (d, h, w)
    c = _ravel(K, I, J, s)
    reads = [c,
             _ravel(_clamp(K - 1, d), I, J, s), _ravel(_clamp(K + 1, d), I, J, s),
             _ravel(K, _clamp(I - 1, h), J, s), _ravel(K, _clamp(I + 1, h), J, s),
             _ravel(K, I, _clamp(J - 1, w), s), _ravel(K, I, _clamp(J + 1, w), s)]
    return {(0, READ): _uniq(reads), (1, WRITE): _uniq([c])}


# ---------------------------------------------------------------------------
# C5 nbody(pos_in, vel, pos_out; N): block (bdx); thread tx of block bx owns
#   the `per_thread` bodies i = bx*per_thread*bdx + tx + u*bdx, guard i < N.
#   Reads every body of pos_in (all-pairs), reads and writes vel[i] (in place),
#   writes pos_out[i].  Elements are float4 bodies.
# ---------------------------------------------------------------------------
def nbody(box, block, n, per_thread=2):
    bdx = block[0]
    _, _, bxs = _block_ranges(box)
    i = (bxs[:, None] * (per_thread * bdx) + np.arange(per_thread * bdx)[None, :]).ravel()
    i = i[i < n]
    allpos = np.arange(n, dtype=np.int64) if i.size else np.zeros(0, dtype=np.int64)
    return {(0, READ): allpos, (1, READ): _uniq([i]), (1, WRITE): _uniq([i]),
            (2, WRITE): _uniq([i])}


def heat3d_tb2(box, d, h, w, zc, cols=120, rows=24, sweeps=2):
    """`sweeps` fused sweeps per launch (heat3d_tb2: 2, heat3d_tb3: 3): logical block
    (bx, by, bz) owns columns [cols*bx, +cols) x rows [rows*by, +rows) x planes
    [zc*bz, +zc); every owned cell reads the clamped (2s+1)^3 cube of u_in around it
    (s = sweeps: each sweep widens the dependence by one cell per direction) and writes
    u_out at the cell."""
    bzs, bys, bxs = _block_ranges(box)
    k = (bzs[:, None] * zc + np.arange(zc)[None, :]).ravel()
    i = (bys[:, None] * rows + np.arange(rows)[None, :]).ravel()
    j = (bxs[:, None] * cols + np.arange(cols)[None, :]).ravel()
    k, i, j = k[k < d], i[i < h], j[j < w]
    Kk, I, J = np.meshgrid(k, i, j, indexing="ij")
    s = (d, h, w)
    rd = [_ravel(_clamp(Kk + dz, d), _clamp(I + dy, h), _clamp(J + dx, w), s)
          for dz in range(-sweeps, sweeps + 1) for dy in range(-sweeps, sweeps + 1)
          for dx in range(-sweeps, sweeps + 1)]
    return {(0, READ): _uniq(rd), (1, WRITE): _uniq([_ravel(Kk, I, J, s)])}


# ---------------------------------------------------------------------------
# C4 gemm(A, B, C; M, N, K, BM, BN): block (bx, by) computes the C tile rows
#   by*BM + r, cols bx*BN + c (guard < M, < N) with the full K loop: reads
#   A[i][0..K), B[0..K)[j], writes C[i][j].
# ---------------------------------------------------------------------------
def gemm(box, m, n, k, bm, bn):
    _, bys, bxs = _block_ranges(box)
    i = (bys[:, None] * bm + np.arange(bm)[None, :]).ravel()
    j = (bxs[:, None] * bn + np.arange(bn)[None, :]).ravel()
    i, j = i[i < m], j[j < n]
    kk = np.arange(k)
    IA, KA = np.meshgrid(i, kk, indexing="ij")
    KB, JB = np.meshgrid(kk, j, indexing="ij")
    IC, JC = np.meshgrid(i, j, indexing="ij")
    return {(0, READ): _uniq([_ravel(IA, KA, (m, k))]),
            (1, READ): _uniq([_ravel(KB, JB, (k, n))]),
            (2, WRITE): _uniq([_ravel(IC, JC, (m, n))])}


def to_byte_ranges(elems: np.ndarray, elem_bytes: int):
    """Sorted unique element indices -> maximal [begin, end) byte ranges."""
    elems = np.asarray(elems, dtype=np.int64)
    if elems.size == 0:
        return []
    breaks = np.nonzero(np.diff(elems) != 1)[0]
    starts = np.concatenate([[elems[0]], elems[breaks + 1]])
    ends = np.concatenate([elems[breaks], [elems[-1]]]) + 1
    return [(int(s) * elem_bytes, int(e) * elem_bytes) for s, e in zip(starts, ends)]


def nbody_soa(box, block, n, per_thread=1):
    """Structure-of-arrays N-body (SURVEY §8(c) paper-vs-validity pin): arguments
    x, y, z (positions in), m (masses, read only), vx, vy, vz (in place), x', y', z'
    (positions out).  Thread tx of block bx owns bodies i = bx*per_thread*bdx + tx + u*bdx,
    guard i < n; it reads x[j], y[j], z[j], m[j] of every body j (all pairs), reads and
    writes vx[i], vy[i], vz[i] and writes x'[i], y'[i], z'[i].  Elements are fp32."""
    bdx = block[0]
    _, _, bxs = _block_ranges(box)
    i = (bxs[:, None] * (per_thread * bdx) + np.arange(per_thread * bdx)[None, :]).ravel()
    i = i[i < n]
    every = np.arange(n, dtype=np.int64) if i.size else np.zeros(0, dtype=np.int64)
    own = _uniq([i])
    out = {}
    for a in range(4):                       # x, y, z, m: every body
        out[(a, READ)] = every
    for a in range(4, 7):                    # vx, vy, vz: own bodies, in place
        out[(a, READ)] = own
        out[(a, WRITE)] = own
    for a in range(7, 10):                   # x', y', z': own bodies
        out[(a, WRITE)] = own
    return out
