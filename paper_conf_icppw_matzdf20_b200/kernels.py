"""Launch geometry of the builtin sm_100a kernels (their published launch contract,
DESIGN.md §4) and user-side programs that drive them through the C-ABI.

These are the single-device host programs of the paper's benchmarks (P:L948-954
Table 1) written against the pk_* calls: register buffers (cudaMalloc +
cudaMemcpy replacements), launch the kernel repeatedly through the
launch replacement (Fig. 4), gather the result.  No arithmetic of
the method happens here.
"""
from __future__ import annotations

import math

from . import abi

# ---------------------------------------------------------------- geometry
JACOBI_BLOCK = (32, 8, 1)
HOTSPOT_BDX, HOTSPOT_TY = 128, 128    # "hotspot2d" (TMA ring) requires bdx = 128
HEAT_BDY, HEAT_ZC = 62, 128           # "heat3d" (TMA ring): bdy <= 62 rows (2 per consumer warp)
NBODY_BDX, NBODY_PER_THREAD = 256, 4


def _cdiv(a, b):
    return -(-a // b)


def jacobi2d_launch(h, w, block=JACOBI_BLOCK):
    return (_cdiv(w, block[0]), _cdiv(h, block[1]), 1), tuple(block), [h, w]


def hotspot2d_launch(h, w, ty=HOTSPOT_TY, bdx=HOTSPOT_BDX):
    return (_cdiv(w, 4 * bdx), _cdiv(h, ty), 1), (bdx, 1, 1), [h, w, ty]


def tbk_cols(k):
    """"hotspot2d_tbk": owned columns per logical block (one halo lane per warp side
    for K <= 4 sweeps, two for K = 5..8)."""
    return 480 if k <= 4 else 448


TBK_COLS = tbk_cols(4)


def hotspot2d_tbk_rows(h, w, k=4, parts=1, ctas=444, lo=48, hi=136):
    """Rows per logical block of "hotspot2d_tbk" for an h x w grid split into `parts` row
    slabs, run by a persistent grid of `ctas` CTAs (148 SMs x 3): the tiles of one partition
    are processed in ceil(tiles / ctas) rounds, and a tile of TY rows costs about
    TY + 2K (halo rows recomputed) + a fixed overhead, so TY minimises rounds x (TY + 2K + 8).
    Measured on one B200 (`scripts/r02/gpu_20.sh`): 16384 rows TY 128 / 131 = 1998 / 2013
    GLUP/s (4480 vs 4410 tiles: 11 vs 10 rounds); 2048 rows (a rank's share at N = 8) TY 64 /
    54 = 1541 / 1626; larger TY than the model's range measured slower (146 / 164 / 218 at
    16384 rows: 1982 / 1924 / 1860)."""
    ncb = _cdiv(w, tbk_cols(k))
    best = None
    for ty in range(lo, hi + 1):
        per = _cdiv(_cdiv(h, ty), parts)          # row blocks of the largest partition
        rounds = _cdiv(per * ncb, ctas)
        if rounds < 3 and ty > lo:
            continue                              # <= 2 tiles per CTA measured poorly (TY 103 at 2048 rows)
        cost = rounds * (ty + 2 * k + 8)
        if best is None or cost < best[0] or (cost == best[0] and ty > best[1]):
            best = (cost, ty)
    return best[1]


def hotspot2d_tbk_launch(h, w, ty=HOTSPOT_TY, k=4):
    """Logical block = tbk_cols(k) columns x ty rows, k sweeps per launch (scalar 3,
    K in 2, 3, 4, 6, 8); scalar 4 = the block's column count."""
    return (_cdiv(w, tbk_cols(k)), _cdiv(h, ty), 1), (128, 1, 1), [h, w, ty, k, tbk_cols(k)]


def heat3d_launch(d, h, w, zc=HEAT_ZC, bdy=HEAT_BDY):
    return (_cdiv(w, 128), _cdiv(h, bdy), _cdiv(d, zc)), (32, bdy, 1), [d, h, w, zc]


HEAT_TB2_COLS, HEAT_TB2_ROWS = 120, 16    # "heat3d_tb2": owned columns x rows per logical block


HEAT_TB2_ZC = 64                          # "heat3d_tb2": planes per logical block (measured: 64 beats 128 by ~3%)


def heat3d_tb2_launch(d, h, w, zc=HEAT_TB2_ZC):
    """Logical block = 120 columns x 16 rows x zc planes, two sweeps per launch."""
    return (_cdiv(w, HEAT_TB2_COLS), _cdiv(h, HEAT_TB2_ROWS), _cdiv(d, zc)), (160, 1, 1), [d, h, w, zc]


HEAT_TB3_ZC = 128                         # "heat3d_tb3": planes per logical block (6 halo planes per block)


def heat3d_tb3_launch(d, h, w, zc=HEAT_TB3_ZC):
    """Logical block = 120 columns x 16 rows x zc planes, three sweeps per launch (256 threads:
    4 row warps, 3 sweep-1 warps, 1 producer warp)."""
    return (_cdiv(w, HEAT_TB2_COLS), _cdiv(h, HEAT_TB2_ROWS), _cdiv(d, zc)), (256, 1, 1), [d, h, w, zc]


def nbody_launch(n, bdx=NBODY_BDX):
    return (_cdiv(n, NBODY_PER_THREAD * bdx), 1, 1), (bdx, 1, 1), [n]


GEMM_BM, GEMM_BN = 128, 256


def sgemm_launch(m, n, k):
    """Logical block = one 128 x 256 C tile (the kernel runs 12 warps per tile)."""
    return (_cdiv(n, GEMM_BN), _cdiv(m, GEMM_BM), 1), (256, 1, 1), [m, n, k]


def sgemm_program(ctx, a_host, b_host, launches=1):
    """C4: upload A (M x K) and B (K x N) (linear H2D), C = A B through the
    partitioned launch; returns (problem, C buffer id)."""
    m, k = a_host.shape
    k2, n = b_host.shape
    assert k == k2
    pr = Problem(ctx, "sgemm_tf32x3")
    a = pr.buffer((m, k), 4, host=a_host)
    b = pr.buffer((k, n), 4, host=b_host)
    c = pr.buffer((m, n), 4)
    grid, blk, sc = sgemm_launch(m, n, k)
    for _ in range(launches):
        pr.launch(grid, blk, [a, b, c, m, n, k], sc)
    pr.geom, pr.mnk, pr.abc = (grid, blk, sc), (m, n, k), (a, b, c)
    return pr, c


# ---------------------------------------------------------------- programs
class Problem:
    """A registered builtin kernel plus its ping-pong buffers on one context."""

    def __init__(self, ctx, kernel_name, tiles=None):
        self.ctx = ctx
        self.k = abi.pk_builtin_kernel(ctx, kernel_name)
        if tiles:   # NEXT-2 tile partitions (tx, ty, tz), tx*ty*tz == P
            abi.pk_set_partition_shape(ctx, self.k, tiles)
        self.bufs = []
        self.direct = False   # True: pk_launch_direct (the E3 single-GPU baseline, P = 1 only)

    def buffer(self, shape, elem_bytes=4, host=None, dev_ptrs=None):
        b = abi.pk_register_buffer(self.ctx, shape, elem_bytes, dev_ptrs=dev_ptrs, host_init=host)
        self.bufs.append(b)
        return b

    def launch(self, grid, block, args, scalars):
        if self.direct:
            abi.pk_launch_direct(self.ctx, self.k, grid, block, args, scalars)
        else:
            abi.pk_launch_partitioned(self.ctx, self.k, grid, block, args, scalars)

    def launch_seq(self, launches):
        """[(grid, block, args, scalars), ...] in order, as one pk_launch_sequence (one graph
        launch in steady state); one by one on the direct (E3 baseline) path."""
        if self.direct:
            for g, b, a, sc in launches:
                abi.pk_launch_direct(self.ctx, self.k, g, b, a, sc)
        else:
            abi.pk_launch_sequence(self.ctx, [(self.k, g, b, a, sc) for g, b, a, sc in launches])


JACOBI_TB_T = 32                          # "jacobi2d_tb": owned rows x columns per logical block


def jacobi2d_tb_launch(h, w, k):
    """Logical block = 32 x 32 cells, k sweeps per launch (256 threads, ghost zones)."""
    return (_cdiv(w, JACOBI_TB_T), _cdiv(h, JACOBI_TB_T), 1), (256, 1, 1), [h, w, k]


def jacobi2d_program(ctx, u_host, iters, block=JACOBI_BLOCK, tiles=None, sequence=False, kernel="jacobi2d",
                     sweeps=1):
    """C1: both buffers carry the Dirichlet boundary (uploaded); returns the buffer id
    that holds the result after `iters` sweeps (sequence=True: the sweeps go out as one
    pk_launch_sequence).  kernel="jacobi2d_tb": `sweeps` (1..16) sweeps per launch."""
    h, w = u_host.shape
    pr = Problem(ctx, kernel, tiles)
    pr.buffer((h, w), 4, host=u_host)
    pr.buffer((h, w), 4, host=u_host)
    pr.sweeps = sweeps if kernel == "jacobi2d_tb" else 1
    pr.geom = jacobi2d_tb_launch(h, w, sweeps) if kernel == "jacobi2d_tb" else jacobi2d_launch(h, w, block)
    pr.cur = 0
    return pr, jacobi2d_iterate(pr, iters, 0, sequence)


def jacobi2d_iterate(pr, iters, start=0, sequence=True):
    """`iters` C1 sweeps from sweep `start` on a jacobi2d_program problem (ping-pong
    u0 -> u1 -> u0 ...), as one pk_launch_sequence or one launch call per sweep; returns
    the buffer id of the result.  jacobi2d_tb: launches of pr.sweeps sweeps, a remainder
    as one shorter launch; the ping-pong state is the launch count (pr.cur)."""
    u0, u1 = pr.bufs[:2]
    grid, blk, sc = pr.geom
    launches = []
    if getattr(pr, "sweeps", 1) > 1:
        k = pr.sweeps
        n, rem = divmod(iters, k)
        for kk in [k] * n + ([rem] if rem else []):
            a, b = pr.bufs[pr.cur], pr.bufs[1 - pr.cur]
            s2 = [sc[0], sc[1], kk]
            launches.append((grid, blk, [a, b, *s2], s2))
            pr.cur = 1 - pr.cur
        if sequence and launches:
            pr.launch_seq(launches)
        else:
            for g, b, a, s in launches:
                pr.launch(g, b, a, s)
        return pr.bufs[pr.cur]
    for t in range(start, start + iters):
        a, b = (u0, u1) if t % 2 == 0 else (u1, u0)
        launches.append((grid, blk, [a, b, sc[0], sc[1]], sc))
    if sequence and launches:
        pr.launch_seq(launches)
    else:
        for g, b, a, s in launches:
            pr.launch(g, b, a, s)
    return u1 if (start + iters) % 2 == 1 else u0


def hotspot2d_setup(ctx, temp_host, power_host, ty=HOTSPOT_TY, bdx=HOTSPOT_BDX, dev_ptrs=None,
                    kernel="hotspot2d", tiles=None, sweeps=4):
    """kernel: hotspot2d (one sweep per launch), hotspot2d_regs, hotspot2d_tb2 (two),
    hotspot2d_tbk (`sweeps` = 2, 3, 4, 6 or 8 per launch)."""
    h, w = temp_host.shape
    pr = Problem(ctx, kernel, tiles)
    t0 = pr.buffer((h, w), 4, host=temp_host, dev_ptrs=dev_ptrs[0] if dev_ptrs else None)
    t1 = pr.buffer((h, w), 4, dev_ptrs=dev_ptrs[1] if dev_ptrs else None)   # undefined (reading Q3)
    pw = pr.buffer((h, w), 4, host=power_host, dev_ptrs=dev_ptrs[2] if dev_ptrs else None)
    if kernel == "hotspot2d_tbk":
        pr.geom = hotspot2d_tbk_launch(h, w, ty, sweeps)
    else:
        pr.geom = hotspot2d_launch(h, w, ty, bdx)
    pr.hw = (h, w)
    pr.tb = (t0, t1, pw)
    pr.sweeps = {"hotspot2d_tb2": 2, "hotspot2d_tbk": sweeps}.get(kernel, 1)   # time steps per launch
    return pr


def hotspot2d_iterate(pr, iters, start=0, sequence=False):
    """`iters` Hotspot time steps starting at step `start` (the tb2/tbk kernels advance
    pr.sweeps steps per launch: iters and start must then be multiples of it);
    sequence=True issues them as one pk_launch_sequence."""
    (t0, t1, pw), (h, w) = pr.tb, pr.hw
    grid, blk, sc = pr.geom
    k = pr.sweeps
    if iters % k or start % k:
        raise ValueError(f"this kernel advances {k} steps per launch")
    launches = []
    for t in range(start // k, (start + iters) // k):
        a, b = (t0, t1) if t % 2 == 0 else (t1, t0)
        launches.append((grid, blk, [a, pw, b, h, w, sc[2]], sc))
    if sequence and launches:
        pr.launch_seq(launches)
    else:
        for g, bl, a, s in launches:
            pr.launch(g, bl, a, s)
    return t1 if ((start + iters) // k) % 2 == 1 else t0


def heat3d_setup(ctx, u_host, zc=None, bdy=HEAT_BDY, kernel="heat3d", tiles=None):
    """kernel: heat3d (one sweep per launch, TMA ring), heat3d_regs, heat3d_tb2 (two), heat3d_tb3 (three)."""
    d, h, w = u_host.shape
    pr = Problem(ctx, kernel, tiles)
    u0 = pr.buffer((d, h, w), 4, host=u_host)
    u1 = pr.buffer((d, h, w), 4)
    if kernel == "heat3d_tb2":
        pr.geom = heat3d_tb2_launch(d, h, w, zc or HEAT_TB2_ZC)
    elif kernel == "heat3d_tb3":
        pr.geom = heat3d_tb3_launch(d, h, w, zc or HEAT_TB3_ZC)
    else:
        pr.geom = heat3d_launch(d, h, w, zc or HEAT_ZC, bdy)
    pr.shape = (d, h, w)
    pr.ub = (u0, u1)
    pr.sweeps = {"heat3d_tb2": 2, "heat3d_tb3": 3}.get(kernel, 1)
    if kernel == "heat3d_tb3":
        # a remainder of 1 or 2 sweeps (C3's 50 = 16 x 3 + 2) runs on heat3d / heat3d_tb2 over the
        # same buffers: every cell is the same expression in all three kernels (bit-identical)
        pr.tail = {1: Problem(ctx, "heat3d", tiles), 2: Problem(ctx, "heat3d_tb2", tiles)}
        pr.tail_geom = {1: heat3d_launch(d, h, w, HEAT_ZC, bdy), 2: heat3d_tb2_launch(d, h, w, HEAT_TB2_ZC)}
        pr.cur = 0
    return pr


def heat3d_iterate(pr, iters, start=0):
    """`iters` sweeps from sweep `start` (multiples of pr.sweeps for heat3d_tb2 / heat3d_tb3)."""
    (u0, u1), (d, h, w) = pr.ub, pr.shape
    grid, blk, sc = pr.geom
    k = pr.sweeps
    if hasattr(pr, "tail"):
        # heat3d_tb3: the ping-pong state is the number of launches so far (pr.cur = buffer
        # holding the current field), since a remainder launch advances fewer sweeps
        n, rem = divmod(iters, k)
        for _ in range(n):
            a, b = pr.ub[pr.cur], pr.ub[1 - pr.cur]
            pr.launch(grid, blk, [a, b, d, h, w, sc[3]], sc)
            pr.cur = 1 - pr.cur
        if rem:
            a, b = pr.ub[pr.cur], pr.ub[1 - pr.cur]
            g2, b2, s2 = pr.tail_geom[rem]
            pr.tail[rem].launch(g2, b2, [a, b, d, h, w, s2[3]], s2)
            pr.cur = 1 - pr.cur
        return pr.ub[pr.cur]
    if iters % k or start % k:
        raise ValueError(f"this kernel advances {k} steps per launch")
    for t in range(start // k, (start + iters) // k):
        a, b = (u0, u1) if t % 2 == 0 else (u1, u0)
        pr.launch(grid, blk, [a, b, d, h, w, sc[3]], sc)
    return u1 if ((start + iters) // k) % 2 == 1 else u0


def nbody_setup(ctx, pos_host, vel_host, bdx=NBODY_BDX):
    n = pos_host.shape[0]
    pr = Problem(ctx, "nbody")
    p0 = pr.buffer((n,), 16, host=pos_host)
    p1 = pr.buffer((n,), 16)
    v = pr.buffer((n,), 16, host=vel_host)
    pr.geom = nbody_launch(n, bdx)
    pr.n = n
    pr.nb = (p0, p1, v)
    return pr


def nbody_iterate(pr, steps, start=0):
    (p0, p1, v), n = pr.nb, pr.n
    grid, blk, sc = pr.geom
    for s in range(start, start + steps):
        a, b = (p0, p1) if s % 2 == 0 else (p1, p0)
        pr.launch(grid, blk, [a, v, b, n], sc)
    return (p1 if (start + steps) % 2 == 1 else p0), v


def flops_per_interaction():
    return 20  # conventional count for the softened all-pairs kernel (SURVEY §8(d) [ext])


def isqrt(n):
    return int(math.isqrt(n))
