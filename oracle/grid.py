"""Grid partitioning, plain definition -- TEST INFRASTRUCTURE ONLY.

PAPER.md P:L607 (§5, task (1) "Partition the execution grid for the available
GPUs"), P:L803-815 (§7: a partition is a 3-tuple of half-open block intervals;
Eq. 8-10) and P:L580-581 (a per-kernel "suggested partitioning strategy").  The
paper does not say how the grid is split; reading Q1: split the
slowest grid dimension whose size exceeds 1 (z, then y, then x) unless the kernel
names one, into P balanced contiguous block ranges [floor(pG/P), floor((p+1)G/P)).

Boxes are 6-tuples in the paper's z, y, x order:
(zmin, zmax, ymin, ymax, xmin, xmax), half-open, in thread blocks.
"""
from __future__ import annotations

X, Y, Z = 0, 1, 2


def split_dim(grid, forced: int = -1) -> int:
    """grid = (gx, gy, gz).  Returns 0/1/2 for x/y/z."""
    if forced >= 0:
        return forced
    for w in (Z, Y, X):
        if grid[w] > 1:
            return w
    return X


def partition_box(grid, nparts: int, p: int, forced: int = -1):
    w = split_dim(grid, forced)
    lo = [0, 0, 0]
    hi = [int(grid[0]), int(grid[1]), int(grid[2])]
    g = hi[w]
    lo[w] = (p * g) // nparts
    hi[w] = ((p + 1) * g) // nparts
    return (lo[Z], hi[Z], lo[Y], hi[Y], lo[X], hi[X])


def tile_box(grid, tiles, p: int):
    """Tile partitions ("suggested partitioning
    strategy"; reading Q24 in DESIGN.md §3): tiles = (tx, ty, tz), tx*ty*tz = P.
    Partition p is tile (p mod tx, (p div tx) mod ty, p div (tx*ty)), x fastest;
    along every dimension the tile index i of t takes blocks [floor(iG/t), floor((i+1)G/t))."""
    tx, ty, tz = (int(t) for t in tiles)
    idx = (p % tx, (p // tx) % ty, p // (tx * ty))
    lo = [idx[d] * int(grid[d]) // (tx, ty, tz)[d] for d in range(3)]
    hi = [(idx[d] + 1) * int(grid[d]) // (tx, ty, tz)[d] for d in range(3)]
    return (lo[Z], hi[Z], lo[Y], hi[Y], lo[X], hi[X])


def box_empty(box) -> bool:
    return box[0] >= box[1] or box[2] >= box[3] or box[4] >= box[5]
