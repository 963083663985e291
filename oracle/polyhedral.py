"""Eq. 1-4 integer sets and the row-wise first/last enumeration -- TEST INFRASTRUCTURE ONLY.

PAPER.md P:L281-290 (§2.4, Eq. 1-4):
  S1 := { [y, x] | 0 <= y <= x  and 0 <= x <= 4 }                      (1)
  M  := { [y, x] -> [y', x'] | y' = y + 1  and  x' = x + 3 }            (2)
  S2 := M(S1) = { [y, x] | 1 <= y <= x - 2  and  3 <= x <= 7 }          (3)
  U  := S1 u S2                                                          (4)
(the extraction prints ":=" as "B", reading Q23).

PAPER.md P:L763-775 (§6.1): enumerate only the first and last element of each row
of the image, computed as the lexicographic min and max with all but the last
dimension fixed; exact for a convex set, an over-approximation for a union,
which "can be eliminated by applying this approach to each convex set of the
union instead of the union set itself".

Sets are plain Python sets of integer tuples, built by brute force over a box.
"""
from __future__ import annotations


def S1():
    return {(y, x) for x in range(0, 5) for y in range(0, x + 1)}


def M(points):
    return {(y + 1, x + 3) for (y, x) in points}


def S2_printed():
    """Eq. 3 as printed: 1 <= y <= x - 2 and 3 <= x <= 7."""
    return {(y, x) for x in range(3, 8) for y in range(1, x - 1)}


def U():
    return S1() | M(S1())


def rowwise_first_last(points):
    """Row y -> [min x, max x] of `points`: one range per row."""
    rows = {}
    for (y, x) in points:
        lo, hi = rows.get(y, (x, x))
        rows[y] = (min(lo, x), max(hi, x))
    return {y: [(lo, hi)] for y, (lo, hi) in rows.items()}


def rowwise_per_piece(pieces):
    """Apply row-wise first/last to each convex piece, then union per row."""
    rows = {}
    for piece in pieces:
        for y, rngs in rowwise_first_last(piece).items():
            rows.setdefault(y, []).extend(rngs)
    out = {}
    for y, rngs in rows.items():
        rngs.sort()
        merged = []
        for lo, hi in rngs:
            if merged and lo <= merged[-1][1] + 1:
                merged[-1] = (merged[-1][0], max(merged[-1][1], hi))
            else:
                merged.append((lo, hi))
        out[y] = merged
    return out


def points_of_rows(rows):
    return {(y, x) for y, rngs in rows.items() for (lo, hi) in rngs for x in range(lo, hi + 1)}
