"""Brute-force evaluation of declared affine descriptors -- TEST INFRASTRUCTURE ONLY.

Follows the definition written in include/pk_api.h (pk_dim_map / pk_affine_access)
element by element, without any closed form: for every block index of the
partition box along the tap's grid dimension and every position inside
[b*scale, b*scale + extent), apply the guard, add the offset, clamp or
bounds-check; the tap's image is the Cartesian product over array dims; taps
are unioned as sets.  The library's analyzer computes the same sets as interval
arithmetic (the paper's per-convex-piece row enumeration, §6.1).

Descriptors here are plain dicts so that nothing is shared with the binding:
  dim = {"grid_dim": g, "scale": s, "extent": e, "offset": o,
         "clamp": bool, "guard": (lo, hi) or None}     (ints already evaluated)
"""
from __future__ import annotations

import itertools

import numpy as np


class OutOfBounds(Exception):
    pass


def dim_indices(dim, box6, shape_k):
    g = dim["grid_dim"]
    pos = set()
    if g < 0:
        pos.update(range(0, max(0, dim["extent"])))
    else:
        lo, hi = box6[2 * (2 - g)], box6[2 * (2 - g) + 1]
        for b in range(lo, hi):
            pos.update(range(b * dim["scale"], b * dim["scale"] + max(0, dim["extent"])))
    if dim.get("guard") is not None:
        glo, ghi = dim["guard"]
        pos = {p for p in pos if glo <= p < ghi}
    out = set()
    oob = False
    for p in pos:
        i = p + dim["offset"]
        if dim.get("clamp"):
            i = min(max(i, 0), shape_k - 1)
        elif not (0 <= i < shape_k):
            oob = True
        out.add(i)
    return sorted(out), oob


def tap_elements(tap_dims, box6, shape):
    """Product of the per-dimension sets.  An empty box or an empty dimension set
    means no thread accesses anything (no error); otherwise an unclamped index
    outside [0, shape) is an error."""
    z0, z1, y0, y1, x0, x1 = box6
    if z0 >= z1 or y0 >= y1 or x0 >= x1:
        return np.zeros(0, dtype=np.int64)
    res = [dim_indices(d, box6, shape[k]) for k, d in enumerate(tap_dims)]
    sets = [s for s, _ in res]
    if any(len(s) == 0 for s in sets):
        return np.zeros(0, dtype=np.int64)
    if any(o for _, o in res):
        raise OutOfBounds(shape)
    pts = np.array(list(itertools.product(*sets)), dtype=np.int64)
    return np.ravel_multi_index(tuple(pts.T), shape).astype(np.int64)


def union_elements(taps, box6, shape):
    parts = [tap_elements(t, box6, shape) for t in taps]
    if not parts:
        return np.zeros(0, dtype=np.int64)
    return np.unique(np.concatenate(parts))
