"""Shadow-memory tracker replaying the paper's launch sequence -- TEST INFRASTRUCTURE ONLY.

SURVEY.md §8(c) row c3.  One P-bit validity mask per ELEMENT (no interval data
structure at all), updated in the order of PAPER.md Fig. 4:

  for each partition p:  for each read array: buffer_synchronize      (l. 2-7)
  [barrier]                                                            (l. 8)
  for each partition p:  launch                                        (l. 10-19)
  for each partition p:  for each written array: buffer_update         (l. 21-26)

buffer_synchronize (§8.3): every element of p's read set whose
latest copy is not on p is stale and is copied "from its most recently
written to GPU".  buffer_update: p's write set now points to p.

Readings:
  Q2  H2D is a linear element-granular distribution [floor(p n/P), floor((p+1) n/P)).
  Q3  a never-uploaded buffer is valid on every partition.
  Q4  default = validity bitmask (a reader becomes a co-holder); single_owner=True
      reproduces the paper's "does not support shared copies".
  Q5  source = the holder q minimising |q - p|, ties to the lower q, chosen from
      the masks as they were BEFORE this launch's synchronisation.
  Q6  a "may" write is synchronised as a read and owned as a write.
  P:L568-577  two partitions writing the same element is a WAW hazard -> error.
  Q25 halo push (PK_MODE_PUSH, not in the paper, which only pulls): after the update,
      for a push-capable output buffer that this launch does not read, the elements
      writer q wrote that partition p read in the last launch that read the buffer
      become valid on p as well -- unless q's pushes would need more than 16 contiguous
      byte runs in total (then q pushes nothing; those bytes are pulled later).
"""
from __future__ import annotations

import numpy as np


class WriteOverlap(Exception):
    pass


class ShadowBuffer:
    def __init__(self, nelem: int, elem_bytes: int, nparts: int):
        self.nelem = int(nelem)
        self.eb = int(elem_bytes)
        self.nparts = nparts
        # Q3: undefined contents are valid everywhere.
        self.mask = np.full(self.nelem, (1 << nparts) - 1, dtype=np.uint64)

    def h2d_linear(self):
        """Q2 / P:L881-895: host buffer split linearly over the partitions."""
        n, P = self.nelem, self.nparts
        for p in range(P):
            self.mask[(p * n) // P:((p + 1) * n) // P] = np.uint64(1 << p)

    def h2d_for(self, read_sets):
        """Read-pattern-aware upload (SURVEY NEXT-1 of P:L888-895): element e goes to
        every partition whose read set contains it; unread elements keep the linear slab."""
        n, P = self.nelem, self.nparts
        m = np.zeros(n, dtype=np.uint64)
        for p, r in enumerate(read_sets):
            if r is not None and len(r):
                m[np.asarray(r, dtype=np.int64)] |= np.uint64(1 << p)
        for p in range(P):
            sl = slice((p * n) // P, ((p + 1) * n) // P)
            part = m[sl]
            part[part == 0] = np.uint64(1 << p)
            m[sl] = part
        self.mask = m

    def rle(self):
        """Canonical (begin_byte, end_byte, mask) runs covering the buffer."""
        m = self.mask
        if m.size == 0:
            return []
        cut = np.nonzero(m[1:] != m[:-1])[0] + 1
        starts = np.concatenate([[0], cut])
        ends = np.concatenate([cut, [m.size]])
        return [(int(s) * self.eb, int(e) * self.eb, int(m[s])) for s, e in zip(starts, ends)]


def choose_source(mask: int, p: int, nparts: int) -> int:
    """Q5: nearest holder, ties to the lower index."""
    best = None
    for q in range(nparts):
        if (mask >> q) & 1:
            key = (abs(q - p), q)
            if best is None or key < best[0]:
                best = (key, q)
    return best[1]


MAX_PUSH_RUNS = 16


def _runs(el):
    """Number of contiguous runs in a sorted element index array."""
    el = np.asarray(el)
    return 0 if el.size == 0 else int(np.count_nonzero(np.diff(el) != 1)) + 1


class Shadow:
    def __init__(self, nparts: int, single_owner: bool = False):
        self.P = nparts
        self.single_owner = single_owner
        self.buffers = {}
        self.stale_bytes = 0
        self.pushed_bytes = 0
        self.last_read = {}   # name -> [elements p read in the last launch that read it] (Q25)
        self.pair_bytes = np.zeros((nparts, nparts), dtype=np.int64)

    def register(self, name, nelem, elem_bytes, uploaded: bool):
        b = ShadowBuffer(nelem, elem_bytes, self.P)
        if uploaded:
            b.h2d_linear()
        self.buffers[name] = b
        return b

    def launch(self, per_part, push=()):
        """per_part[p] = {buffer_name: (read_elems, write_elems)} (None for empty partitions);
        push = names of the buffers the kernel may halo-push (Q25; empty: the paper's pull only).

        Returns {"stale": [bytes per p], "copies": {(name, src, dst): sorted elems}}.
        """
        P = self.P
        # injective writes across partitions, else WAW.
        for name in self.buffers:
            owner = {}
            seen = np.zeros(self.buffers[name].nelem, dtype=np.int64)
            for p in range(P):
                if per_part[p] is None or name not in per_part[p]:
                    continue
                w = per_part[p][name][1]
                if w is not None and len(w):
                    seen[w] += 1
            if np.any(seen > 1):
                raise WriteOverlap(name)
            del owner
        pre = {name: b.mask.copy() for name, b in self.buffers.items()}
        stale = [0] * P
        copies = {}
        # Fig. 4 lines 2-7: synchronise every read set against the pre-launch state.
        for p in range(P):
            if per_part[p] is None:
                continue
            for name, (r, _w) in per_part[p].items():
                if r is None or len(r) == 0:
                    continue
                b = self.buffers[name]
                m = pre[name][r]
                st = r[(m >> np.uint64(p)) & np.uint64(1) == 0]
                stale[p] += int(st.size) * b.eb
                if st.size:
                    ms = pre[name][st]
                    for mv in np.unique(ms):
                        q = choose_source(int(mv), p, P)
                        el = st[ms == mv]
                        key = (name, q, p)
                        copies[key] = np.union1d(copies.get(key, np.zeros(0, np.int64)), el)
                        self.pair_bytes[q, p] += int(el.size) * b.eb
        # Validity mode: the reader becomes a co-holder (not in the paper's tracker).
        if not self.single_owner:
            for p in range(P):
                if per_part[p] is None:
                    continue
                for name, (r, _w) in per_part[p].items():
                    if r is not None and len(r):
                        self.buffers[name].mask[r] |= np.uint64(1 << p)
        # Fig. 4 lines 21-26: buffer_update, writes now owned by p only.
        for p in range(P):
            if per_part[p] is None:
                continue
            for name, (_r, w) in per_part[p].items():
                if w is not None and len(w):
                    self.buffers[name].mask[w] = np.uint64(1 << p)
        # Q25: halo push of written buffers that this launch does not read
        if not self.single_owner:
            for name in push:
                if any(per_part[p] is not None and name in per_part[p] and per_part[p][name][0] is not None
                       and len(per_part[p][name][0]) for p in range(P)):
                    continue
                last = self.last_read.get(name)
                if last is None:
                    continue
                for q in range(P):
                    if per_part[q] is None or name not in per_part[q]:
                        continue
                    w = per_part[q][name][1]
                    if w is None or not len(w):
                        continue
                    xs = {p: np.intersect1d(w, last[p]) for p in range(P)
                          if p != q and last[p] is not None and len(last[p])}
                    xs = {p: x for p, x in xs.items() if x.size}
                    if not xs or sum(_runs(x) for x in xs.values()) > MAX_PUSH_RUNS:
                        continue
                    for p, x in xs.items():
                        self.buffers[name].mask[x] |= np.uint64(1 << p)
                        self.pushed_bytes += int(x.size) * self.buffers[name].eb
        # read sets of this launch: the prediction for the next writer (Q25)
        for p in range(P):
            if per_part[p] is None:
                continue
            for name, (r, _w) in per_part[p].items():
                if r is not None and len(r):
                    self.last_read.setdefault(name, [None] * P)[p] = np.asarray(r)
        self.stale_bytes += sum(stale)
        return {"stale": stale, "copies": copies}
