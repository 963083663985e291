"""Access-recording worker (run by tests/test_gpu_trace.py in a subprocess with
PK_TRACE_ACCESS=1, so that abi loads libpk_trace.so) -- test infrastructure.

For every case of tests/access_cases.py and P partitions on cuda:0: run the case's
launches one at a time; before each, clear the bitmaps; after it, compare per
(buffer, partition):
  stored  == declared writes (pk_enumerate, PK_WRITE)          -- exact
  fetched <= declared reads dilated by the case's stated TMA over-fetch
and print one JSON line per case.
"""
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import access_cases as AC  # noqa: E402
from paper_conf_icppw_matzdf20_b200 import abi  # noqa: E402


def run(name, P):
    ctx = abi.pk_init(P, part_device=[0] * P)
    abi.pk_set_mode(ctx, abi.PK_MODE_NO_GRAPHS)

    def make(shape, eb, host):
        return abi.pk_register_buffer(ctx, shape, eb, host_init=host)

    kid, launches, buffers = AC.CASES[name](ctx, make)
    res = {"case": name, "P": P, "launches": len(launches), "write_mismatch": [], "read_outside": [],
           "overfetch_words": 0, "declared_unfetched_words": 0, "stored_words": 0, "fetched_words": 0}
    for li, launch in enumerate(launches):
        abi.pk_trace_reset(ctx)
        grid, blk, args, sc = launch
        abi.pk_launch_partitioned(ctx, kid, grid, blk, args, sc)
        dec = AC.declared(ctx, kid, launch, buffers, P)
        for (b, p), (r, w) in dec.items():
            shape, eb = buffers[b]
            nbytes = int(np.prod(shape)) * eb
            fetched = abi.pk_trace_fetch(ctx, b, p, 0, nbytes)
            stored = abi.pk_trace_fetch(ctx, b, p, 1, nbytes)
            res["stored_words"] += int(stored.sum())
            res["fetched_words"] += int(fetched.sum())
            if not np.array_equal(stored, w):
                res["write_mismatch"].append({"launch": li, "buf": int(b), "part": p,
                                              "extra": int((stored & ~w).sum()), "missing": int((w & ~stored).sum())})
            arg = [a for a, x in enumerate(args) if x == b and r.any()]
            ov = (0, 0, 0)
            for a in arg:
                ov = tuple(max(u, v) for u, v in zip(ov, AC.OVERFETCH.get((name, a), (0, 0, 0))))
            allowed = AC.dilate(r, shape, eb, *ov) if any(ov) else r
            outside = fetched & ~allowed
            if outside.any():
                idx = np.nonzero(outside)[0]
                res["read_outside"].append({"launch": li, "buf": int(b), "part": p, "words": int(idx.size),
                                            "first": int(idx[0])})
            res["overfetch_words"] += int((fetched & ~r).sum())
            res["declared_unfetched_words"] += int((r & ~fetched).sum())
    res["stray"] = abi.pk_trace_stray(ctx)
    abi.pk_finalize(ctx)
    return res


if __name__ == "__main__":
    assert abi.pk_trace_available(), "libpk_trace.so not loaded (PK_TRACE_ACCESS=1)"
    cases = sys.argv[1].split(",") if len(sys.argv) > 1 else list(AC.CASES)
    for name in cases:
        for P in AC.parts(name):
            print(json.dumps(run(name, P)), flush=True)
