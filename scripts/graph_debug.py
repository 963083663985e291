"""Launch-by-launch comparison of graph replay vs eager execution (debug aid)."""
import sys

import numpy as np

sys.path.insert(0, ".")
import synth  # noqa: E402
from paper_conf_icppw_matzdf20_b200 import abi  # noqa: E402
from paper_conf_icppw_matzdf20_b200 import kernels as K  # noqa: E402


def run(h, w, ty, P, iters, mode):
    t, p = synth.hotspot_grids(h, w)
    ctx = abi.pk_init(P, part_device=[0] * P)
    abi.pk_set_mode(ctx, mode)
    pr = K.hotspot2d_setup(ctx, t, p, ty=ty)
    outs, stats = [], []
    for it in range(iters):
        out = K.hotspot2d_iterate(pr, 1, start=it)
        g = np.empty_like(t)
        abi.pk_sync_to_host(ctx, out, g)
        outs.append(g)
        s = abi.pk_get_stats(ctx)
        stats.append((s["graph_captures"], s["graph_replays"], s["stale_bytes"]))
    abi.pk_finalize(ctx)
    return outs, stats


def run_nosync(h, w, ty, P, iters, mode):
    t, p = synth.hotspot_grids(h, w)
    ctx = abi.pk_init(P, part_device=[0] * P)
    abi.pk_set_mode(ctx, mode)
    pr = K.hotspot2d_setup(ctx, t, p, ty=ty)
    out = K.hotspot2d_iterate(pr, iters)
    g = np.empty_like(t)
    abi.pk_sync_to_host(ctx, out, g)
    s = abi.pk_get_stats(ctx)
    abi.pk_finalize(ctx)
    return g, s


if __name__ == "__main__":
    h, w, ty, P, iters = 129, 1028, 64, 4, 20
    a, sa = run(h, w, ty, P, iters, abi.PK_MODE_NO_GRAPHS)
    b, sb = run(h, w, ty, P, iters, 0)
    for i in range(iters):
        print(i, np.array_equal(a[i], b[i]), sa[i], sb[i], flush=True)
    for P in (2, 3, 4):
        g0, s0 = run_nosync(h, w, ty, P, iters, abi.PK_MODE_NO_GRAPHS)
        g1, s1 = run_nosync(h, w, ty, P, iters, 0)
        bad = np.argwhere(g0 != g1)
        print("nosync P", P, np.array_equal(g0, g1), s1["graph_captures"], s1["graph_replays"],
              "first bad", bad[:3].tolist(), "rows", sorted(set(bad[:, 0].tolist()))[:10] if len(bad) else [],
              flush=True)
