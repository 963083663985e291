"""Probe: hotspot2d_tbk at K = 2..8 against the oracle on a small ragged grid, P = 1 vs 3 bit-identity."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import synth
from oracle import kernels as ok
from paper_conf_icppw_matzdf20_b200 import abi, kernels as K

h, w = 300, 2048
t, p = synth.hotspot_grids(h, w)
for k in (2, 3, 4, 5, 6, 7, 8):
    it = 3 * k
    ref = ok.hotspot2d(t, p, it)
    rms = float(np.sqrt(np.mean(ref * ref)))
    outs = []
    for P in (1, 3):
        ctx = abi.pk_init(P, part_device=[0] * P)
        pr = K.hotspot2d_setup(ctx, t, p, ty=32, kernel="hotspot2d_tbk", sweeps=k)
        out = K.hotspot2d_iterate(pr, it)
        g = np.empty_like(t)
        abi.pk_sync_to_host(ctx, out, g)
        abi.pk_finalize(ctx)
        outs.append(g)
    err = np.max(np.abs(outs[0] - ref) / np.maximum(np.abs(ref), rms))
    print("K", k, "err", err, "bitid", np.array_equal(outs[0], outs[1]))
