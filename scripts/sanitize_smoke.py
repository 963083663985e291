"""Small invocation of every builtin kernel (P = 2 virtual partitions) for compute-sanitizer.

    compute-sanitizer --tool memcheck python scripts/sanitize_smoke.py
    compute-sanitizer --tool racecheck python scripts/sanitize_smoke.py
"""
import sys

import numpy as np

sys.path.insert(0, ".")
import synth  # noqa: E402
from paper_conf_icppw_matzdf20_b200 import abi  # noqa: E402
from paper_conf_icppw_matzdf20_b200 import kernels as K  # noqa: E402


def main():
    P = 2
    ctx = abi.pk_init(P, part_device=[0] * P)
    u = synth.jacobi_grid(70, 90)
    _, jb = K.jacobi2d_program(ctx, u, 3)
    pj, _ = K.jacobi2d_program(ctx, u, 0)               # launch sequences (graph capture + replay, PDL)
    for s in range(4):
        K.jacobi2d_iterate(pj, 4, 4 * s, sequence=True)
    t, p = synth.hotspot_grids(150, 1100)
    pr = K.hotspot2d_setup(ctx, t, p, ty=16)
    hb = K.hotspot2d_iterate(pr, 3)
    pr2 = K.hotspot2d_setup(ctx, t, p, ty=16, bdx=64, kernel="hotspot2d_regs")
    K.hotspot2d_iterate(pr2, 2)
    h = synth.heat_grid(20, 70, 260)
    ph = K.heat3d_setup(ctx, h, zc=8, bdy=61)
    K.heat3d_iterate(ph, 3)
    ph2 = K.heat3d_setup(ctx, h, zc=8, bdy=8, kernel="heat3d_regs")
    K.heat3d_iterate(ph2, 2)
    for kern, kw in (("hotspot2d_tb2", {}), ("hotspot2d_tbk", {"sweeps": 4}), ("hotspot2d_tbk", {"sweeps": 8})):
        pk = K.hotspot2d_setup(ctx, t, p, ty=16, kernel=kern, **kw)
        K.hotspot2d_iterate(pk, 8 if kw.get("sweeps") == 8 else 4)
    ph3 = K.heat3d_setup(ctx, h, zc=8, kernel="heat3d_tb2")
    K.heat3d_iterate(ph3, 4)
    # asynchronous host copies and the fused halo push
    import torch
    tp = torch.from_numpy(t).pin_memory()
    abi.pk_copy_from_host_async(ctx, pr.tb[0], tp)
    hb2 = K.hotspot2d_iterate(pr, 3)
    ho = torch.empty(t.shape, dtype=torch.float32).pin_memory()
    abi.pk_sync_to_host_async(ctx, hb2, ho)
    abi.pk_synchronize(ctx)
    abi.pk_set_mode(ctx, abi.PK_MODE_PUSH)
    pp = K.hotspot2d_setup(ctx, t, p, ty=16, kernel="hotspot2d_tbk", sweeps=4)
    K.hotspot2d_iterate(pp, 12)
    ph4 = K.heat3d_setup(ctx, h, zc=8, kernel="heat3d_tb2")
    K.heat3d_iterate(ph4, 6)
    abi.pk_synchronize(ctx)
    abi.pk_set_mode(ctx, 0)
    pos, vel = synth.nbody_bodies(3000)
    pn = K.nbody_setup(ctx, pos, vel)
    K.nbody_iterate(pn, 2)
    a, b = synth.gemm_operands(300, 520, 200)
    _, cb = K.sgemm_program(ctx, a, b)
    out = np.empty((300, 520), np.float32)
    abi.pk_sync_to_host(ctx, cb, out)
    abi.pk_synchronize(ctx)
    abi.pk_finalize(ctx)
    print("sanitize smoke done", float(out[0, 0]))


if __name__ == "__main__":
    main()
