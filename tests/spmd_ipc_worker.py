"""Worker of tests/test_gpu_spmd_ipc.py (launched by torch.distributed.run, one
process per partition, every process on cuda:0 -- the GPU box has one GPU, and
CUDA IPC + stream memory operations work between processes sharing a device the
same way they do between processes on NVSwitch peers).

Each case runs the same host program on every rank through pk_init_spmd_ipc
(replicated plan, pull copies out of IPC-mapped peer instances, device epoch
flags), gathers the result to rank 0 and compares it there with

  * the 1-way result of a single-process P = 1 context (bit-identical),
  * the fp64 CPU oracle (reading Q18 tolerance) where it is cheap,
  * the stale/moved bytes of the closed forms (summed over ranks).

Rank 0 writes a JSON report to argv[1]; any failed check raises -> non-zero exit.
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

import synth  # noqa: E402
from paper_conf_icppw_matzdf20_b200 import abi, spmd  # noqa: E402
from paper_conf_icppw_matzdf20_b200 import kernels as K  # noqa: E402


def main():
    out_path = sys.argv[1]
    dist.init_process_group("gloo")
    rank, world = dist.get_rank(), dist.get_world_size()
    torch.cuda.set_device(0)
    ag = spmd.dist_allgather()
    report = {"world": world, "cases": {}}

    def new_ctx(mode=0):
        ctx = abi.pk_init_spmd_ipc(world, rank, world, list(range(world)), ag, part_device=[0] * world)
        if mode:
            abi.pk_set_mode(ctx, mode)
        return ctx

    def gather(ctx, buf, shape, dtype=np.float32):
        host = np.empty(shape, dtype) if rank == 0 else None
        nbytes = int(np.prod(shape)) * np.dtype(dtype).itemsize
        abi.pk_sync_to_host(ctx, buf, host, nbytes)
        return host

    def summed(ctx):
        st = abi.pk_get_stats(ctx)
        # stale bytes are counted by the replicated plan (identical on every rank); moved
        # bytes, copies and kernels by the rank that pulls / launches them -> summed
        t = torch.tensor([st["moved_bytes"], st["copies"], st["kernel_launches"], st["pushed_bytes"]],
                         dtype=torch.float64)
        dist.all_reduce(t)
        return {"stale": int(st["stale_bytes"]), "moved": int(t[0]), "copies": int(t[1]), "launches": int(t[2]),
                "pushed": int(t[3])}

    def one_way(fn):
        ctx = abi.pk_init(1, part_device=[0])
        try:
            return fn(ctx)
        finally:
            abi.pk_finalize(ctx)

    def record(name, ok, **kw):
        report["cases"][name] = dict(ok=bool(ok), **kw)
        if not ok:
            raise AssertionError(f"{name}: {kw}")

    # --- hotspot2d (one sweep, TMA ring) and hotspot2d_tb2 (two sweeps per launch)
    h, w, iters = 300, 2048, 10
    t, p = synth.hotspot_grids(h, w)
    for kern, ty in (("hotspot2d", 32), ("hotspot2d_tb2", 32), ("hotspot2d_tbk", 32)):
        for mode in (0, abi.PK_MODE_GLOBAL_BARRIER, abi.PK_MODE_PUSH):
            its = 8 if kern == "hotspot2d_tbk" else iters      # K = 4 sweeps per launch
            ctx = new_ctx(mode)
            pr = K.hotspot2d_setup(ctx, t, p, ty=ty, kernel=kern)
            ob = K.hotspot2d_iterate(pr, its)
            g = gather(ctx, ob, (h, w))
            s = summed(ctx)
            abi.pk_finalize(ctx)
            if rank == 0:
                def f1(c):
                    q = K.hotspot2d_setup(c, t, p, ty=ty, kernel=kern)
                    o = K.hotspot2d_iterate(q, its)
                    r = np.empty((h, w), np.float32)
                    abi.pk_sync_to_host(c, o, r)
                    return r
                ref = one_way(f1)
                launches = its // pr.sweeps
                # halo rows per cut and launch: 1 row per sweep of temp (+1 power row for tb2, once)
                ok = np.array_equal(g, ref) and s["stale"] == s["moved"] and s["launches"] == launches * world
                if mode == abi.PK_MODE_PUSH and kern != "hotspot2d_tb2":   # tb2 cannot push
                    ok = ok and s["pushed"] > 0
                record(f"{kern}/mode{mode}", ok, bitwise=bool(np.array_equal(g, ref)), **s)
            dist.barrier()

    # oracle check on one case (fp64 CPU reference, reading Q18)
    if rank == 0:
        from gpu_util import rel_ok
        from oracle import kernels as ok_
        ref = ok_.hotspot2d(t, p, iters)
    ctx = new_ctx()
    pr = K.hotspot2d_setup(ctx, t, p, ty=32)
    K.hotspot2d_iterate(pr, 1)          # the first launch also repairs the linear H2D split (Q2)
    abi.pk_reset_stats(ctx)
    g = gather(ctx, K.hotspot2d_iterate(pr, iters - 1, start=1), (h, w))
    s = summed(ctx)
    abi.pk_finalize(ctx)
    if rank == 0:
        good, err = rel_ok(g, ref, 1e-5)
        expect = (iters - 1) * 2 * w * 4 * (world - 1)  # two 1-row halos per cut per sweep
        record("hotspot2d/oracle", good and s["stale"] == expect == s["moved"], max_err=err, expect=expect, **s)
    dist.barrier()

    # --- C1 Jacobi 512^2, 10 iterations: 40,800 stale bytes at P = 2
    u = synth.jacobi_grid(512, 512)
    ctx = new_ctx()
    _, ob = K.jacobi2d_program(ctx, u, 10)
    g = gather(ctx, ob, (512, 512))
    s = summed(ctx)
    abi.pk_finalize(ctx)
    if rank == 0:
        ref = one_way(lambda c: (lambda pr_ob: _fetch(c, pr_ob[1], (512, 512)))(K.jacobi2d_program(c, u, 10)))
        ok = np.array_equal(g, ref) and (world != 2 or s["stale"] == 40800) and s["stale"] == s["moved"]
        record("jacobi2d/C1", ok, **s)
    dist.barrier()

    # --- heat3d (3-D tensor-TMA ring), ragged z/y/x
    d3, h3, w3 = 40, 36, 132
    u3 = synth.heat_grid(d3, h3, w3)
    ctx = new_ctx()
    pr = K.heat3d_setup(ctx, u3, zc=8, bdy=16)
    g = gather(ctx, K.heat3d_iterate(pr, 6), (d3, h3, w3))
    s = summed(ctx)
    abi.pk_finalize(ctx)
    if rank == 0:
        def f3(c):
            q = K.heat3d_setup(c, u3, zc=8, bdy=16)
            return _fetch(c, K.heat3d_iterate(q, 6), (d3, h3, w3))
        ref = one_way(f3)
        record("heat3d", np.array_equal(g, ref) and s["stale"] == s["moved"], **s)
    dist.barrier()

    # --- nbody: per-step position all-gather (every partition reads every body)
    n = 3000
    pos, vel = synth.nbody_bodies(n)
    ctx = new_ctx()
    pr = K.nbody_setup(ctx, pos, vel, bdx=64)
    pb, vb = K.nbody_iterate(pr, 3)
    gp = gather(ctx, pb, (n, 4))
    gv = gather(ctx, vb, (n, 4))
    s = summed(ctx)
    abi.pk_finalize(ctx)
    if rank == 0:
        def f5(c):
            q = K.nbody_setup(c, pos, vel, bdx=64)
            a, b = K.nbody_iterate(q, 3)
            return _fetch(c, a, (n, 4)), _fetch(c, b, (n, 4))
        rp, rv = one_way(f5)
        record("nbody", np.array_equal(gp, rp) and np.array_equal(gv, rv) and s["stale"] == s["moved"] > 0, **s)
    dist.barrier()

    # --- sgemm 3xTF32: B read whole by every partition (operand broadcast)
    m, nn, kk = 300, 520, 200
    a, b = synth.gemm_operands(m, nn, kk)
    ctx = new_ctx()
    _, cb = K.sgemm_program(ctx, a, b)
    g = gather(ctx, cb, (m, nn))
    s = summed(ctx)
    abi.pk_finalize(ctx)
    if rank == 0:
        ref = one_way(lambda c: _fetch(c, K.sgemm_program(c, a, b)[1], (m, nn)))
        record("sgemm", np.array_equal(g, ref) and s["stale"] == s["moved"] > 0, **s)
    dist.barrier()

    # --- buffer lifecycle: unregister (collective unmap) and re-register, then launch again
    ctx = new_ctx()
    pr = K.hotspot2d_setup(ctx, t, p, ty=32)
    K.hotspot2d_iterate(pr, 2)
    for bb in pr.tb:
        abi.pk_unregister_buffer(ctx, bb)
    pr = K.hotspot2d_setup(ctx, t, p, ty=32)
    g = gather(ctx, K.hotspot2d_iterate(pr, 4), (h, w))
    abi.pk_finalize(ctx)
    if rank == 0:
        def f6(c):
            q = K.hotspot2d_setup(c, t, p, ty=32)
            return _fetch(c, K.hotspot2d_iterate(q, 4), (h, w))
        record("lifecycle", np.array_equal(g, one_way(f6)))
    dist.barrier()

    # --- seeded random launch programs (two kernels on shared ping-pong buffers, collective
    # re-uploads and mid-program gathers), pulled and pushed halos: every read bit-identical
    for seed in (0, 1):
        for mode in (0, abi.PK_MODE_PUSH):
            ctx = new_ctx(mode)
            reads = _random_program(ctx, seed, lambda c, bb, sh: gather(c, bb, sh))
            s = summed(ctx)
            abi.pk_finalize(ctx)
            if rank == 0:
                ref = one_way(lambda c: _random_program(c, seed, _fetch))
                ok = len(reads) == len(ref) and all(np.array_equal(x, y) for x, y in zip(reads, ref))
                record(f"random/{seed}/mode{mode}", ok and s["stale"] == s["moved"], reads=len(reads), **s)
            dist.barrier()

    if rank == 0:
        with open(out_path, "w") as f:
            json.dump(report, f, indent=1)
        print("SPMD-IPC ALL OK", json.dumps({k: v["ok"] for k, v in report["cases"].items()}), flush=True)
    dist.barrier()
    dist.destroy_process_group()


def _random_program(ctx, seed, read, h=200, w=1028):
    """tests/test_gpu_parity.py's random launch program through any context; `read(ctx, buf,
    shape)` returns the host copy (a collective gather in SPMD)."""
    rng = np.random.default_rng(seed)
    t, p = synth.hotspot_grids(h, w)
    t2 = (t + np.float32(1.5)).astype(np.float32)
    k1 = abi.pk_builtin_kernel(ctx, "hotspot2d")
    k4 = abi.pk_builtin_kernel(ctx, "hotspot2d_tbk")
    b = [abi.pk_register_buffer(ctx, (h, w), 4, host_init=t), abi.pk_register_buffer(ctx, (h, w), 4)]
    pw = abi.pk_register_buffer(ctx, (h, w), 4, host_init=p)
    g1, bl1, s1 = K.hotspot2d_launch(h, w, 16, K.HOTSPOT_BDX)
    g4, bl4, s4 = K.hotspot2d_tbk_launch(h, w, 16, 4)
    cur, reads = 0, []
    for op in rng.choice(["s1", "s1", "s4", "s4", "s4", "up", "rd"], size=30):
        if op == "s1":
            abi.pk_launch_partitioned(ctx, k1, g1, bl1, [b[cur], pw, b[1 - cur], h, w, s1[2]], s1)
            cur = 1 - cur
        elif op == "s4":
            abi.pk_launch_partitioned(ctx, k4, g4, bl4, [b[cur], pw, b[1 - cur], h, w, s4[2]], s4)
            cur = 1 - cur
        elif op == "up":
            abi.pk_copy_from_host(ctx, b[cur], t2 if len(reads) % 2 else t)
        else:
            reads.append(read(ctx, b[cur], (h, w)))
    reads.append(read(ctx, b[cur], (h, w)))
    return reads


def _fetch(ctx, buf, shape):
    r = np.empty(shape, np.float32)
    abi.pk_sync_to_host(ctx, buf, r)
    return r


if __name__ == "__main__":
    main()
