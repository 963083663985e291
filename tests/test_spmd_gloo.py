"""Multi-process SPMD path on CPU: world_size-2 gloo process group, host-only contexts.

Every rank runs the same pk_* sequence (one partition per rank).  The replicated
host state -- regions, stale detection, copy plan, tracker -- must be identical
on every rank and identical to the single-process plan, and the cross-rank copies
each rank would issue (NCCL send on the source's rank, recv on the destination's
rank, in global plan order) must pair up exactly.  (Execution needs one GPU per
rank and NCCL, which this CPU suite cannot run; the plan it executes is what is
checked here.)
"""
import os
import socket

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _sequence(abi, K, ctx, kernel, world):
    """Run a short launch sequence; return per-launch (plan, stats delta, tracker dumps)."""
    out = []
    if kernel == "hotspot2d":
        h, w = 64, 1024
        t = np.zeros((h, w), np.float32)
        pr = K.hotspot2d_setup(ctx, t, t, ty=8)
        for it in range(4):
            K.hotspot2d_iterate(pr, 1, start=it)
            out.append((abi.pk_last_plan(ctx), abi.pk_get_stats(ctx)["stale_bytes"],
                        [abi.pk_tracker_dump(ctx, b) for b in pr.tb]))
    elif kernel == "nbody":
        n = 2048
        pos = np.zeros((n, 4), np.float32)
        pr = K.nbody_setup(ctx, pos, pos, bdx=64)
        for s in range(3):
            K.nbody_iterate(pr, 1, start=s)
            out.append((abi.pk_last_plan(ctx), abi.pk_get_stats(ctx)["stale_bytes"],
                        [abi.pk_tracker_dump(ctx, b) for b in pr.nb]))
    elif kernel == "jacobi2d_seq":
        # the same 5 Jacobi launches as below, issued as pk_launch_sequence chunks of 2 + 3
        n = 64
        pr, _ = K.jacobi2d_program(ctx, np.zeros((n, n), np.float32), 0)
        t = 0
        for c in (2, 3):
            K.jacobi2d_iterate(pr, c, t, sequence=True)
            t += c
            out.append((abi.pk_last_plan(ctx), abi.pk_get_stats(ctx)["stale_bytes"],
                        [abi.pk_tracker_dump(ctx, x) for x in pr.bufs]))
    else:
        n = 64
        pr = K.Problem(ctx, "jacobi2d")
        u = np.zeros((n, n), np.float32)
        b0, b1 = pr.buffer((n, n), 4, host=u), pr.buffer((n, n), 4, host=u)
        grid, blk, sc = K.jacobi2d_launch(n, n)
        for t in range(5):
            a, b = (b0, b1) if t % 2 == 0 else (b1, b0)
            pr.launch(grid, blk, [a, b, n, n], sc)
            out.append((abi.pk_last_plan(ctx), abi.pk_get_stats(ctx)["stale_bytes"],
                        [abi.pk_tracker_dump(ctx, x) for x in (b0, b1)]))
    return out


def _worker(rank, world, port, kernel, qdir, transport="nccl"):
    import sys
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_icppw_matzdf20_b200 import abi
    from paper_conf_icppw_matzdf20_b200 import kernels as K
    if transport == "ipc":   # peer-memory transport: the host all-gather callback runs (handshake)
        from paper_conf_icppw_matzdf20_b200 import spmd
        ctx = abi.pk_init_spmd_ipc(world, rank, world, list(range(world)), spmd.dist_allgather(),
                                   flags=abi.PK_INIT_HOST_ONLY)
    else:
        ctx = abi.pk_init_spmd(world, rank, world, list(range(world)), flags=abi.PK_INIT_HOST_ONLY)
    seq = _sequence(abi, K, ctx, kernel, world)
    st = abi.pk_get_stats(ctx)
    launches = st["kernel_launches"]
    abi.pk_finalize(ctx)
    allseq = [None] * world
    dist.all_gather_object(allseq, (seq, launches, st["collectives"]))
    if rank == 0:
        import pickle
        with open(os.path.join(qdir, "res.pkl"), "wb") as f:
            pickle.dump(allseq, f)
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("kernel,transport", [("jacobi2d", "nccl"), ("hotspot2d", "nccl"), ("nbody", "nccl"),
                                              ("hotspot2d", "ipc"), ("nbody", "ipc")])
def test_spmd_two_ranks_replicated_plan_and_matched_transfers(kernel, transport, tmp_path):
    world = 2
    mp.spawn(_worker, args=(world, _free_port(), kernel, str(tmp_path), transport), nprocs=world, join=True)
    import pickle
    allseq = pickle.load(open(tmp_path / "res.pkl", "rb"))
    (seq0, l0, c0), (seq1, l1, c1) = allseq
    # NCCL transport: the N-body position reads (every partition reads all bodies, slab
    # holders in rank order) are one in-place all-gather per step; stencils have none
    assert c0 == c1 == (3 if (kernel == "nbody" and transport == "nccl") else 0)
    # 1. replicated host state is identical on both ranks
    assert seq0 == seq1
    # 2. ... and identical to the single-process plan for the same P
    from paper_conf_icppw_matzdf20_b200 import abi
    from paper_conf_icppw_matzdf20_b200 import kernels as K
    ref_ctx = abi.pk_init(world, flags=abi.PK_INIT_HOST_ONLY)
    ref = _sequence(abi, K, ref_ctx, kernel, world)
    abi.pk_finalize(ref_ctx)
    assert seq0 == ref
    # 3. every rank launches only its own partition
    assert l0 == l1 == len(seq0)
    # 4. NCCL pairing: rank r's sends to s, in plan order, are exactly rank s's recvs from r
    owner = list(range(world))
    moved = 0
    for plan, _, _ in seq0:
        for r in range(world):
            for s in range(world):
                if r == s:
                    continue
                sends = [(b, lo, hi) for (b, src, dst, lo, hi) in plan if owner[src] == r and owner[dst] == s]
                recvs = [(b, lo, hi) for (b, src, dst, lo, hi) in plan if owner[dst] == s and owner[src] == r]
                assert sends == recvs
                moved += sum(hi - lo for (_, lo, hi) in sends)
    assert moved == seq0[-1][1] > 0          # all stale bytes cross ranks (one partition per rank)


@pytest.mark.parametrize("transport", ["nccl", "ipc"])
def test_spmd_launch_sequence_replicated(transport, tmp_path):
    """pk_launch_sequence in SPMD contexts (issued launch by launch there): replicated state
    identical on both ranks, equal to the single-process sequence, and after the 5 launches
    equal to the same launches issued one by one."""
    world = 2
    mp.spawn(_worker, args=(world, _free_port(), "jacobi2d_seq", str(tmp_path), transport), nprocs=world, join=True)
    import pickle
    (seq0, l0, _), (seq1, l1, _) = pickle.load(open(tmp_path / "res.pkl", "rb"))
    assert seq0 == seq1 and l0 == l1 == 5
    from paper_conf_icppw_matzdf20_b200 import abi
    from paper_conf_icppw_matzdf20_b200 import kernels as K
    ref_ctx = abi.pk_init(world, flags=abi.PK_INIT_HOST_ONLY)
    ref = _sequence(abi, K, ref_ctx, "jacobi2d_seq", world)
    abi.pk_finalize(ref_ctx)
    assert seq0 == ref
    one_ctx = abi.pk_init(world, flags=abi.PK_INIT_HOST_ONLY)
    single = _sequence(abi, K, one_ctx, "jacobi2d", world)
    abi.pk_finalize(one_ctx)
    assert seq0[-1][1:] == single[-1][1:]           # same stale bytes and trackers after 5 launches
    assert seq0[0][1:] == single[1][1:]             # ... and after the first chunk of 2


def _mismatch_worker(rank, world, port, qdir):
    import sys
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_icppw_matzdf20_b200 import abi, spmd
    part_rank = [0, 1] if rank == 0 else [1, 0]      # the ranks disagree on the partition map
    err = None
    try:
        ctx = abi.pk_init_spmd_ipc(2, rank, world, part_rank, spmd.dist_allgather(), flags=abi.PK_INIT_HOST_ONLY)
        abi.pk_finalize(ctx)
    except abi.PkError as e:
        err = e.name
    with open(os.path.join(qdir, f"r{rank}.txt"), "w") as f:
        f.write(str(err))
    dist.barrier()
    dist.destroy_process_group()


def test_spmd_ipc_handshake_rejects_inconsistent_ranks(tmp_path):
    """pk_init_spmd_ipc's collective handshake: every rank fails PK_ERR_INVALID."""
    mp.spawn(_mismatch_worker, args=(2, _free_port(), str(tmp_path)), nprocs=2, join=True)
    assert [(tmp_path / f"r{r}.txt").read_text() for r in range(2)] == ["PK_ERR_INVALID"] * 2
