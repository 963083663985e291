#!/usr/bin/env python
"""Measured ceilings behind the roofline denominators (SURVEY.md §8(d) "Measured ceilings on
the box: torch TF32 matmul (allow_tf32), P2P copy bandwidth and latency, NCCL all-gather
busbw").  Prints one JSON object.

    python scripts/probe_peaks.py                 # TF32 matmul, D2D copy, P2P matrix (>= 2 GPUs)
    python scripts/probe_peaks.py --sustained 4   # D2D copy back to back for 4 s (power-limited)
    torchrun --nproc-per-node N scripts/probe_peaks.py --nccl   # NCCL all-gather busbw (N >= 2)

Every number is CUDA-event timed on the device after warm-up; nothing here is used by the
product path (bench.py measures its own TF32 ceiling in the same run).
"""
import argparse
import json
import os

import torch


def ev_time(fn, reps, warm=3):
    for _ in range(warm):
        fn()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


def tf32_matmul(n):
    torch.backends.cuda.matmul.allow_tf32 = True
    a, b = torch.randn(n, n, device="cuda"), torch.randn(n, n, device="cuda")
    ms = ev_time(lambda: torch.matmul(a, b), 10)
    return {"n": n, "ms": ms, "tflops": 2 * n ** 3 / ms / 1e9}


def d2d_copy(nbytes):
    a = torch.empty(nbytes // 4, device="cuda")
    b = torch.empty_like(a)
    ms = ev_time(lambda: b.copy_(a), 20)
    return {"bytes": nbytes, "ms": ms, "gbs_read_plus_write": 2 * nbytes / ms / 1e6}


def d2d_copy_sustained(nbytes, seconds):
    """Back-to-back copies for `seconds` (long enough for the board power limiter to act):
    the sustained HBM figure next to the best-of-20 burst one."""
    a = torch.empty(nbytes // 4, device="cuda")
    b = torch.empty_like(a)
    one = ev_time(lambda: b.copy_(a), 5)
    reps = max(1, int(seconds * 1e3 / one))
    ms = ev_time(lambda: b.copy_(a), reps)
    return {"bytes": nbytes, "reps": reps, "seconds": reps * ms / 1e3, "ms": ms,
            "gbs_read_plus_write": 2 * nbytes / ms / 1e6}


def p2p(src, dst, nbytes):
    a = torch.empty(nbytes // 4, device=f"cuda:{src}")
    b = torch.empty(nbytes // 4, device=f"cuda:{dst}")
    with torch.cuda.device(dst):
        ms = ev_time(lambda: b.copy_(a, non_blocking=True), 20 if nbytes > (1 << 20) else 200)
    return ms


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--nccl", action="store_true")
    ap.add_argument("--sustained", type=float, default=0.0,
                    help="only the sustained D2D copy over this many seconds")
    args = ap.parse_args()
    out = {}
    if args.nccl:
        import torch.distributed as dist
        dist.init_process_group("nccl")
        r, w = dist.get_rank(), dist.get_world_size()
        torch.cuda.set_device(int(os.environ.get("LOCAL_RANK", r)))
        res = []
        for nbytes in (1 << 20, 16 << 20, 128 << 20, 1 << 30):
            per = nbytes // w // 4
            x = torch.empty(per, device="cuda")
            y = torch.empty(per * w, device="cuda")
            ms = ev_time(lambda: dist.all_gather_into_tensor(y, x), 10)
            t = torch.tensor([ms], device="cuda")
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ms = float(t)
            algbw = nbytes / ms / 1e6
            res.append({"bytes": nbytes, "ms": ms, "algbw_gbs": algbw, "busbw_gbs": algbw * (w - 1) / w})
        if r == 0:
            print(json.dumps({"nccl_allgather": res, "world": w}))
        dist.destroy_process_group()
        return
    if args.sustained:
        print(json.dumps({"d2d_copy_sustained": d2d_copy_sustained(1 << 30, args.sustained),
                          "d2d_copy_burst": d2d_copy(1 << 30)}))
        return
    n_dev = torch.cuda.device_count()
    out["device"] = torch.cuda.get_device_name(0)
    out["tf32_matmul"] = [tf32_matmul(n) for n in (8192, 16384)]
    out["d2d_copy_one_gpu"] = [d2d_copy(nb) for nb in (1 << 26, 1 << 30)]
    if n_dev >= 2:
        mat = {}
        for s in range(n_dev):
            for d in range(n_dev):
                if s != d:
                    ms = p2p(s, d, 1 << 30)
                    mat[f"{s}->{d}"] = (1 << 30) / ms / 1e6
        lat = p2p(0, 1, 4096) * 1e3
        out["p2p_gbs_1GiB"] = mat
        out["p2p_latency_us_4KiB_0to1"] = lat
        out["p2p_sizes_0to1"] = {str(nb): nb / p2p(0, 1, nb) / 1e6 for nb in (1 << 16, 1 << 20, 1 << 24, 1 << 28)}
    else:
        out["p2p"] = "skipped: one visible GPU (the partition sweep's transfers are D2D copies on it)"
    print(json.dumps(out))


if __name__ == "__main__":
    main()
