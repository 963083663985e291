"""Poison test: every byte a kernel's RESULT depends on is declared (SURVEY.md §5 / hard
part H5; P:L568-569 reads may over-approximate but must cover the kernel's reads).

For every builtin (tests/access_cases.py) at P = 3 partitions, with caller-owned torch
instances: before every launch, each partition's instance is overwritten with NaN on
every byte the validity tracker does NOT hold valid on that partition (pk_tracker_dump).
Those bytes are garbage by the method's own bookkeeping; if a kernel used any of them
without declaring it -- e.g. the TMA halo over-fetch the access-recording test
(tests/test_gpu_trace.py) reports -- the NaN would reach the output.  The results must
equal an unpoisoned run bit for bit.
"""
import numpy as np
import pytest
import torch

import access_cases as AC
from paper_conf_icppw_matzdf20_b200 import abi

pytestmark = pytest.mark.gpu


def _run(name, poison):
    P = max(AC.parts(name))
    ctx = abi.pk_init(P, part_device=[0] * P)
    tensors = {}

    def make(shape, eb, host):
        nfloat = int(np.prod(shape)) * eb // 4
        ts = [torch.zeros(nfloat, dtype=torch.float32, device="cuda:0") for _ in range(P)]
        torch.cuda.synchronize()
        b = abi.pk_register_buffer(ctx, shape, eb, dev_ptrs=[t.data_ptr() for t in ts], host_init=host)
        tensors[b] = ts
        return b

    kid, launches, buffers = AC.CASES[name](ctx, make)
    poisoned = 0
    for grid, blk, args, sc in launches:
        if poison:
            abi.pk_synchronize(ctx)
            for b, ts in tensors.items():
                for (lo, hi, mask) in abi.pk_tracker_dump(ctx, b):
                    for p in range(P):
                        if not (mask >> p) & 1:
                            ts[p][lo // 4:hi // 4] = float("nan")
                            poisoned += (hi - lo) // 4
            torch.cuda.synchronize()
        abi.pk_launch_partitioned(ctx, kid, grid, blk, args, sc)
    out = {}
    for b, (shape, eb) in buffers.items():
        h = np.empty(int(np.prod(shape)) * eb // 4, dtype=np.float32)
        abi.pk_sync_to_host(ctx, b, h)
        out[b] = h
    abi.pk_finalize(ctx)
    return out, poisoned


@pytest.mark.parametrize("name", list(AC.CASES))
def test_undeclared_bytes_do_not_reach_results(name):
    ref, _ = _run(name, False)
    got, poisoned = _run(name, True)
    assert poisoned > 0
    for b in ref:
        assert np.array_equal(ref[b].view(np.uint32), got[b].view(np.uint32)), (name, b)
        assert not np.isnan(got[b]).any()
