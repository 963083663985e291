"""Host-side plumbing of the multi-process SPMD mode: the host all-gather that
``pk_init_spmd_ipc`` calls back into (handle exchange and barriers at collective
pk_* calls), over an existing torch.distributed process group (gloo or any backend
with CPU tensors).  No arithmetic of the method happens here."""
from __future__ import annotations


def dist_allgather(group=None):
    """Return ``f(data: bytes) -> bytes``: the rank-ordered concatenation of every
    rank's equally sized ``data``."""
    import torch
    import torch.distributed as dist

    def f(data: bytes) -> bytes:
        world = dist.get_world_size(group)
        t = torch.frombuffer(bytearray(data), dtype=torch.uint8) if data else torch.empty(0, dtype=torch.uint8)
        outs = [torch.empty_like(t) for _ in range(world)]
        dist.all_gather(outs, t, group=group)
        return b"".join(bytes(o.numpy().tobytes()) for o in outs)

    return f
