# probe: can two NCCL ranks share one GPU? (SPMD test feasibility on a 1-GPU box)
import os, torch, torch.distributed as dist
dist.init_process_group("nccl")
r = dist.get_rank()
torch.cuda.set_device(0)
x = torch.full((4,), float(r + 1), device="cuda:0")
try:
    dist.all_reduce(x)
    torch.cuda.synchronize()
    print("rank", r, "allreduce ok", x.tolist(), flush=True)
except Exception as e:
    print("rank", r, "FAILED", type(e).__name__, str(e)[:300], flush=True)
dist.destroy_process_group()
