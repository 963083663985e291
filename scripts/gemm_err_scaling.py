# error of the 3xTF32 tcgen05 SGEMM vs fp64 as K grows (Q18 tolerance scaling); cuBLAS FP32 beside it
import sys, numpy as np, torch
sys.path.insert(0, '.'); sys.path.insert(0, 'tests')
import synth
from paper_conf_icppw_matzdf20_b200 import abi, kernels as K
from gpu_util import fetch, gpu_ctx
m = n = 512
for k in (1024, 4096, 16384, 65536):
    a, b = synth.gemm_operands(m, n, k)
    ctx = gpu_ctx(1)
    _, cb = K.sgemm_program(ctx, a, b)
    g = fetch(ctx, cb, (m, n)).astype(np.float64)
    abi.pk_finalize(ctx)
    o = a.astype(np.float64) @ b.astype(np.float64)
    rms = np.sqrt(np.mean(o * o))
    e = np.abs(g - o) / np.maximum(np.abs(o), rms)
    torch.backends.cuda.matmul.allow_tf32 = False
    c32 = (torch.from_numpy(a).cuda() @ torch.from_numpy(b).cuda()).cpu().numpy().astype(np.float64)
    e32 = np.abs(c32 - o) / np.maximum(np.abs(o), rms)
    bias = np.mean((g - o) / rms)
    print(f"K={k}: 3xTF32 max {e.max():.2e} mean {e.mean():.2e} bias {bias:+.2e} | cuBLAS fp32 max {e32.max():.2e} mean {e32.mean():.2e}", flush=True)
