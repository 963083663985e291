"""GEMM debug: error vs the fp64 oracle and zero fraction for several shapes (P = 1, 2)."""
import sys
import numpy as np
sys.path.insert(0, ".")
sys.path.insert(0, "tests")
import synth
from oracle import kernels as ok
from paper_conf_icppw_matzdf20_b200 import abi
from paper_conf_icppw_matzdf20_b200 import kernels as K
from gpu_util import fetch, gpu_ctx, rel_ok

shapes = [tuple(int(x) for x in s.split("x")) for s in sys.argv[1:]] or [(256, 256, 512), (256, 256, 1024), (256, 512, 2048), (384, 512, 4096)]
for (m, n, k) in shapes:
    a, b = synth.gemm_operands(m, n, k)
    for P in (1, 2):
        ctx = gpu_ctx(P)
        _, cb = K.sgemm_program(ctx, a, b)
        g = fetch(ctx, cb, (m, n))
        abi.pk_finalize(ctx)
        if m * n * k <= 1 << 31:
            ref = ok.gemm(a, b)
            good, err = rel_ok(g, ref, 1e-4)
        else:
            rows = np.arange(0, m, m // 64); cols = np.arange(0, n, n // 64)
            R, Cc = np.meshgrid(rows, cols, indexing="ij")
            ref = ok.gemm_entries(a, b, R.ravel(), Cc.ravel())
            good, err = rel_ok(g[R.ravel(), Cc.ravel()], ref, 1e-4)
        print(m, n, k, "P", P, "ok" if good else "BAD", "err", err, "zeros", float((g == 0).mean()), g.ravel()[:4], flush=True)
