"""Small tcgen05 GEMM probes (run under `timeout`): prints max errors vs numpy."""
import sys
import time

import numpy as np

sys.path.insert(0, ".")
from paper_conf_icppw_matzdf20_b200 import abi  # noqa: E402
from paper_conf_icppw_matzdf20_b200 import kernels as K  # noqa: E402


def run(m, n, k, kind="rand"):
    rng = np.random.default_rng(0)
    if kind == "eye":
        a = np.eye(m, k, dtype=np.float32)
        b = rng.uniform(-1, 1, size=(k, n)).astype(np.float32)
    elif kind == "ones":
        a = np.ones((m, k), np.float32)
        b = np.ones((k, n), np.float32)
    else:
        a = rng.uniform(-1, 1, size=(m, k)).astype(np.float32)
        b = rng.uniform(-1, 1, size=(k, n)).astype(np.float32)
    ctx = abi.pk_init(1, part_device=[0])
    t0 = time.time()
    pr, c = K.sgemm_program(ctx, a, b)
    out = np.empty((m, n), np.float32)
    abi.pk_sync_to_host(ctx, c, out)
    abi.pk_finalize(ctx)
    ref = a.astype(np.float64) @ b.astype(np.float64)
    err = np.abs(out - ref)
    rms = np.sqrt(np.mean(ref ** 2)) + 1e-30
    bad = np.argwhere(err > 1e-3 * np.maximum(np.abs(ref), rms))
    print(f"{kind} {m}x{n}x{k}: max abs err {err.max():.3e} rel/rms {err.max() / rms:.3e} "
          f"bad {len(bad)} t {time.time() - t0:.2f}s", flush=True)
    if len(bad):
        i, j = bad[0]
        print("  first bad", i, j, out[i, j], ref[i, j], " row0:", out[0, :6], ref[0, :6], flush=True)


if __name__ == "__main__":
    for args in [(128, 256, 16, "ones"), (128, 256, 16, "eye"), (128, 256, 16), (128, 256, 64), (256, 512, 128),
                 (300, 520, 200)]:
        run(*args)
