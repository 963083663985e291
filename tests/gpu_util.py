"""Helpers for the -m gpu tests (test infrastructure)."""
import numpy as np

from paper_conf_icppw_matzdf20_b200 import abi


def rel_ok(g, o, rtol):
    """Reading Q18: |g - o| <= rtol * max(|o|, RMS(o)) element-wise."""
    g = np.asarray(g, dtype=np.float64)
    o = np.asarray(o, dtype=np.float64)
    rms = float(np.sqrt(np.mean(o * o))) if o.size else 0.0
    tol = rtol * np.maximum(np.abs(o), rms)
    err = np.abs(g - o)
    return bool(np.all(err <= tol)), float(np.max(err / np.maximum(tol / rtol, 1e-300))) if o.size else 0.0


def fetch(ctx, buf, shape, dtype=np.float32):
    out = np.empty(shape, dtype=dtype)
    abi.pk_sync_to_host(ctx, buf, out)
    return out


def gpu_ctx(P, mode=0):
    ctx = abi.pk_init(P, part_device=[0] * P)
    if mode:
        abi.pk_set_mode(ctx, mode)
    return ctx
