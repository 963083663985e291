"""Build the in-tree C-ABI library ``libpk.so`` for sm_100a (nvcc + g++).

    python -m paper_conf_icppw_matzdf20_b200.build [--force] [--verbose]

Sources: csrc/core/*.cpp (pure host C++), csrc/runtime/*.cu, csrc/kernels/*.cu.
Compiled with ``-gencode arch=compute_100a,code=sm_100a -lineinfo -O3``; the
CUDA runtime is linked statically so the library only needs the driver.
"""
from __future__ import annotations

import concurrent.futures as cf
import glob
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INCLUDE = os.path.join(ROOT, "include")
LIB = os.path.join(PKG, "libpk.so")
OBJ = os.path.join(PKG, "build")
# access-recording variant (kernels/trace.cuh): same sources, -DPK_TRACE_ACCESS, relocatable
# device code so that every kernel file shares the one device-side trace table
TRACE_LIB = os.path.join(PKG, "libpk_trace.so")
TRACE_OBJ = os.path.join(PKG, "build_trace")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def sources():
    return (sorted(glob.glob(os.path.join(CSRC, "core", "*.cpp")))
            + sorted(glob.glob(os.path.join(CSRC, "runtime", "*.cu")))
            + sorted(glob.glob(os.path.join(CSRC, "kernels", "*.cu"))))


def headers():
    return (glob.glob(os.path.join(CSRC, "**", "*.h"), recursive=True)
            + glob.glob(os.path.join(CSRC, "**", "*.cuh"), recursive=True)
            + glob.glob(os.path.join(INCLUDE, "*.h")))


def _obj(src, trace=False):
    rel = os.path.relpath(src, CSRC).replace(os.sep, "_")
    return os.path.join(TRACE_OBJ if trace else OBJ, rel + ".o")


def _compile(src, verbose, trace=False):
    out = _obj(src, trace)
    inc = ["-I", INCLUDE, "-I", CSRC]
    if src.endswith(".cpp"):
        cmd = ["g++", "-std=c++17", "-O2", "-fPIC", "-Wall", "-c", src, "-o", out] + inc
    else:
        cmd = [NVCC, "-std=c++17", "-O3", "-lineinfo", *ARCH, "-Xcompiler", "-fPIC",
               "--expt-relaxed-constexpr", "-c", src, "-o", out] + inc + os.environ.get("PK_NVCC_FLAGS", "").split()
        if trace:
            cmd += ["-DPK_TRACE_ACCESS", "-rdc=true"]
        if verbose:
            cmd += ["-Xptxas", "-v"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"compile failed: {' '.join(cmd)}\n{r.stdout}\n{r.stderr}")
    return out, r.stderr


def build(force: bool = False, verbose: bool = False, trace: bool = False) -> str:
    lib, obj = (TRACE_LIB, TRACE_OBJ) if trace else (LIB, OBJ)
    srcs = sources()
    newest = max(os.path.getmtime(p) for p in srcs + headers() + [__file__])
    if not force and os.path.exists(lib) and os.path.getmtime(lib) >= newest:
        return lib
    os.makedirs(obj, exist_ok=True)
    with cf.ThreadPoolExecutor(max_workers=min(8, len(srcs))) as ex:
        results = list(ex.map(lambda s: _compile(s, verbose, trace), srcs))
    if verbose:
        for _, log in results:
            if log.strip():
                print(log, file=sys.stderr)
    objs = [o for o, _ in results]
    tmp = lib + ".tmp"
    rdc = ["-rdc=true"] if trace else []
    cmd = [NVCC, *ARCH, *rdc, "-shared", "-o", tmp, *objs, "-lcuda"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        # the driver library may be absent at link time on a CPU-only host: use the stub
        cmd = [NVCC, *ARCH, *rdc, "-shared", "-o", tmp, *objs, "-L/usr/local/cuda/lib64/stubs", "-lcuda"]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"link failed: {' '.join(cmd)}\n{r.stdout}\n{r.stderr}")
    os.replace(tmp, lib)
    return lib


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="--verbose" in sys.argv, trace="--trace" in sys.argv))
