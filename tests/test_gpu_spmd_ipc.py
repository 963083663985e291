"""Multi-process SPMD over peer memory (pk_init_spmd_ipc) on the GPU.

One process per partition (torch.distributed.run, gloo for the host all-gather),
all on cuda:0: every rank maps the other ranks' instances and epoch flags through
CUDA IPC, pulls its stale ranges straight out of them and orders itself against the
others with device-side flag waits (no NCCL, no host barrier inside a launch).
The worker (tests/spmd_ipc_worker.py) checks each case on rank 0: gathered result
bit-identical to the 1-way result, oracle tolerance, stale == moved bytes, C1's
40,800 bytes at P = 2.
"""
import json
import os
import socket
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


@pytest.mark.gpu
@pytest.mark.parametrize("world,flags_on_sm", [(2, False), (3, False), (2, True)])
def test_spmd_ipc_processes_match_one_way(world, flags_on_sm, tmp_path):
    """flags_on_sm: epoch flags by the SM spin/store kernels instead of stream memory operations."""
    out = tmp_path / "report.json"
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={world}",
           "--master-addr=127.0.0.1", f"--master-port={_free_port()}",
           os.path.join(ROOT, "tests", "spmd_ipc_worker.py"), str(out)]
    env = dict(os.environ, OMP_NUM_THREADS="1")
    env.pop("PK_FLAGS_SM", None)
    if flags_on_sm:
        env["PK_FLAGS_SM"] = "1"
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=600, env=env, cwd=ROOT)
    assert r.returncode == 0, (r.stdout[-4000:], r.stderr[-4000:])
    rep = json.loads(out.read_text())
    assert rep["world"] == world
    names = set(rep["cases"])
    assert {"hotspot2d/mode0", "hotspot2d_tb2/mode0", "hotspot2d_tbk/mode0", "hotspot2d/oracle", "jacobi2d/C1", "heat3d", "nbody",
            "sgemm", "lifecycle", "random/0/mode0", "random/1/mode64"} <= names
    assert all(c["ok"] for c in rep["cases"].values()), rep
    if world == 2:
        assert rep["cases"]["jacobi2d/C1"]["stale"] == 40800
