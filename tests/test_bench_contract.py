"""bench.py on a CPU host: the reference arm's JSON line (the oracle timed on the host
cores) and the launch-configuration choice for the slab one GPU holds."""
import importlib.util
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _bench_module():
    spec = importlib.util.spec_from_file_location("bench", os.path.join(ROOT, "bench.py"))
    m = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(m)
    return m


def test_reference_arm_json_line():
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--workload", "jacobi2d",
                        "--steps", "1", "--warmup", "1"], capture_output=True, text=True, timeout=300, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    line = json.loads(r.stdout.strip().splitlines()[-1])
    assert line["impl"] == "reference" and line["metric"] == "jacobi2d_glups" and line["unit"] == "GLUP/s"
    assert line["value"] > 0 and line["higher_is_better"] is True
    cb = line["cpu_baseline"]
    assert cb["kind"] == "oracle" and cb["cores"] >= 1 and cb["value"] == line["value"] and cb["sample"]
    assert line["e2e"] == {"value": line["value"], "unit": "GLUP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}


def test_block_depth_follows_the_slab_per_gpu():
    b = _bench_module()
    from paper_conf_icppw_matzdf20_b200 import kernels as K
    w = b.Workload.__new__(b.Workload)
    w.name, w.shape, w.K, w.tile = "heat3d", (1024, 1024, 1024), K, 0
    for g, depth in {1: 64, 2: 32, 4: 16, 8: 16}.items():
        w.gpus_used = g
        assert w.block_depth() == depth, g
        assert (1024 // depth) % g == 0       # the slab of each GPU is a whole number of blocks
    w.tile = 40
    assert w.block_depth() == 40              # --tile wins
    # Hotspot: rows per tile from the persistent grid's rounds (444 CTAs)
    assert K.hotspot2d_tbk_rows(16384, 16384) == 131       # 126 x 35 tiles: 10 rounds (128 rows: 11)
    assert K.hotspot2d_tbk_rows(16384, 16384, parts=8) == 54   # a rank's 38 x 35 tiles: 3 rounds
    for h, parts in ((16384, 1), (16384, 2), (16384, 4), (16384, 8), (2048, 1), (300, 1)):
        ty = K.hotspot2d_tbk_rows(h, 16384, parts=parts)
        ncb = -(-16384 // K.tbk_cols(4))
        cost = lambda t: -(-(-(-(-(-h // t)) // parts)) * ncb // 444) * (t + 16)
        rounds = lambda t: -(-(-(-(-(-h // t)) // parts)) * ncb // 444)
        ok_t = [t for t in range(48, 137) if rounds(t) >= 3] or [48]
        assert 48 <= ty <= 136 and all(cost(ty) <= cost(t) for t in ok_t)


def test_reference_arm_under_torchrun_uses_all_host_cores():
    """torchrun sets OMP_NUM_THREADS=1 per worker; rank 0 alone runs the oracle on all cores."""
    r = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
                        "--master-addr", "127.0.0.1", "--master-port", "29647", os.path.join(ROOT, "bench.py"),
                        "--gpus", "2", "--impl", "reference", "--workload", "jacobi2d", "--steps", "1",
                        "--warmup", "1"], capture_output=True, text=True, timeout=300, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.strip().splitlines() if l.startswith("{")]
    assert len(lines) == 1                     # rank 0 prints the one line
    line = json.loads(lines[0])
    assert line["n_gpus"] == 2 and line["cpu_baseline"]["cores"] == len(os.sched_getaffinity(0))


def test_halo_transport_choice():
    b = _bench_module()
    assert b.halo_push("auto", 1, "hotspot2d") is False          # one GPU: pull (copy engines)
    assert b.halo_push("auto", 8, "hotspot2d") is True           # across GPUs: fused push
    assert b.halo_push("auto", 2, "heat3d") and b.halo_push("auto", 2, "jacobi2d")
    assert not b.halo_push("auto", 8, "sgemm") and not b.halo_push("auto", 8, "nbody")
    assert b.halo_push("push", 1, "hotspot2d") and not b.halo_push("pull", 8, "hotspot2d")
