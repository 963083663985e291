#!/usr/bin/env python
"""Benchmark of the partitioned hot path (BASELINE.json metric: GLUP/s and roofline
fraction; stale bytes moved).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload hotspot2d|heat3d|jacobi2d|nbody]
                    [--parts P] [--impl pk|reference]

A "step" is one pass of the whole hot path over one batch: for the default
workload (C2, BASELINE.json configs[1]) that is 100 Hotspot iterations on a
16384 x 16384 fp32 grid, each iteration one pk_launch_partitioned (grid
partition -> regions -> stale plan -> transfers -> partitioned kernels ->
tracker update).  ``value`` is device-timed (CUDA events on the library's
streams via pk_timer_begin/end) with the inputs resident in HBM; ``e2e`` adds
the H2D upload (pk_copy_from_host from pinned memory) and the D2H gather
(pk_sync_to_host) of every step and is wall-clock timed.

Process model: without torchrun one host process drives every
partition, as in the paper: ``--gpus N`` puts one partition on each
of devices 0..N-1.  Under torchrun with N ranks (the driver's multi-GPU launch)
every rank owns ONE partition on its own GPU (SPMD, NEXT-4): the ranks replay the
same deterministic plan and pull their stale ranges from the holders' CUDA-IPC-
mapped instances (``--transport nccl``: NCCL send/recv); the reported time is the
max over ranks.  ``--parts P`` runs P partitions as virtual devices on the visible
GPUs (transfers then are D2D copies).
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

WORKLOADS = {
    # name: (config text, default iterations/steps per bench step)
    "hotspot2d": ("C2 Hotspot-style 2D stencil 16384x16384 fp32 (temp+power), 100 iterations/step", 100),
    "heat3d": ("C3 3D 7-point heat stencil 1024^3 fp32, 50 iterations/step", 50),
    "jacobi2d": ("C1 2D 5-point Jacobi 512x512 fp32, 10 iterations/step", 10),
    "nbody": ("C5 all-pairs N-body 2^20 bodies fp32, 10 steps/step", 10),
    "sgemm": ("C4 dense SGEMM 16384^3 fp32 (3xTF32 on tcgen05), 1 launch/step", 1),
}


def halo_push(halo, n_gpus, workload):
    """--halo: pull (copies on the reader's stream), push (PK_MODE_PUSH: the producing kernel stores
    the halo into the readers' instances) or auto = push when the partitions span several GPUs for
    the stencils (a pull there puts a copy between the producer's kernel and the reader's next one;
    on one GPU a pushed halo takes SM time while a pulled one runs on the copy engines).  The GEMM
    and N-body read whole buffers: streamed operand / all-gather, nothing to push."""
    if halo == "push":
        return True
    if halo == "pull":
        return False
    return n_gpus > 1 and workload in ("hotspot2d", "heat3d", "jacobi2d")


def env_int(name, default):
    try:
        return int(os.environ.get(name, default))
    except ValueError:
        return default


def load_peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return None


def ncu_traffic(kernel):
    """dram__bytes_read.sum + dram__bytes_write.sum per launch from a committed ncu capture."""
    try:
        d = json.load(open(os.path.join(ROOT, "profiles", "ncu_traffic.json")))
        v = d.get(kernel)
        return None if v is None else v.get("dram_bytes_per_launch")
    except Exception:
        return None


class ClockSampler:
    """nvidia-smi clocks/throttle reasons sampled DURING the timed region."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpus):
        self.gpus = set(gpus)
        self.lines = []
        self.proc = None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                                          "-lms", "100"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL,
                                         text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        self.t.join(timeout=2)
        sm, smax, reasons, power = [], [], set(), []
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 9:
                continue
            try:
                idx = int(f[0])
            except ValueError:
                continue
            if idx not in self.gpus:
                continue
            try:
                sm.append(float(f[1]))
                smax.append(float(f[2]))
                power.append(float(f[3]))
            except ValueError:
                pass
            for n, v in zip(names, f[5:9]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(smax) if smax else None,
                "reasons": sorted(reasons), "samples": len(sm),
                "power_w_max": max(power) if power else None}


class NvlinkCounters:
    """NVML NVLink data counters (KiB, cumulative over all links) of the GPUs in use, read
    around the timed region -- the hardware's count of inter-GPU bytes, to set beside the
    library's moved + pushed bytes.  None where NVML or the field is missing."""

    def __init__(self, gpus):
        self.gpus, self.h, self.t0 = list(gpus), None, None
        try:
            import pynvml as nv
            nv.nvmlInit()
            self.nv = nv
            self.h = [nv.nvmlDeviceGetHandleByIndex(g) for g in self.gpus]
        except Exception:
            self.h = None

    def _read(self):
        nv = self.nv
        tot = [0, 0]
        for h in self.h:
            vals = nv.nvmlDeviceGetFieldValues(h, [nv.NVML_FI_DEV_NVLINK_THROUGHPUT_DATA_TX,
                                                   nv.NVML_FI_DEV_NVLINK_THROUGHPUT_DATA_RX])
            for i, v in enumerate(vals):
                if v.nvmlReturn != 0:
                    raise RuntimeError("field unavailable")
                tot[i] += int(v.value.ullVal) * 1024
        return tot

    def start(self):
        try:
            self.t0 = self._read() if self.h else None
        except Exception:
            self.t0 = None

    def stop(self):
        if not self.t0:
            return None
        try:
            t1 = self._read()
        except Exception:
            return None
        return {"tx_bytes": t1[0] - self.t0[0], "rx_bytes": t1[1] - self.t0[1], "gpus": self.gpus,
                "source": "NVML NVML_FI_DEV_NVLINK_THROUGHPUT_DATA_TX/RX over the timed region"}


def nvlink_check(measured, st, P, part_dev, world):
    """Set NVML's NVLink byte counters beside the library's inter-GPU bytes (moved + pushed
    between partitions on different GPUs): on an NVSwitch box the NVML RX bytes must cover them
    (protocol overhead and other traffic only add)."""
    if measured is None:
        return None
    if world > 1:
        # SPMD (rank 0's view): the bytes rank 0 pulled; with one GPU per rank they all crossed NVLink
        lib = st["moved_bytes"] + st["pushed_bytes"]
    else:
        devs = [part_dev[p % len(part_dev)] for p in range(P)] if part_dev else [0] * P
        lib = sum(st["pair_bytes"][q][p] for q in range(min(P, 16)) for p in range(min(P, 16))
                  if devs[q] != devs[p]) + (st["pushed_bytes"] if len(set(devs)) > 1 else 0)
    out = dict(measured)
    out["library_interdevice_bytes"] = int(lib)
    out["rx_covers_library_bytes"] = (measured["rx_bytes"] >= lib) if lib else None
    return out


def measure_tf32_ceiling(device, n=8192, reps=10):
    """Dense TF32 tensor-core ceiling of this GPU in this run: cuBLAS through torch.matmul on
    fp32 inputs with TF32 enabled (SURVEY.md §8(d) "measured ceilings"), CUDA events."""
    try:
        import torch
        with torch.cuda.device(device):
            old = torch.backends.cuda.matmul.allow_tf32
            torch.backends.cuda.matmul.allow_tf32 = True
            a = torch.randn(n, n, device="cuda")
            b = torch.randn(n, n, device="cuda")
            for _ in range(3):
                torch.matmul(a, b)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize()
            e0.record()
            for _ in range(reps):
                torch.matmul(a, b)
            e1.record()
            torch.cuda.synchronize()
            ms = e0.elapsed_time(e1) / reps
            torch.backends.cuda.matmul.allow_tf32 = old
            del a, b
            torch.cuda.empty_cache()
        return {"tflops": 2.0 * n ** 3 / (ms / 1e3) / 1e12, "shape": [n, n, n], "ms": ms,
                "how": "torch.matmul fp32 with allow_tf32 (cuBLAS), mean of %d after 3 warm-up" % reps}
    except Exception as e:  # pragma: no cover
        return None


# ------------------------------------------------------------------ workloads
class Workload:
    """Inputs, setup and per-step loop of one config, driven through the C-ABI."""

    def __init__(self, name, iters):
        self.name, self.iters = name, iters
        import synth
        from paper_conf_icppw_matzdf20_b200 import kernels as K
        self.K = K
        if name == "hotspot2d":
            # PK_BENCH_ROWS (experiments only): fewer rows, e.g. one SPMD rank's share at N = 8
            self.shape = (int(os.environ.get("PK_BENCH_ROWS", 16384)), 16384)
            self.host = synth.hotspot_grids(*self.shape)
            self.units_per_iter = self.shape[0] * self.shape[1]
            self.bytes_per_unit = 12          # temp read + power read + temp write
            self.unit, self.metric = "GLUP/s", "hotspot2d_glups"
        elif name == "heat3d":
            # PK_BENCH_PLANES (experiments only): fewer planes, e.g. one SPMD rank's share at N = 8
            self.shape = (int(os.environ.get("PK_BENCH_PLANES", 1024)), 1024, 1024)
            self.host = (synth.heat_grid(*self.shape),)
            self.units_per_iter = int(np.prod(self.shape))
            self.bytes_per_unit = 8
            self.unit, self.metric = "GLUP/s", "heat3d_glups"
        elif name == "jacobi2d":
            self.shape = (512, 512)
            self.host = (synth.jacobi_grid(*self.shape),)
            self.units_per_iter = (self.shape[0] - 2) * (self.shape[1] - 2)
            self.bytes_per_unit = 8
            self.unit, self.metric = "GLUP/s", "jacobi2d_glups"
        elif name == "nbody":
            n = 1 << 20
            self.shape = (n,)
            self.host = synth.nbody_bodies(n)
            self.units_per_iter = n * n
            self.bytes_per_unit = 0
            self.unit, self.metric = "Ginteractions/s", "nbody_ginteractions"
        elif name == "sgemm":
            m = n = k = 16384
            self.shape = (m, n, k)
            a, b = synth.gemm_operands(m, n, k)
            # Each step is one partitioned GEMM X' = A X whose operand X is the previous step's
            # output: partition p wrote row slab p of it, so every step reads the whole operand
            # from all partitions -- the (P-1)|B| broadcast of BASELINE's C4 config happens
            # inside every timed step.  A is scaled by sqrt(3/K) (entry variance 1/K) so the
            # iterates keep their magnitude (DESIGN.md §3 input recipe).
            a *= np.float32(math.sqrt(3.0 / k))
            self.host = (a, b)
            self.units_per_iter = 2 * m * n * k          # FP32-equivalent flops
            self.bytes_per_unit = 0
            self.scale = 1e12
            self.unit, self.metric = "TFLOP/s", "sgemm_fp32_equiv_tflops"
        else:
            raise SystemExit(f"unknown workload {name}")
        self.scale = getattr(self, "scale", 1e9)
        # kernels launched per partition per pk_launch_partitioned (gpu_launches)
        self.kernels_per_launch = {"nbody": 2}.get(name, 1)

    def block_depth(self):
        """Rows per tile (Hotspot) / planes per block (Heat) when --tile is not given: the
        persistent Hotspot grid and the Heat block grid quantise into waves of resident
        CTAs, which matters once one GPU holds only a slab (SPMD at N = 4, 8).  Measured on
        one B200 with a rank's share of the grid (PK_BENCH_ROWS / PK_BENCH_PLANES):
        Hotspot 2048 rows TY 128 / 96 / 64 = 1274 / 1554 / 1536 GLUP/s, 4096 rows 1712 /
        - / 1729, 16384 rows flat; Heat 128 planes ZC 64 / 24 / 16 = 1121 / 1185 / 1173,
        256 planes 1154 / - / 1260 (ZC 32: 1234), 1024 planes 1268 / 1255 (24) / 1234."""
        tile = getattr(self, "tile", 0)
        if tile:
            return tile
        g = max(1, getattr(self, "gpus_used", 1))
        if self.name == "hotspot2d":
            if getattr(self, "variant", None):
                return self.K.HOTSPOT_TY
            # the partitions of the full grid one process runs: one per rank (SPMD) or all (one process)
            parts = g if g > 1 else 1
            return self.K.hotspot2d_tbk_rows(self.shape[0], self.shape[1], getattr(self, "sweeps_arg", 4), parts,
                                             self.ctas())
        if self.name == "heat3d":
            return min(64, max(16, (self.shape[0] // g) // 16 // 8 * 8))
        return 0

    def ctas(self):
        """Persistent CTAs of hotspot2d_tbk on this GPU: 3 per SM (2 for K > 4)."""
        try:
            import torch
            sms = torch.cuda.get_device_properties(torch.cuda.current_device()).multi_processor_count
        except Exception:
            sms = 148
        return sms * (3 if getattr(self, "sweeps_arg", 4) <= 4 else 2)

    def setup(self, ctx):
        K = self.K
        tile = self.block_depth()
        if self.name == "hotspot2d":
            self.pr = K.hotspot2d_setup(ctx, *self.host, ty=tile or K.HOTSPOT_TY,
                                        kernel=getattr(self, "variant", None) or "hotspot2d_tbk",
                                        tiles=self.tiles, sweeps=getattr(self, "sweeps_arg", 4))
            # sweeps fused per launch: 4 for the default hotspot2d_tbk, 2 for hotspot2d_tb2
            # (one HBM pass = 12 B per cell per launch)
            self.sweeps = self.pr.sweeps
            self.bytes_per_unit = 12 / self.sweeps
            self.upload_bufs = [(self.pr.tb[0], self.host[0]), (self.pr.tb[2], self.host[1])]
        elif self.name == "heat3d":
            self.pr = K.heat3d_setup(ctx, self.host[0], zc=tile or None,
                                     kernel=getattr(self, "variant", None) or "heat3d_tb2", tiles=self.tiles)
            # two sweeps per launch for the default heat3d_tb2: 8 B per cell per launch = 4 B/LU
            self.sweeps = self.pr.sweeps
            self.bytes_per_unit = 8 / self.sweeps
            self.upload_bufs = [(self.pr.ub[0], self.host[0])]
        elif self.name == "sgemm":
            self.pr, _ = K.sgemm_program(ctx, *self.host, launches=0)
            self.upload_bufs = [(self.pr.abc[0], self.host[0]), (self.pr.abc[1], self.host[1])]
            self.gemm_t = 0    # X_t = buffer B (t even) / C (t odd)
            # settle: the two alternating launches are captured into replay graphs here, before
            # the driver's warm-up (one launch per step would otherwise capture one in the timed region)
            for _ in range(4):
                self.step_once()
        elif self.name == "jacobi2d":
            if (getattr(self, "variant", None) or "jacobi2d_tb") == "jacobi2d_tb":
                # default C1 kernel: K sweeps per launch (ghost zones), K = --sweeps or half a
                # step's iterations (two launches per step: an even count replays one graph per
                # step; odd counts alternate two graphs and measured 2x slower, scripts/r02/gpu_70.sh)
                k = getattr(self, "sweeps_jacobi", None) or (self.iters // 2 if self.iters % 2 == 0 and
                                                              self.iters <= 32 else min(self.iters, 16))
                self.pr, _ = K.jacobi2d_program(ctx, self.host[0], 0, tiles=self.tiles, kernel="jacobi2d_tb",
                                                sweeps=k)
                self.sweeps = k
                self.bytes_per_unit = 8 / k
            else:
                self.pr, _ = K.jacobi2d_program(ctx, self.host[0], 0, tiles=self.tiles)
            self.upload_bufs = [(b, self.host[0]) for b in self.pr.bufs]
        elif self.name == "nbody":
            self.pr = K.nbody_setup(ctx, *self.host)
            self.upload_bufs = [(self.pr.nb[0], self.host[0]), (self.pr.nb[2], self.host[1])]
        self.t = 0

    def step(self):
        K, pr = self.K, self.pr
        if self.name == "hotspot2d":
            out = K.hotspot2d_iterate(pr, self.iters, self.t)
        elif self.name == "heat3d":
            out = K.heat3d_iterate(pr, self.iters, self.t)
        elif self.name == "jacobi2d":
            # the step's sweeps as one pk_launch_sequence: one graph launch in steady state
            out = K.jacobi2d_iterate(pr, self.iters, self.t, sequence=True)
        elif self.name == "sgemm":
            for _ in range(self.iters):
                out = self.step_once()
        else:
            out, _ = K.nbody_iterate(pr, self.iters, self.t)
        self.t += self.iters
        return out

    def step_once(self):
        """C4: one launch X_{t+1} = A X_t (ping-pong between the B and C buffers)."""
        pr = self.pr
        grid, blk, sc = pr.geom
        a, b, c = pr.abc
        m, n, k = pr.mnk
        x, y = (b, c) if self.gemm_t % 2 == 0 else (c, b)
        pr.launch(grid, blk, [a, x, y, m, n, k], sc)
        self.gemm_t += 1
        return y

    def out_shape(self):
        if self.name == "sgemm":
            return (self.shape[0], self.shape[1])
        return (self.shape[0], 4) if self.name == "nbody" else self.shape

    def stale_min(self, P):
        from_cf = {
            "hotspot2d": lambda: 2 * self.shape[1] * 4 * (P - 1),
            "heat3d": lambda: 2 * self.shape[1] * self.shape[2] * 4 * (P - 1),
            "jacobi2d": lambda: 2 * (self.shape[1] - 2) * 4 * (P - 1),
            "nbody": lambda: self.shape[0] * 16 * (P - 1),
            "sgemm": lambda: (P - 1) * self.shape[2] * self.shape[1] * 4,   # the whole operand X, every step
        }
        return from_cf[self.name]() * self.iters


def cpu_oracle_rate(w: Workload, budget_s=10.0, max_iters=1000):
    """Time the oracle as it stands on a bounded sample of the same workload."""
    import ctypes
    from oracle import kernels as ok
    L = ok.lib()
    D = ctypes.POINTER(ctypes.c_double)
    t0 = time.perf_counter()
    if w.name in ("hotspot2d", "jacobi2d", "heat3d"):
        if w.name == "hotspot2d":
            rows = min(4096, w.shape[0])
            a = np.ascontiguousarray(w.host[0][:rows], dtype=np.float64)
            p = np.ascontiguousarray(w.host[1][:rows], dtype=np.float64)
            b = np.empty_like(a)
            cells = a.size
            sample = f"{rows}x{w.shape[1]} band of the 16384^2 grid"

            def one(src, dst):
                L.oracle_hotspot2d_sweep(src.ctypes.data_as(D), p.ctypes.data_as(D), dst.ctypes.data_as(D),
                                         ctypes.c_int64(rows), ctypes.c_int64(w.shape[1]),
                                         ctypes.c_double(ok.HOTSPOT_CAP), ctypes.c_double(ok.HOTSPOT_RX1),
                                         ctypes.c_double(ok.HOTSPOT_RY1), ctypes.c_double(ok.HOTSPOT_RZ1),
                                         ctypes.c_double(ok.HOTSPOT_AMB))
        elif w.name == "heat3d":
            planes = min(128, w.shape[0])
            a = np.ascontiguousarray(w.host[0][:planes], dtype=np.float64)
            b = np.empty_like(a)
            cells = a.size
            sample = f"{planes} planes of the 1024^3 grid"

            def one(src, dst):
                L.oracle_heat3d_sweep(src.ctypes.data_as(D), dst.ctypes.data_as(D), ctypes.c_int64(planes),
                                      ctypes.c_int64(w.shape[1]), ctypes.c_int64(w.shape[2]),
                                      ctypes.c_double(ok.HEAT_ALPHA))
        else:
            a = np.ascontiguousarray(w.host[0], dtype=np.float64)
            b = a.copy()
            cells = (w.shape[0] - 2) * (w.shape[1] - 2)
            sample = "full 512^2 grid"

            def one(src, dst):
                L.oracle_jacobi2d_sweep(src.ctypes.data_as(D), dst.ctypes.data_as(D), ctypes.c_int64(w.shape[0]),
                                        ctypes.c_int64(w.shape[1]))
        for fn in ("oracle_hotspot2d_sweep", "oracle_heat3d_sweep", "oracle_jacobi2d_sweep"):
            getattr(L, fn).restype = None
        its, el = 0, 0.0
        ts = time.perf_counter()
        while its < max_iters and el < budget_s:
            if its % 2 == 0:
                one(a, b)
            else:
                one(b, a)
            its += 1
            el = time.perf_counter() - ts
        rate = cells * its / el / 1e9
        sample += f", {its} iterations"
    elif w.name == "sgemm":
        m, n, k = w.shape
        ns = 4096
        rows = (np.arange(ns, dtype=np.int64) * 7919) % m
        cols = (np.arange(ns, dtype=np.int64) * 104729) % n
        ts = time.perf_counter()
        ok.gemm_entries(w.host[0], w.host[1], rows, cols)
        el = time.perf_counter() - ts
        rate = 2.0 * ns * k / el / 1e12
        sample = f"{ns} sampled C entries x K = {k} (fp64 accumulation)"
    else:
        nt = 256
        pos = np.ascontiguousarray(w.host[0], dtype=np.float64)
        tg = np.arange(0, w.shape[0], w.shape[0] // nt, dtype=np.int64)[:nt]
        ts = time.perf_counter()
        ok.nbody_accel(pos, tg)
        el = time.perf_counter() - ts
        rate = nt * w.shape[0] / el / 1e9
        sample = f"{nt} sampled targets x {w.shape[0]} sources, 1 step (fp64)"
    return {"value": rate, "unit": w.unit, "cores": ok.num_threads(), "kind": "oracle", "sample": sample,
            "seconds": round(time.perf_counter() - t0, 2)}


def run_reference(args, w: Workload, rank):
    """--impl reference: the oracle as it stands, on the host cores, same metric."""
    if rank != 0:
        return None
    # torchrun sets OMP_NUM_THREADS=1 per worker; rank 0 runs the oracle alone on the host
    # cores (the other ranks do no work), so give its OpenMP runtime all of them
    if env_int("WORLD_SIZE", 1) > 1:
        n = len(os.sched_getaffinity(0))
        os.environ["OMP_NUM_THREADS"] = str(n)
        from oracle import kernels as ok
        ok.lib().omp_set_num_threads(n)    # the OpenMP runtime may have read the variable already
    # each step is a bounded sample; warmup steps are run untimed
    for _ in range(args.warmup):
        cpu_oracle_rate(w, budget_s=1.0, max_iters=1)
    vals = [cpu_oracle_rate(w, budget_s=5.0, max_iters=4) for _ in range(args.steps)]
    v = statistics.median(x["value"] for x in vals)
    line = {"impl": "reference", "metric": w.metric, "value": v, "unit": w.unit, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "higher_is_better": True, "dtype": "f64",
            "data": "synthetic", "config": {"workload": WORKLOADS[w.name][0]},
            "cpu_baseline": {"value": v, "unit": w.unit, "cores": vals[0]["cores"], "kind": "oracle",
                             "sample": vals[0]["sample"] + " per step"},
            "e2e": {"value": v, "unit": w.unit, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
            "vs_baseline": None}
    return line


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--workload", default="hotspot2d", choices=sorted(WORKLOADS))
    ap.add_argument("--parts", type=int, default=0, help="partitions (default: one per GPU)")
    ap.add_argument("--iters", type=int, default=0, help="iterations per step (default: the config's)")
    ap.add_argument("--impl", default="pk", choices=["pk", "reference"])
    ap.add_argument("--e2e-steps", type=int, default=8)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--variant", default=None, help="kernel variant (hotspot2d_regs: register-window Hotspot)")
    ap.add_argument("--sweeps", type=int, default=None,
                    help="time steps per launch: hotspot2d_tbk 2..8 (default 4; iterations must be a multiple), "
                         "jacobi2d_tb 1..16 (default: a step's iterations)")
    ap.add_argument("--tile", type=int, default=0, help="rows per block (hotspot2d TY) / planes per block (heat3d ZC)")
    ap.add_argument("--tiles", default=None,
                    help="tile partitions TXxTY[xTZ] (NEXT-2) instead of 1-D slabs; product = partitions")
    ap.add_argument("--transport", default="ipc", choices=["ipc", "nccl"],
                    help="SPMD (torchrun, N > 1) cross-rank transport: CUDA IPC peer memory or NCCL send/recv")
    ap.add_argument("--halo", default="auto", choices=["auto", "pull", "push"],
                    help="stencil halo transport: pull = copies on the reader's stream after the producer's kernel; "
                         "push = PK_MODE_PUSH, the producing kernel also stores the halo into the readers' instances "
                         "(peer stores over NVLink, no copy on the critical path); auto = push when the partitions "
                         "span several GPUs, else pull (on one GPU a pushed halo costs SM time, a pulled one runs on "
                         "the copy engines: profiles/r02/push_vs_pull.txt)")
    ap.add_argument("--push", action="store_true", help="same as --halo push")
    ap.add_argument("--abg", action="store_true",
                    help="also run the paper's alpha/beta/gamma overhead decomposition (P:L1164-1181)")
    ap.add_argument("--abg-repeats", type=int, default=3)
    ap.add_argument("--no-e3", action="store_true", help="skip the P = 1 library vs direct-launch comparison")
    ap.add_argument("--no-overlap", action="store_true",
                    help="PK_MODE_NO_OVERLAP: copy streamed operands (GEMM B) before the kernel instead of under it")
    args = ap.parse_args()
    if args.warmup < 3 and args.impl == "pk":
        print("warning: fewer than 3 warm-up steps", file=sys.stderr)

    rank, world = env_int("RANK", 0), env_int("WORLD_SIZE", 1)
    dist = None
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("gloo")
    w = Workload(args.workload, args.iters or WORKLOADS[args.workload][1])
    w.variant = args.variant
    w.sweeps_arg = args.sweeps or 4
    w.sweeps_jacobi = args.sweeps
    w.tile = args.tile
    w.tiles = None
    if args.tiles:
        t = [int(x) for x in args.tiles.lower().split("x")]
        w.tiles = tuple(t + [1] * (3 - len(t)))

    if args.impl == "reference":
        line = run_reference(args, w, rank)
        if dist:
            dist.barrier()
        if rank == 0:
            print(json.dumps(line), flush=True)
        return

    import torch
    from paper_conf_icppw_matzdf20_b200 import abi

    ngpu = max(1, args.gpus)
    result = {}
    if world > 1:
        # SPMD: one process per GPU, one partition per rank.  Default
        # transport: peer memory (CUDA IPC instances + device epoch flags, each rank pulls
        # its stale ranges over NVLink); --transport nccl: NCCL send/recv pairs.
        P = world
        local_rank = env_int("LOCAL_RANK", rank)
        ndev = torch.cuda.device_count()
        dev = local_rank % max(1, ndev)          # ranks share a GPU only on boxes with fewer GPUs
        torch.cuda.set_device(dev)
        if args.transport == "nccl":
            nid = [abi.pk_nccl_unique_id() if rank == 0 else None]
            dist.broadcast_object_list(nid, src=0)
            ctx = abi.pk_init_spmd(P, rank, world, list(range(world)), part_device=[dev] * P, nccl_id=nid[0])
            process_model = "SPMD: one process per GPU, replicated tracker, NCCL send/recv for cross-rank copies"
        else:
            from paper_conf_icppw_matzdf20_b200 import spmd
            ctx = abi.pk_init_spmd_ipc(P, rank, world, list(range(world)), spmd.dist_allgather(),
                                       part_device=[dev] * P)
            process_model = ("SPMD: one process per GPU, replicated tracker, pull copies from CUDA-IPC-mapped "
                             "peer instances ordered by device epoch flags")
        devices = list(range(min(ngpu, max(1, ndev))))
    else:
        P = args.parts or ngpu
        ndev = torch.cuda.device_count()
        if ndev < ngpu:
            raise SystemExit(f"--gpus {ngpu} but only {ndev} visible")
        ctx = abi.pk_init(P, part_device=[p % ngpu for p in range(P)])
        devices = sorted(set(p % ngpu for p in range(P)))
        process_model = "one host process drives all partitions"
    if args.push:
        args.halo = "push"
    args.push = halo_push(args.halo, world if world > 1 else len(devices), w.name)
    base_mode = (abi.PK_MODE_PUSH if args.push else 0) | (abi.PK_MODE_NO_OVERLAP if args.no_overlap else 0)
    abi.pk_set_mode(ctx, base_mode)
    w.gpus_used = world if world > 1 else len(devices)
    devices_used = list(range(min(world, torch.cuda.device_count()))) if world > 1 else devices
    w.setup(ctx)
    for _ in range(args.warmup):
        w.step()
    abi.pk_synchronize(ctx)
    abi.pk_reset_stats(ctx)
    if dist:
        dist.barrier()
    sampler = ClockSampler(range(min(ngpu, torch.cuda.device_count()))) if rank == 0 else None
    if sampler:
        sampler.start()
        time.sleep(0.3)
    # (1) the timed region, in the production mode (steady-state graph replay on for
    # single-process contexts).  Launches of 100 us and more (every config but the
    # latency-bound C1) are timed live in it: PK_MODE_TIME_KERNELS records CUDA events
    # around every replayed launch on the stream it runs on (around every partition kernel
    # when a launch runs eagerly: SPMD ranks).  C1 (microsecond launches) takes its events
    # from a second pass of the same steps.
    nvl = NvlinkCounters(devices_used if world == 1 else [env_int("LOCAL_RANK", rank) % max(1, torch.cuda.device_count())])
    live = w.name != "jacobi2d"
    if live:
        abi.pk_set_mode(ctx, base_mode | abi.PK_MODE_TIME_KERNELS)
    abi.pk_synchronize(ctx)
    nvl.start()
    abi.pk_timer_begin(ctx)
    for _ in range(args.steps):
        w.step()
    elapsed_ms = abi.pk_timer_end(ctx)
    nvlink_measured = nvl.stop()
    st = abi.pk_get_stats(ctx)
    if live:
        stk = st
        abi.pk_set_mode(ctx, base_mode)
    else:
        # (2) CUDA events for the roofline from a second pass of the same steps
        abi.pk_reset_stats(ctx)
        abi.pk_set_mode(ctx, base_mode | abi.PK_MODE_TIME_KERNELS)
        for _ in range(max(1, min(args.steps, 3))):
            w.step()
        abi.pk_synchronize(ctx)
        stk = abi.pk_get_stats(ctx)
        abi.pk_set_mode(ctx, base_mode)
    clocks = sampler.stop() if sampler else {}
    for key_ in ("kernel_ms", "timed_kernels", "kernel_ms_max_launch", "graph_launch_ms", "timed_graph_launches",
                 "timed_eager_launches", "launches"):
        st["t_" + key_] = stk[key_]
    # (3) host overhead without launch-queue back-pressure: one step issued into idle
    # streams (the timed region's launches queue up behind running kernels, and a full
    # queue blocks the issuing thread inside the CUDA calls)
    abi.pk_synchronize(ctx)
    abi.pk_reset_stats(ctx)
    w.step()
    sh = abi.pk_get_stats(ctx)
    abi.pk_synchronize(ctx)
    st_local = dict(st)        # this rank's own counters (its GPU's NVLink bytes are what NVML sees here)
    if dist:
        tt = torch.tensor([elapsed_ms, st["kernel_launches"], st["moved_bytes"], st["copies"], st["pushed_bytes"]],
                          dtype=torch.float64)
        mx = tt.clone()
        dist.all_reduce(mx, op=dist.ReduceOp.MAX)
        dist.all_reduce(tt, op=dist.ReduceOp.SUM)
        elapsed_ms = float(mx[0])                 # max over ranks
        st["kernel_launches"], st["moved_bytes"], st["copies"] = int(tt[1]), int(tt[2]), int(tt[3])
        st["pushed_bytes"] = int(tt[4])

    units = w.units_per_iter * w.iters * args.steps
    value = units / (elapsed_ms / 1e3) / w.scale
    peaks = load_peaks()
    kname = getattr(w, "variant", None) or {"hotspot2d": "hotspot2d_tbk", "heat3d": "heat3d_tb2",
                                            "jacobi2d": "jacobi2d_tb"}.get(w.name, w.name)
    # duration of one timed launch: a replayed graph (single process: every partition's
    # copies + kernels of the launch) or, launched eagerly, the slowest partition kernel
    # (a launch captured into a graph inside the timed region carries no events: not counted)
    n_timed = st["t_timed_graph_launches"] + st["t_timed_eager_launches"]
    avg_kernel_ms = (st["t_graph_launch_ms"] + st["t_kernel_ms_max_launch"]) / max(1, n_timed)
    # units of one timed launch: all partitions of this process (one per SPMD rank)
    per_launch_units = w.units_per_iter * getattr(w, "sweeps", 1) / (P if world > 1 else 1)
    if w.name == "sgemm":
        # tensor bound: 3 TF32 MMAs per FP32-equivalent product, against the TF32 ceiling measured
        # in this run (cuBLAS via torch.matmul, allow_tf32, 8192^3); the bf16-derived figure beside it
        tf32 = measure_tf32_ceiling(devices[0] if world == 1 else torch.cuda.current_device())
        bf16 = (peaks or {}).get("bf16_tflops", 1668.4)
        derived = bf16 * 1.1 / 2.25
        # the denominator is the HIGHER of the two: cuBLAS' TF32 GEMM measured in this run (it
        # measured 723 TF/s at 8192^3, i.e. below what the 3xTF32 kernel sustains, so it is not a
        # ceiling on its own) and measured bf16 x the nominal TF32/BF16 ratio
        peak = max(tf32["tflops"] if tf32 else 0.0, derived)
        achieved = 3 * per_launch_units / (avg_kernel_ms / 1e3) / 1e12
        roofline = {"bound": "tensor", "achieved": achieved, "peak": peak, "unit": "TFLOP/s",
                    "frac": achieved / peak, "traffic": ncu_traffic(kname),
                    "peak_bf16_derived": derived, "frac_of_bf16_derived": achieved / derived,
                    "tf32_ceiling": tf32,
                    "frac_of_cublas_tf32": (achieved / tf32["tflops"]) if tf32 else None,
                    "peak_source": "max(TF32 GEMM of cuBLAS measured in this run: torch.matmul fp32 with allow_tf32, "
                                   "8192^3, CUDA events; MEASURED_PEAKS.json bf16_tflops x 1.1/2.25, the nominal "
                                   "TF32/BF16 ratio); achieved = 3 x 2MNK TF32 flops / launch time"}
    elif w.name == "nbody":
        # FP32-ALU bound: 12 FP32-pipe instructions per interaction on 128 lanes/SM
        sm_mhz = clocks.get("sm_mhz") or (peaks or {}).get("sm_max_mhz", 1965.0)
        peak = 148 * 128 / 12 * (sm_mhz * 1e6) / 1e9
        achieved = per_launch_units / (avg_kernel_ms / 1e3) / 1e9
        roofline = {"bound": "alu", "achieved": achieved, "peak": peak, "unit": "Ginteractions/s",
                    "frac": achieved / peak, "traffic": None,
                    "peak_source": f"148 SMs x 128 FP32 lanes / 12 ops per interaction at {sm_mhz:.0f} MHz"}
    else:
        bytes_per_launch = w.bytes_per_unit * per_launch_units
        achieved = bytes_per_launch / (avg_kernel_ms / 1e3) / 1e9
        peak = (peaks or {}).get("hbm_gbs", 6650.0)
        roofline = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                    "frac": achieved / peak, "traffic": ncu_traffic(kname),
                    "peak_source": "MEASURED_PEAKS.json hbm_gbs (measured)" if peaks else "fallback 6.65 TB/s"}
    result.update({
        "metric": w.metric, "value": value, "unit": w.unit, "n_gpus": ngpu, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": elapsed_ms / args.steps, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
        "config": {"workload": WORKLOADS[w.name][0], "iterations_per_step": w.iters, "partitions": P,
                   "partition_devices": devices,
                   "l2": "inputs larger than the 126 MB L2 (no flush)" if w.name != "jacobi2d"
                   else "1 MB working set stays in L2 (latency-bound C1)",
                   "process_model": process_model,
                   "halo_push": bool(args.push),
                   "overlap": not args.no_overlap,
                   "kernel": getattr(w, "variant", None) or {"hotspot2d": "hotspot2d_tbk", "heat3d": "heat3d_tb2",
                                                             "jacobi2d": "jacobi2d_tb"}.get(w.name, w.name),
                   "sweeps_per_launch": getattr(w, "sweeps", 1),
                   **({"rows_per_tile": w.block_depth()} if w.name == "hotspot2d" and not w.variant else {}),
                   **({"planes_per_block": w.block_depth()} if w.name == "heat3d" and not w.variant else {}),
                   "partition_shape": list(w.tiles) if w.tiles else "1-D slabs of the slowest grid dim"},
        "gpu_launches": int(st["kernel_launches"] * w.kernels_per_launch + st["copy_kernels"]),
        "graph_replays": int(st.get("graph_replays", 0)),
        "clocks": clocks,
        "roofline": roofline,
        "kernel_ms_avg": avg_kernel_ms,
        "kernel_timing": (("CUDA events on the launching stream inside the timed region, production mode: "
                           "around each replayed graph launch (%d launches)%s" %
                           (st["t_timed_graph_launches"],
                            "" if st["t_timed_graph_launches"] == n_timed else
                            ", around every partition kernel of the %d eager launches" % (n_timed - st["t_timed_graph_launches"]))
                           + ("" if n_timed == st["t_launches"] else
                              "; %d launch(es) captured in the region untimed" % (st["t_launches"] - n_timed)))
                          if live else "CUDA events on the launching stream, second pass of the same steps right "
                          "after the timed region (C1: microsecond launches)"),
        "transfers": {"stale_bytes": int(st["stale_bytes"]), "moved_bytes": int(st["moved_bytes"]),
                      "analytic_min_bytes": w.stale_min(P) * args.steps if not w.tiles else None,
                      "copies": int(st["copies"]), "strided_copies": int(st["strided_copies"]),
                      "pushed_bytes": int(st["pushed_bytes"]),
                      "streamed_bytes": int(st["streamed_bytes"]),
                      "halo_copy_kernels": int(st["copy_kernels"])},
        # inter-GPU bytes (NVLink/NVSwitch when the partitions sit on different GPUs): received
        # per GPU per step, and that rate averaged over the whole step against 900 GB/s per
        # direction -- a lower bound of the transfer-phase fraction (copies overlap kernels)
        "nvlink": ({"bytes_per_gpu_per_step": (st["moved_bytes"] + st["pushed_bytes"]) / len(devices_used)
                    / args.steps,
                    "step_avg_frac_of_900GBs": (st["moved_bytes"] + st["pushed_bytes"]) / len(devices_used)
                    / (elapsed_ms / 1e3) / 900e9,
                    "note": "moved + pushed bytes between partitions on different GPUs; averaged over the step"}
                   if len(devices_used) > 1 else None),
        # host time inside pk_launch_partitioned, from one step issued into idle streams (no
        # launch-queue back-pressure); thread CPU time beside the wall time
        "host_us_per_launch": (sh["host_ns_partition"] + sh["host_ns_regions"] + sh["host_ns_plan"]
                               + sh["host_ns_issue"] + sh["host_ns_update"]) / 1e3 / max(1, sh["launches"]),
        "host_cpu_us_per_launch": sh["host_cpu_ns"] / 1e3 / max(1, sh["launches"]),
        "host_us_per_launch_phases": {k: sh["host_ns_" + k] / 1e3 / max(1, sh["launches"])
                                      for k in ("partition", "regions", "plan", "issue", "update")},
        "host_us_per_launch_timed_region": {
            "wall": (st["host_ns_partition"] + st["host_ns_regions"] + st["host_ns_plan"] + st["host_ns_issue"]
                     + st["host_ns_update"]) / 1e3 / max(1, st["launches"]),
            "thread_cpu": st["host_cpu_ns"] / 1e3 / max(1, st["launches"]),
            "note": "includes time blocked in CUDA calls once the launch queue is full (launches are issued "
                    "far ahead of the GPU)"},
        "nvlink_nvml": nvlink_check(nvlink_measured, st_local, P, devices if world == 1 else None, world),
        "us_per_launch": elapsed_ms * 1e3 * getattr(w, "sweeps", 1) / max(1, w.iters * args.steps),
    })

    # ---- alpha / beta / gamma (§9.2) ----
    if args.abg:
        # R repeats per mode, interleaved (alpha, beta, gamma, alpha, ...) so that clock drift
        # hits all three alike; each repeat = args.steps steps, device-timed (pk_timer), max over ranks
        reps = {"alpha": [], "beta": [], "gamma": []}
        modes = (("alpha", 0), ("beta", abi.PK_MODE_NO_TRANSFERS), ("gamma", abi.PK_MODE_NO_TRACKING))
        for r in range(args.abg_repeats):
            for name, mode in modes:
                abi.pk_set_mode(ctx, mode | (base_mode if mode == 0 else 0))
                w.step()                                   # settle the mode (tracker state, caches, graphs)
                abi.pk_synchronize(ctx)
                if dist:
                    dist.barrier()
                abi.pk_timer_begin(ctx)
                for _ in range(args.steps):
                    w.step()
                el = abi.pk_timer_end(ctx) / 1e3
                if dist:
                    te = torch.tensor([el], dtype=torch.float64)
                    dist.all_reduce(te, op=dist.ReduceOp.MAX)
                    el = float(te[0])
                reps[name].append(el)
        abi.pk_set_mode(ctx, base_mode)
        med = {k: statistics.median(v) for k, v in reps.items()}
        a, b, g = med["alpha"], med["beta"], med["gamma"]
        # per-repeat fractions (same repeat index) give the spread of each share
        fr = {"T_application": [rg / ra for ra, rg in zip(reps["alpha"], reps["gamma"])],
              "T_transfers": [(ra - rb) / ra for ra, rb in zip(reps["alpha"], reps["beta"])],
              "T_patterns": [(rb - rg) / ra for ra, rb, rg in zip(reps["alpha"], reps["beta"], reps["gamma"])]}
        result["overhead"] = {"alpha_s": a, "beta_s": b, "gamma_s": g, "T_application": g / a,
                              "T_transfers": (a - b) / a, "T_patterns": (b - g) / a,
                              "repeats": args.abg_repeats, "seconds": reps,
                              "spread": {k: [min(v), max(v)] for k, v in fr.items()},
                              "note": "device time (pk_timer) of the same steps, median over interleaved repeats, "
                                      "[min, max] of the per-repeat shares; beta = no transfers (results wrong by "
                                      "design), gamma = no dependency resolution / tracking (P:L1164-1181)"}

    # ---- E3: P = 1 through the library vs the original single-GPU launches ----
    if P == 1 and world == 1 and not args.no_e3:
        lib_ms, dir_ms = [], []
        per_step = elapsed_ms / args.steps
        n3 = max(1, min(args.steps, int(2000 / max(per_step, 1e-3))))     # ~2 s per pass
        for r in range(2):
            for direct in (False, True):
                w.pr.direct = direct
                if per_step < 500:
                    w.step()                                   # settle (graphs of the library path)
                abi.pk_synchronize(ctx)
                abi.pk_timer_begin(ctx)
                for _ in range(n3):
                    w.step()
                (dir_ms if direct else lib_ms).append(abi.pk_timer_end(ctx))
        w.pr.direct = False
        lm, dm = statistics.median(lib_ms), statistics.median(dir_ms)
        result["e3_single_gpu_slowdown"] = {
            "library_ms_per_step": lm / n3, "direct_ms_per_step": dm / n3, "steps_per_pass": n3,
            "slowdown_pct": 100.0 * (lm / dm - 1.0),
            "note": "device time of the same steps: pk_launch_partitioned at P = 1 (graph replay, production mode) vs "
                    "pk_launch_direct (the kernel's full grid, no partitioning / tracking); median of 2 interleaved "
                    "repeats; the paper reports a median 2.1 % slowdown (P:L1156-1161)"}

    # ---- e2e: same metric with the H2D upload and D2H gather inside every step ----
    if not args.no_e2e:
        pinned_of = {}
        def pinned(host):
            if id(host) not in pinned_of:
                pinned_of[id(host)] = torch.from_numpy(host).pin_memory()
            return pinned_of[id(host)]
        # Single process: two contexts (two device copies of the problem) and the asynchronous
        # host copies, so that step i+1's H2D overlaps step i's kernels and D2H (the host link is
        # full duplex); every step still uploads its inputs and reads its result back.
        # SPMD ranks, or too little free HBM for a second copy: one context, blocking copies.
        free_b, total_b = torch.cuda.mem_get_info(devices[0])
        # Contexts in flight: a step's chain (H2D -> kernels -> D2H) must be covered by the others'
        # copies.  Measured (e2e GLUP/s or TF/s, 2 vs 3 contexts): C3 (4 GiB each way) 482 vs 538,
        # C2 598 vs 596, C4 170 vs 81 (three concurrent persistent GEMMs contend) -> 3 for C3 only.
        used_b = total_b - free_b
        want = 3 if w.name == "heat3d" else 2
        n_ctx = 1 if dist is not None or os.environ.get("PK_E2E_BLOCKING") else \
            min(want, 3 if free_b > 2.2 * used_b + (8 << 30) else 2 if free_b > 1.2 * used_b + (8 << 30) else 1)
        n_ctx = min(n_ctx, int(os.environ.get("PK_E2E_CONTEXTS", n_ctx)))
        pipelined = n_ctx > 1
        ctxs, ws = [ctx], [w]
        import copy
        for _ in range(n_ctx - 1):
            c2 = abi.pk_init(P, part_device=[p % ngpu for p in range(P)])
            abi.pk_set_mode(c2, base_mode)
            w2 = copy.copy(w)
            w2.setup(c2)
            ctxs.append(c2)
            ws.append(w2)
        outs = [torch.empty(w.out_shape(), dtype=torch.float32).pin_memory() for _ in ctxs]
        for ws_ in ws:                       # pin (once) before the timed region
            for _, host in ws_.upload_bufs:
                pinned(host)
        for c in ctxs:
            abi.pk_synchronize(c)
        if dist:
            dist.barrier()
        t0 = time.perf_counter()
        h2d = d2h = 0
        for s in range(args.e2e_steps):
            c, ws_, out_host = ctxs[s % len(ctxs)], ws[s % len(ctxs)], outs[s % len(ctxs)]
            for b, host in ws_.upload_bufs:
                hbuf = pinned(host)
                (abi.pk_copy_from_host_async if pipelined else abi.pk_copy_from_host)(c, b, hbuf)
                h2d += hbuf.numel() * hbuf.element_size()
            ws_.t = 0
            if hasattr(ws_.pr, "cur"):
                ws_.pr.cur = 0               # heat3d_tb3 keeps its ping-pong state per launch
            ws_.gemm_t = 0                   # e2e C4: C = A B from the uploaded operands every step
            out = ws_.step()
            (abi.pk_sync_to_host_async if pipelined else abi.pk_sync_to_host)(c, out, out_host)
            d2h += out_host.numel() * out_host.element_size()
            if os.environ.get("PK_E2E_TRACE"):
                print(f"e2e step {s}: enqueued at {time.perf_counter() - t0:.4f} s", file=sys.stderr, flush=True)
        for c in ctxs:
            abi.pk_synchronize(c)
        el = time.perf_counter() - t0
        if dist:
            te = torch.tensor([el], dtype=torch.float64)
            dist.all_reduce(te, op=dist.ReduceOp.MAX)
            el = float(te[0])
        result["e2e"] = {"value": w.units_per_iter * w.iters * args.e2e_steps / el / w.scale, "unit": w.unit,
                         "h2d_bytes_per_step": h2d // args.e2e_steps, "d2h_bytes_per_step": d2h // args.e2e_steps,
                         "steps": args.e2e_steps,
                         "timing": ("wall clock over all steps: per step pk_copy_from_host_async of the inputs + "
                                    "launches + pk_sync_to_host_async of the result, steps rotating over %d contexts (H2D "
                                    "of one overlaps kernels + D2H of the others), pinned host buffers, all contexts "
                                    "synchronised at the end" % len(ctxs) if pipelined else
                                    "wall clock around pk_copy_from_host + launches + pk_sync_to_host per step "
                                    "(pinned host buffers)")}
        for c in ctxs[1:]:
            abi.pk_finalize(c)
    abi.pk_finalize(ctx)
    if not args.no_cpu_baseline and ngpu == 1:
        result["cpu_baseline"] = cpu_oracle_rate(w)
    if dist:
        dist.barrier()
    if rank == 0:
        print(json.dumps(result), flush=True)


if __name__ == "__main__":
    main()
