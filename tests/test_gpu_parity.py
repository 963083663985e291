"""GPU parity: the CUDA path (through the C-ABI) vs the oracle, and P-way vs 1-way.

Bars (BASELINE.json north_star):
  - partitioned results bit-identical to the 1-partition GPU result;
  - fp32 kernels within 1e-5 relative of the fp64 oracle (reading Q18 metric);
  - stale/moved bytes equal to the closed-form minimum; moved == stale;
  - PK_MODE_NO_TRANSFERS (beta) must change the result (negative control).
P > 1 runs as virtual partitions on cuda:0 (one full-size instance each).
"""
import numpy as np
import pytest

import synth
from oracle import closed_forms as cf
from oracle import kernels as ok
from paper_conf_icppw_matzdf20_b200 import abi
from paper_conf_icppw_matzdf20_b200 import kernels as K
from gpu_util import fetch, gpu_ctx, rel_ok

pytestmark = pytest.mark.gpu


# ------------------------------------------------------------------ C1 Jacobi
def _jacobi(u, iters, P, mode=0, block=K.JACOBI_BLOCK):
    ctx = gpu_ctx(P, mode)
    pr, out = K.jacobi2d_program(ctx, u, iters, block)
    res = fetch(ctx, out, u.shape)
    st = abi.pk_get_stats(ctx)
    abi.pk_finalize(ctx)
    return res, st


def test_c1_jacobi_512_p2_oracle_stale_and_bitwise():
    u = synth.jacobi_grid(512, 512)
    g1, s1 = _jacobi(u, 10, 1)
    g2, s2 = _jacobi(u, 10, 2)
    assert np.array_equal(g1, g2)
    ok_, err = rel_ok(g2, ok.jacobi2d(u, 10), 1e-5)
    assert ok_, err
    assert s2["stale_bytes"] == 40800 == s2["moved_bytes"]
    assert s1["stale_bytes"] == 0 and s1["moved_bytes"] == 0
    assert s2["kernel_launches"] == 20 and s2["pair_bytes"][0][1] == s2["pair_bytes"][1][0] == 20400


@pytest.mark.parametrize("P", [1, 2, 3])
def test_launch_sequence_graph_replay_equals_single_launches(P):
    """pk_launch_sequence (the bench's C1 step): 6 sequences of 10 sweeps are captured and
    then replayed as one graph each, and give bit-for-bit the result of the 60 launches one
    by one (and the 1-way result), within 1e-5 of the fp64 oracle, with the same stale bytes."""
    u = synth.jacobi_grid(512, 512)
    ref, s_single = _jacobi(u, 60, P)
    one, _ = _jacobi(u, 60, 1)
    ctx = gpu_ctx(P)
    pr, out = K.jacobi2d_program(ctx, u, 0)
    for step in range(6):
        out = K.jacobi2d_iterate(pr, 10, 10 * step, sequence=True)
    res = fetch(ctx, out, u.shape)
    st = abi.pk_get_stats(ctx)
    abi.pk_finalize(ctx)
    assert np.array_equal(res, ref) and np.array_equal(res, one)
    ok_, err = rel_ok(res, ok.jacobi2d(u, 60), 1e-5)
    assert ok_, err
    assert st["launches"] == 60 and st["kernel_launches"] == 60 * P
    assert st["stale_bytes"] == s_single["stale_bytes"] and st["moved_bytes"] == s_single["moved_bytes"]
    assert st["graph_fallbacks"] == 0
    assert st["graph_captures"] >= 10 and st["graph_replays"] >= 10   # captured, then replayed whole


@pytest.mark.parametrize("single", [False, True])
def test_paper_vs_validity_tracker_measured_on_gpu(single):
    """SURVEY NEXT-1 / §8(c) paper-vs-validity pins, measured through the library on the GPU
    (the hand derivations are in tests/test_oracle_regions_shadow.py): Jacobi 64^2 at P = 3
    moves exactly 2,540 / 1,056 / 992... B per launch with shared copies, 1,056 B per launch
    from the second on without them; the same GEMM launched twice moves (P-1)|B|
    once vs twice.  Results bit-identical to 1-way in both modes."""
    mode = abi.PK_MODE_SINGLE_OWNER if single else 0
    u = synth.uniform((64, 64), 0, 1, seed=64)
    ref, _ = _jacobi(u, 6, 1)
    ctx = gpu_ctx(3, mode)
    pr = K.Problem(ctx, "jacobi2d")
    b0, b1 = pr.buffer((64, 64), 4, host=u), pr.buffer((64, 64), 4, host=u)
    grid, blk, sc = K.jacobi2d_launch(64, 64)
    per = []
    for t in range(6):
        a, b = (b0, b1) if t % 2 == 0 else (b1, b0)
        abi.pk_reset_stats(ctx)
        pr.launch(grid, blk, [a, b, 64, 64], sc)
        st = abi.pk_get_stats(ctx)
        assert st["moved_bytes"] == st["stale_bytes"]
        per.append(st["moved_bytes"])
    g = fetch(ctx, b0, (64, 64))
    abi.pk_finalize(ctx)
    assert np.array_equal(g, ref)
    assert per == ([2540, 1056, 1056, 1056, 1056, 1056] if single else [2540, 1056, 992, 992, 992, 992])
    m, n, k = 512, 512, 192           # 4 tile rows: one per partition, A's linear slabs aligned
    a_, b_ = synth.gemm_operands(m, n, k)
    g1, _ = _gemm(a_, b_, 1)
    ctx = gpu_ctx(4, mode)
    pr, cb = K.sgemm_program(ctx, a_, b_, launches=2)
    g = fetch(ctx, cb, (m, n))
    st = abi.pk_get_stats(ctx)
    abi.pk_finalize(ctx)
    assert np.array_equal(g, g1)
    assert st["moved_bytes"] == st["stale_bytes"] == (2 if single else 1) * 3 * k * n * 4


def test_c1_harmonic_fixed_point_bit_exact_on_gpu():
    n = 512
    i = np.arange(n, dtype=np.float32)[:, None]
    u = (i * i.T).astype(np.float32)
    g, _ = _jacobi(u, 10, 2)
    assert np.array_equal(g, u)


@pytest.mark.parametrize("h,w", [(37, 50), (64, 64), (130, 257)])
@pytest.mark.parametrize("P", [3, 5, 8])
def test_jacobi_ragged_bitwise(h, w, P):
    u = synth.uniform((h, w), 0, 1, seed=h * w)
    g1, _ = _jacobi(u, 7, 1)
    gp, st = _jacobi(u, 7, P)
    assert np.array_equal(g1, gp)
    assert st["moved_bytes"] == st["stale_bytes"]
    assert rel_ok(gp, ok.jacobi2d(u, 7), 1e-5)[0]


def test_no_transfers_negative_control_and_barrier_mode():
    u = synth.jacobi_grid(128, 128)
    g1, _ = _jacobi(u, 6, 1)
    gb, _ = _jacobi(u, 6, 2, abi.PK_MODE_NO_TRANSFERS)
    assert not np.array_equal(g1, gb)
    gg, _ = _jacobi(u, 6, 4, abi.PK_MODE_GLOBAL_BARRIER)
    assert np.array_equal(g1, gg)
    gs, ss = _jacobi(u, 6, 3, abi.PK_MODE_SINGLE_OWNER)
    assert np.array_equal(g1, gs)


# ------------------------------------------------------------------ C2 Hotspot
def _hotspot(t, p, iters, P, ty=16, bdx=128, mode=0, kernel="hotspot2d", tiles=None):
    ctx = gpu_ctx(P, mode)
    pr = K.hotspot2d_setup(ctx, t, p, ty, bdx, kernel=kernel, tiles=tiles)
    out = K.hotspot2d_iterate(pr, iters)
    res = fetch(ctx, out, t.shape)
    st = abi.pk_get_stats(ctx)
    abi.pk_finalize(ctx)
    return res, st


@pytest.mark.parametrize("kernel,h,w,ty,bdx", [("hotspot2d", 200, 520, 16, 128), ("hotspot2d", 129, 1028, 64, 128),
                                               ("hotspot2d", 3, 4, 64, 128), ("hotspot2d", 300, 2048, 7, 128),
                                               ("hotspot2d_regs", 64, 64, 4, 32), ("hotspot2d_regs", 200, 520, 16, 128)])
def test_hotspot_oracle_and_bitwise(kernel, h, w, ty, bdx):
    t, p = synth.hotspot_grids(h, w)
    iters = 20
    ref = ok.hotspot2d(t, p, iters)
    g1, _ = _hotspot(t, p, iters, 1, ty, bdx, kernel=kernel)
    assert rel_ok(g1, ref, 1e-5)[0]
    for P in (2, 3, 4, 8):
        gp, st = _hotspot(t, p, iters, P, ty, bdx, kernel=kernel)
        assert np.array_equal(g1, gp), P
        assert st["moved_bytes"] == st["stale_bytes"]


def test_hotspot_stale_bytes_closed_form():
    h = w = 1024
    t, p = synth.hotspot_grids(h, w)
    for P in (2, 4, 8):
        _, st = _hotspot(t, p, 10, P, 64, 128)
        assert st["stale_bytes"] == 10 * cf.hotspot2d_stale_per_iter(w, P) == st["moved_bytes"]


@pytest.mark.parametrize("h,w,ty", [(200, 520, 16), (129, 1028, 64), (3, 4, 64), (300, 2048, 7), (64, 1536, 128)])
def test_hotspot_tb2_oracle_and_bitwise(h, w, ty):
    """Two fused sweeps per launch (NEXT-3): oracle within 1e-5, P-way bit-identical."""
    t, p = synth.hotspot_grids(h, w)
    iters = 20
    ref = ok.hotspot2d(t, p, iters)
    g1, s1 = _hotspot(t, p, iters, 1, ty, kernel="hotspot2d_tb2")
    ok_, err = rel_ok(g1, ref, 1e-5)
    assert ok_, err
    assert s1["kernel_launches"] == iters // 2
    for P in (2, 3, 4, 8):
        gp, st = _hotspot(t, p, iters, P, ty, kernel="hotspot2d_tb2")
        assert np.array_equal(g1, gp), P
        assert st["moved_bytes"] == st["stale_bytes"]


@pytest.mark.parametrize("h,w,ty,k", [(200, 520, 16, 4), (129, 1028, 64, 3), (3, 4, 64, 2), (300, 2048, 7, 4),
                                      (64, 1536, 128, 4), (40, 960, 5, 2), (257, 964, 32, 3),
                                      (300, 2048, 32, 6), (131, 900, 16, 8), (70, 452, 9, 5), (64, 1348, 40, 7)])
def test_hotspot_tbk_oracle_and_bitwise(h, w, ty, k):
    """K fused sweeps per launch (NEXT-3, K = 2..8): oracle within 1e-5, P-way bit-identical."""
    t, p = synth.hotspot_grids(h, w)
    iters = 12 if 12 % k == 0 else 2 * k
    ref = ok.hotspot2d(t, p, iters)
    g1, s1 = _hotspot_k(t, p, iters, 1, ty, k)
    ok_, err = rel_ok(g1, ref, 1e-5)
    assert ok_, err
    assert s1["kernel_launches"] == iters // k
    for P in (2, 3, 4, 8):
        gp, st = _hotspot_k(t, p, iters, P, ty, k)
        assert np.array_equal(g1, gp), P
        assert st["moved_bytes"] == st["stale_bytes"]


def _hotspot_k(t, p, iters, P, ty, k):
    ctx = gpu_ctx(P)
    pr = K.hotspot2d_setup(ctx, t, p, ty=ty, kernel="hotspot2d_tbk", sweeps=k)
    out = K.hotspot2d_iterate(pr, iters)
    res = fetch(ctx, out, t.shape)
    st = abi.pk_get_stats(ctx)
    abi.pk_finalize(ctx)
    return res, st


def test_hotspot_tbk_long_run_tolerance():
    """100 time steps (the C2 step) in 25 four-sweep launches stay within 1e-5 of the oracle."""
    h, w = 256, 1920
    t, p = synth.hotspot_grids(h, w)
    ref = ok.hotspot2d(t, p, 100)
    g, _ = _hotspot_k(t, p, 100, 2, 32, 4)
    ok_, err = rel_ok(g, ref, 1e-5)
    assert ok_, err


def test_hotspot_uniform_closed_form_on_gpu():
    h, w = 96, 256
    t = np.full((h, w), 323.0, np.float32)
    p = np.full((h, w), 0.004, np.float32)
    g, _ = _hotspot(t, p, 25, 3)
    exp = cf.hotspot_uniform(323.0, 0.004, 25, ok.HOTSPOT_CAP, ok.HOTSPOT_RZ1, ok.HOTSPOT_AMB)
    assert np.all(np.abs(g - exp) <= 1e-5 * exp)


# ------------------------------------------------------------------ C3 Heat
def _heat(u, iters, P, zc=8, bdy=8, kernel="heat3d", tiles=None, mode=0):
    ctx = gpu_ctx(P, mode)
    pr = K.heat3d_setup(ctx, u, zc, bdy, kernel=kernel, tiles=tiles)
    out = K.heat3d_iterate(pr, iters)
    res = fetch(ctx, out, u.shape)
    st = abi.pk_get_stats(ctx)
    abi.pk_finalize(ctx)
    return res, st


@pytest.mark.parametrize("kernel,d,h,w,zc,bdy", [("heat3d", 40, 36, 132, 8, 8), ("heat3d", 17, 9, 256, 4, 31),
                                                  ("heat3d", 64, 64, 64, 64, 62), ("heat3d", 9, 70, 260, 3, 1),
                                                  ("heat3d", 20, 130, 132, 7, 61),
                                                  ("heat3d", 130, 62, 132, 128, 31),
                                                  ("heat3d_regs", 40, 36, 132, 8, 8),
                                                  ("heat3d_regs", 17, 9, 256, 4, 32)])
def test_heat_oracle_and_bitwise(kernel, d, h, w, zc, bdy):
    u = synth.heat_grid(d, h, w)
    iters = 10
    ref = ok.heat3d(u, iters)
    g1, _ = _heat(u, iters, 1, zc, bdy, kernel)
    assert rel_ok(g1, ref, 1e-5)[0]
    for P in (2, 3, 5):
        gp, st = _heat(u, iters, P, zc, bdy, kernel)
        assert np.array_equal(g1, gp), P
        assert st["moved_bytes"] == st["stale_bytes"]


def test_heat_conservation_on_gpu():
    u = synth.heat_grid(32, 32, 64)
    g, st = _heat(u, 20, 4)
    assert abs(float(g.astype(np.float64).sum()) - float(u.astype(np.float64).sum())) < 1e-5 * u.size
    assert st["stale_bytes"] == 20 * cf.heat3d_stale_per_iter(32, 64, 4)


# ------------------------------------------------------------------ C5 N-body
def _nbody(pos, vel, steps, P, bdx=256):
    ctx = gpu_ctx(P)
    pr = K.nbody_setup(ctx, pos, vel, bdx)
    pb, vb = K.nbody_iterate(pr, steps)
    p_out = fetch(ctx, pb, pos.shape)
    v_out = fetch(ctx, vb, vel.shape)
    st = abi.pk_get_stats(ctx)
    abi.pk_finalize(ctx)
    return p_out, v_out, st


@pytest.mark.parametrize("n", [3000, 1024, 4097])
def test_nbody_oracle_and_bitwise(n):
    """Per step, the oracle advances the GPU's own previous state (fp64), so fp32
    storage rounding of positions is not compounded through close encounters
    (SURVEY §8(c) N-body pin: per-step recomputation from the GPU state)."""
    pos, vel = synth.nbody_bodies(n)
    steps = 3
    ctx = gpu_ctx(2)
    pr = K.nbody_setup(ctx, pos, vel)
    prev_p, prev_v = pos, vel
    for s in range(steps):
        pb, vb = K.nbody_iterate(pr, 1, start=s)
        gp, gv = fetch(ctx, pb, pos.shape), fetch(ctx, vb, vel.shape)
        rp, rv = ok.nbody(prev_p, prev_v, 1)
        assert rel_ok(gv[:, :3], rv[:, :3], 1e-5)[0], rel_ok(gv[:, :3], rv[:, :3], 1e-5)
        assert rel_ok(gp[:, :3], rp[:, :3], 1e-5)[0]
        assert np.array_equal(gp[:, 3], pos[:, 3])
        prev_p, prev_v = gp, gv
    abi.pk_finalize(ctx)
    p1, v1, _ = _nbody(pos, vel, steps, 1)
    for P in (2, 3, 8):
        pp, vp, st = _nbody(pos, vel, steps, P)
        assert np.array_equal(p1, pp) and np.array_equal(v1, vp)
        assert st["moved_bytes"] == st["stale_bytes"]


def test_nbody_two_bodies_and_momentum():
    pos = np.array([[0.1, -0.2, 0.3, 0.5], [0.4, 0.2, -0.1, 0.25]], np.float32)
    vel = np.zeros_like(pos)
    _, v, _ = _nbody(pos, vel, 1, 1)
    a0 = cf.nbody_two_body_accel(pos[0, :3], pos[1, :3], 0.25, ok.NBODY_EPS2)
    assert np.allclose(v[0, :3], a0 * ok.NBODY_DT, rtol=1e-5)
    rpos, rvel = synth.nbody_bodies(2048)
    _, v, _ = _nbody(rpos, rvel, 1, 2)
    mom = (rpos[:, 3:4].astype(np.float64) * v[:, :3]).sum(axis=0)
    assert np.max(np.abs(mom)) < 1e-5 * np.max(np.abs(v[:, :3]))


# ------------------------------------------------------------------ generic path
def test_generic_register_kernel_with_python_descriptors_matches_builtin():
    """pk_register_kernel(pk_builtin_fn) + descriptors declared through the binding
    (the paper's flow: kernel model record + per-argument maps)."""
    n = 200
    u = synth.jacobi_grid(n, n)
    ref, _ = _jacobi(u, 5, 1)
    ctx = gpu_ctx(3)
    fn = abi.pk_builtin_fn("jacobi2d")
    assert fn
    k = abi.pk_register_kernel(ctx, "jacobi_user", fn, [abi.PK_ARG_BUFFER, abi.PK_ARG_BUFFER,
                                                        abi.PK_ARG_SCALAR, abi.PK_ARG_SCALAR])
    H = abi.expr(-1, scalars={0: 1})
    W = abi.expr(-1, scalars={1: 1})
    bdx, bdy = abi.expr(0, blockdim={0: 1}), abi.expr(0, blockdim={1: 1})
    for di, dj in ((-1, 0), (1, 0), (0, -1), (0, 1)):
        abi.pk_declare_affine_access(ctx, k, 0, abi.PK_READ, abi.affine_access([
            abi.dim_map(1, bdy, bdy, di, guard=(1, H)), abi.dim_map(0, bdx, bdx, dj, guard=(1, W))]))
    abi.pk_declare_affine_access(ctx, k, 1, abi.PK_WRITE, abi.affine_access([
        abi.dim_map(1, bdy, bdy, 0, guard=(1, H)), abi.dim_map(0, bdx, bdx, 0, guard=(1, W))]))
    b0 = abi.pk_register_buffer(ctx, (n, n), 4, host_init=u)
    b1 = abi.pk_register_buffer(ctx, (n, n), 4, host_init=u)
    grid, blk, sc = K.jacobi2d_launch(n, n)
    for t in range(5):
        a, b = (b0, b1) if t % 2 == 0 else (b1, b0)
        abi.pk_launch_partitioned(ctx, k, grid, blk, [a, b, n, n], sc)
    g = fetch(ctx, b1, (n, n))
    abi.pk_finalize(ctx)
    assert np.array_equal(g, ref)


def test_caller_owned_torch_instances_and_timer():
    import torch
    h, w = 256, 512
    t, p = synth.hotspot_grids(h, w)
    ref, _ = _hotspot(t, p, 8, 1)
    P = 2
    tens = [[torch.empty((h, w), dtype=torch.float32, device="cuda:0") for _ in range(P)] for _ in range(3)]
    ctx = gpu_ctx(P)
    pr = K.hotspot2d_setup(ctx, t, p, dev_ptrs=[[x.data_ptr() for x in b] for b in tens])
    abi.pk_timer_begin(ctx)
    out = K.hotspot2d_iterate(pr, 8)
    ms = abi.pk_timer_end(ctx)
    assert ms > 0
    g = fetch(ctx, out, (h, w))
    abi.pk_finalize(ctx)
    assert np.array_equal(g, ref)
    # partition 0's instance holds its own rows of the result
    torch.cuda.synchronize()
    assert np.array_equal(tens[0][0][: h // 2].cpu().numpy(), ref[: h // 2])


# ------------------------------------------------------------------ C4 SGEMM (tcgen05 3xTF32)
def _gemm(a, b, P):
    ctx = gpu_ctx(P)
    pr, c = K.sgemm_program(ctx, a, b)
    out = fetch(ctx, c, (a.shape[0], b.shape[1]))
    st = abi.pk_get_stats(ctx)
    abi.pk_finalize(ctx)
    return out, st


def test_gemm_identity_and_rank1_exact():
    rng = np.random.default_rng(21)
    n = 512
    b = rng.uniform(-1, 1, size=(n, n)).astype(np.float32)
    g, _ = _gemm(np.eye(n, dtype=np.float32), b, 1)
    # A = I: C = hi(b) + lo(b) exactly (hi keeps 11 significant bits, lo = rna_tf32(b - hi)
    # has its leading bit at most 2^-11 |b|, so its rounding error is <= 2^-22 |b|; the sum
    # spans <= 22 bits and is exact in the FP32 accumulator) -- SURVEY §8(c) GEMM pin
    assert np.all(np.abs(g.astype(np.float64) - b) <= 2.0 ** -22 * np.abs(b.astype(np.float64)))
    m, nn, k = 256, 512, 64
    u = np.arange(1, m + 1, dtype=np.float32) % 17 + 1
    v = np.arange(1, nn + 1, dtype=np.float32) % 13 + 1
    a = np.repeat(u[:, None], k, axis=1)
    bb = np.repeat(v[None, :], k, axis=0)
    g, _ = _gemm(a, bb, 1)
    assert np.array_equal(g, (k * np.outer(u, v)).astype(np.float32))


def test_gemm_tf32_sensitive_pin():
    # A = 1 + 2^-12 is not a TF32 value: 1xTF32 would give K, 3xTF32 gives K (1 + 2^-12) exactly
    m, n, k = 128, 256, 256
    a = np.full((m, k), 1.0 + 2.0 ** -12, np.float32)
    b = np.ones((k, n), np.float32)
    g, _ = _gemm(a, b, 1)
    assert np.all(g == np.float32(k * (1.0 + 2.0 ** -12)))


@pytest.mark.parametrize("m,n,k", [(300, 520, 200), (512, 512, 512), (1024, 768, 1040)])
def test_gemm_oracle_and_bitwise(m, n, k):
    a, b = synth.gemm_operands(m, n, k)
    ref = ok.gemm(a, b)
    g1, _ = _gemm(a, b, 1)
    ok_, err = rel_ok(g1, ref, 1e-4)
    assert ok_, err
    for P in (2, 3):
        gp, st = _gemm(a, b, P)
        assert np.array_equal(g1, gp), P
        assert st["moved_bytes"] == st["stale_bytes"]


def _gemm_chain(a, b, P, launches, mode=0):
    """X_{t+1} = A X_t (the bench's C4 step): every launch reads the operand the previous
    launch wrote in row slabs, so every launch broadcasts (P-1)/P of it."""
    m, k = a.shape
    n = b.shape[1]
    ctx = gpu_ctx(P, mode)
    pr, _ = K.sgemm_program(ctx, a, b, launches=0)
    grid, blk, sc = pr.geom
    ab, bb, cb = pr.abc
    out = cb
    for t in range(launches):
        x, y = (bb, cb) if t % 2 == 0 else (cb, bb)
        pr.launch(grid, blk, [ab, x, y, m, n, k], sc)
        out = y
    g = fetch(ctx, out, (m, n))
    st = abi.pk_get_stats(ctx)
    abi.pk_finalize(ctx)
    return g, st


@pytest.mark.parametrize("P", [2, 3, 4])
def test_gemm_streamed_operand_overlap(P, monkeypatch):
    """Streamed B (the operand broadcast overlapped with the GEMM, pk_api.h): bit-identical to
    the copy-before-kernel path (PK_MODE_NO_OVERLAP) and to 1-way, every stale byte of the
    operand moved on the side stream, graphs captured and replayed without a fallback."""
    monkeypatch.setenv("PK_STREAM_SAME_DEVICE", "1")   # virtual partitions: stream the D2D copies too
    m = k = n = 1024
    a, b = synth.gemm_operands(m, n, k)
    a *= np.float32((3.0 / k) ** 0.5)
    launches = 6
    g1, _ = _gemm_chain(a, b, 1, launches)
    gs, ss = _gemm_chain(a, b, P, launches)
    gn, sn = _gemm_chain(a, b, P, launches, abi.PK_MODE_NO_OVERLAP)
    assert np.array_equal(gs, g1) and np.array_equal(gn, g1)
    per = (P - 1) * k * n * 4     # the operand X, every launch (A moves only where its linear
    assert ss["streamed_bytes"] == launches * per     # H2D split misses the tile rows: P = 3)
    assert ss["stale_bytes"] == ss["moved_bytes"] == sn["moved_bytes"] == sn["stale_bytes"]
    assert sn["streamed_bytes"] == 0
    assert ss["graph_fallbacks"] == 0 and ss["graph_replays"] >= 1
    # the chain against the oracle: the same X_t from the fp64 product of the GPU's own X_{t-1}
    ref = ok.gemm(a, _gemm_chain(a, b, 1, launches - 1)[0])
    good, err = rel_ok(gs, ref, 1e-4)
    assert good, err


def test_gemm_operand_aliased_is_not_streamed(monkeypatch):
    """C = A A: the streamed argument's buffer is also the A operand, whose loads do not poll the
    arrival flags, so its copies must land before the kernel (no streaming)."""
    monkeypatch.setenv("PK_STREAM_SAME_DEVICE", "1")
    n = 512
    a, _ = synth.gemm_operands(n, n, n)
    ref = ok.gemm(a, a)
    ctx = gpu_ctx(3)
    pr = K.Problem(ctx, "sgemm_tf32x3")
    ab, cb = pr.buffer((n, n), 4, host=a), pr.buffer((n, n), 4)
    grid, blk, sc = K.sgemm_launch(n, n, n)
    pr.launch(grid, blk, [ab, ab, cb, n, n, n], sc)
    g = fetch(ctx, cb, (n, n))
    st = abi.pk_get_stats(ctx)
    abi.pk_finalize(ctx)
    assert st["streamed_bytes"] == 0 and st["moved_bytes"] == st["stale_bytes"] > 0
    good, err = rel_ok(g, ref, 1e-4)
    assert good, err


def test_gemm_read_pattern_placement_moves_nothing():
    """NEXT-1: operands uploaded where the launch reads them (pk_copy_from_host_for)."""
    m, n, k = 768, 512, 256
    a, b = synth.gemm_operands(m, n, k)
    ref, _ = _gemm(a, b, 1)
    ctx = gpu_ctx(3)
    pr = K.Problem(ctx, "sgemm_tf32x3")
    ab, bb, cb = pr.buffer((m, k), 4), pr.buffer((k, n), 4), pr.buffer((m, n), 4)
    grid, blk, sc = K.sgemm_launch(m, n, k)
    abi.pk_copy_from_host_for(ctx, ab, a, pr.k, 0, grid, blk, sc)
    abi.pk_copy_from_host_for(ctx, bb, b, pr.k, 1, grid, blk, sc)
    pr.launch(grid, blk, [ab, bb, cb, m, n, k], sc)
    g = fetch(ctx, cb, (m, n))
    st = abi.pk_get_stats(ctx)
    abi.pk_finalize(ctx)
    assert np.array_equal(g, ref)
    assert st["stale_bytes"] == 0 == st["moved_bytes"]
    good, err = rel_ok(g, ok.gemm(a, b), 1e-4)     # and the oracle, not only the 1-way run
    assert good, err


# ------------------------------------------------------------------ steady-state graph replay
@pytest.mark.parametrize("P", [1, 2, 4])
def test_graph_replay_matches_eager_and_one_way(P):
    t, p = synth.hotspot_grids(256, 1024)
    iters = 24
    ref, _ = _hotspot(t, p, iters, 1)
    ge, se = _hotspot(t, p, iters, P, mode=abi.PK_MODE_NO_GRAPHS)
    gg, sg = _hotspot(t, p, iters, P)
    assert np.array_equal(ge, ref) and np.array_equal(gg, ref)
    assert se["graph_replays"] == 0 and sg["graph_replays"] >= iters - 6 and sg["graph_captures"] >= 1
    for key in ("stale_bytes", "moved_bytes", "copies", "kernel_launches", "launches"):
        assert se[key] == sg[key], key


def test_direct_launch_equals_partitioned_p1():
    """pk_launch_direct (E3 baseline: the original single-GPU launch) computes exactly what
    the library computes at P = 1, and refuses multi-partition contexts."""
    t, p = synth.hotspot_grids(200, 1028)
    ref, _ = _hotspot(t, p, 8, 1, kernel="hotspot2d_tbk")
    ctx = gpu_ctx(1)
    pr = K.hotspot2d_setup(ctx, t, p, 16, kernel="hotspot2d_tbk")
    pr.direct = True
    out = K.hotspot2d_iterate(pr, 8)
    g = fetch(ctx, out, t.shape)
    st = abi.pk_get_stats(ctx)
    abi.pk_finalize(ctx)
    assert np.array_equal(g, ref)
    assert st["launches"] == 0          # nothing went through the partitioned path
    ctx = gpu_ctx(2)
    pr = K.hotspot2d_setup(ctx, t, p, 16)
    pr.direct = True
    with pytest.raises(abi.PkError):
        K.hotspot2d_iterate(pr, 1)
    abi.pk_finalize(ctx)


@pytest.mark.parametrize("P", [1, 3])
def test_failed_capture_falls_back_to_eager(P, monkeypatch):
    """A capture that fails (forced by the PK_DEBUG_FAIL_CAPTURE hook) must not lose the
    launch: its bookkeeping is rolled back, it runs eagerly, and the context stays eager."""
    t, p = synth.hotspot_grids(200, 1028)
    iters = 12
    ref, sref = _hotspot(t, p, iters, P, mode=abi.PK_MODE_NO_GRAPHS)
    monkeypatch.setenv("PK_DEBUG_FAIL_CAPTURE", "1")
    g, st = _hotspot(t, p, iters, P)
    assert np.array_equal(g, ref)
    assert st["graph_fallbacks"] == 1 and st["graph_replays"] == 0 and st["graph_captures"] == 0
    for key in ("stale_bytes", "moved_bytes", "copies", "kernel_launches", "launches"):
        assert st[key] == sref[key], key


def test_graph_mode_interleaved_with_eager_work():
    """Graph replay, then a re-upload (H2D), eager launches (mode switch) and more replay."""
    h, w = 200, 1028
    t, p = synth.hotspot_grids(h, w)
    ctx = gpu_ctx(3)
    pr = K.hotspot2d_setup(ctx, t, p, ty=16)
    K.hotspot2d_iterate(pr, 10)
    abi.pk_copy_from_host(ctx, pr.tb[0], t)            # restart from the initial field
    K.hotspot2d_iterate(pr, 6, start=0)
    abi.pk_set_mode(ctx, abi.PK_MODE_NO_GRAPHS)
    K.hotspot2d_iterate(pr, 3, start=6)
    abi.pk_set_mode(ctx, 0)
    out = K.hotspot2d_iterate(pr, 11, start=9)
    g = fetch(ctx, out, (h, w))
    st = abi.pk_get_stats(ctx)
    abi.pk_finalize(ctx)
    ref, _ = _hotspot(t, p, 20, 1)
    assert np.array_equal(g, ref)
    assert st["graph_replays"] > 0


# ------------------------------------------------------------------ tile partitions (NEXT-2)
@pytest.mark.parametrize("kernel,tiles,bdx", [("hotspot2d", (2, 2, 1), 128), ("hotspot2d", (3, 2, 1), 128),
                                              ("hotspot2d_tb2", (2, 2, 1), 128), ("hotspot2d_tb2", (2, 4, 1), 128),
                                              ("hotspot2d_regs", (4, 2, 1), 32)])
def test_hotspot_tile_partitions_bitwise(kernel, tiles, bdx):
    """px x py tiles: bit-identical to 1-way; halo columns moved as strided 2-D copies;
    with graph replay and eagerly (NO_GRAPHS)."""
    h, w = 300, 1800
    t, p = synth.hotspot_grids(h, w)
    iters = 12
    g1, _ = _hotspot(t, p, iters, 1, 16, bdx, kernel=kernel)
    assert rel_ok(g1, ok.hotspot2d(t, p, iters), 1e-5)[0]
    P = tiles[0] * tiles[1]
    for mode in (0, abi.PK_MODE_NO_GRAPHS):
        gp, st = _hotspot(t, p, iters, P, 16, bdx, mode=mode, kernel=kernel, tiles=tiles)
        assert np.array_equal(g1, gp), (tiles, mode)
        assert st["moved_bytes"] == st["stale_bytes"] > 0
        assert st["strided_copies"] > 0 and st["copy_kernels"] > 0


def test_hotspot_tile_stale_closed_form_on_gpu():
    h, w = 512, 2048
    t, p = synth.hotspot_grids(h, w)
    _, s2 = _hotspot(t, p, 2, 8, 64, tiles=(4, 2, 1))
    _, s6 = _hotspot(t, p, 6, 8, 64, tiles=(4, 2, 1))
    # launches 3..6 are steady state: every internal cut moves one row / column each way
    assert s6["stale_bytes"] - s2["stale_bytes"] == 4 * cf.hotspot2d_tile_stale_per_iter(h, w, 4, 2)
    assert s6["moved_bytes"] == s6["stale_bytes"]


def test_jacobi_tile_partitions_bitwise():
    u = synth.jacobi_grid(200, 300)
    ctx = gpu_ctx(1)
    _, o1 = K.jacobi2d_program(ctx, u, 9)
    g1 = fetch(ctx, o1, u.shape)
    abi.pk_finalize(ctx)
    assert rel_ok(g1, ok.jacobi2d(u, 9), 1e-5)[0]
    for tiles in ((2, 2, 1), (5, 1, 1), (3, 3, 1)):
        ctx = gpu_ctx(tiles[0] * tiles[1])
        _, o = K.jacobi2d_program(ctx, u, 9, tiles=tiles)
        g = fetch(ctx, o, u.shape)
        st = abi.pk_get_stats(ctx)
        abi.pk_finalize(ctx)
        assert np.array_equal(g, g1), tiles
        assert st["moved_bytes"] == st["stale_bytes"]


@pytest.mark.parametrize("kernel", ["heat3d", "heat3d_regs"])
def test_heat_tile_partitions_bitwise(kernel):
    d, h, w = 24, 40, 260
    u = synth.heat_grid(d, h, w)
    iters = 6
    g1, _ = _heat(u, iters, 1, 4, 8, kernel)
    assert rel_ok(g1, ok.heat3d(u, iters), 1e-5)[0]
    for tiles in ((1, 2, 2), (3, 1, 2), (2, 2, 1)):
        for mode in (0, abi.PK_MODE_NO_GRAPHS):
            gp, st = _heat(u, iters, tiles[0] * tiles[1] * tiles[2], 4, 8, kernel, tiles=tiles, mode=mode)
            assert np.array_equal(g1, gp), (tiles, mode)
            assert st["moved_bytes"] == st["stale_bytes"] > 0


# ------------------------------------------------------------------ fused halo push (PK_MODE_PUSH, Q25)
_PUSH_MODES = [abi.PK_MODE_PUSH, abi.PK_MODE_PUSH | abi.PK_MODE_NO_GRAPHS,
               abi.PK_MODE_PUSH | abi.PK_MODE_GLOBAL_BARRIER]


@pytest.mark.parametrize("mode", _PUSH_MODES)
@pytest.mark.parametrize("P", [2, 3, 8])
def test_push_hotspot_bitwise(P, mode):
    """Producing kernels store the neighbours' halo rows into their instances: after the
    first two launches nothing is stale, the result stays bit-identical to 1-way."""
    h, w, iters = 300, 2048, 12
    t, p = synth.hotspot_grids(h, w)
    g1, _ = _hotspot(t, p, iters, 1, 16)
    gp, st = _hotspot(t, p, iters, P, 16, mode=mode)
    assert np.array_equal(g1, gp)
    assert st["pushed_bytes"] > 0 and st["moved_bytes"] == st["stale_bytes"]
    # launches 3.. need nothing: stale bytes = those of the first two launches only
    _, st2 = _hotspot(t, p, 2, P, 16)
    assert st["stale_bytes"] == st2["stale_bytes"]


@pytest.mark.parametrize("P", [2, 4, 5])
def test_push_hotspot_tbk_bitwise(P):
    h, w, iters = 260, 1920, 16
    t, p = synth.hotspot_grids(h, w)
    g1, _ = _hotspot_k(t, p, iters, 1, 32, 4)
    ctx = gpu_ctx(P, abi.PK_MODE_PUSH)
    pr = K.hotspot2d_setup(ctx, t, p, ty=32, kernel="hotspot2d_tbk", sweeps=4)
    gp = fetch(ctx, K.hotspot2d_iterate(pr, iters), t.shape)
    st = abi.pk_get_stats(ctx)
    abi.pk_finalize(ctx)
    assert np.array_equal(g1, gp)
    # steady state: every launch pushes 4 rows each way per cut
    assert st["pushed_bytes"] == (iters // 4 - 1) * 4 * cf.hotspot2d_stale_per_iter(w, P)


@pytest.mark.parametrize("P", [2, 3])
def test_push_heat_and_jacobi_bitwise(P):
    u = synth.heat_grid(40, 36, 132)
    r1, _ = _heat(u, 6, 1)
    rp, st = _heat(u, 6, P, mode=abi.PK_MODE_PUSH)
    assert np.array_equal(r1, rp) and st["pushed_bytes"] == 5 * cf.heat3d_stale_per_iter(36, 132, P)
    uj = synth.jacobi_grid(512, 512)
    c1 = gpu_ctx(1)
    _, ob = K.jacobi2d_program(c1, uj, 10)
    j1 = fetch(c1, ob, uj.shape)
    abi.pk_finalize(c1)
    cp = gpu_ctx(P, abi.PK_MODE_PUSH)
    _, ob = K.jacobi2d_program(cp, uj, 10)
    jp = fetch(cp, ob, uj.shape)
    st = abi.pk_get_stats(cp)
    abi.pk_finalize(cp)
    assert np.array_equal(j1, jp)
    if P == 2:   # C1: 2 x 4,080 B pulled instead of 40,800 B, the rest pushed
        assert st["stale_bytes"] == 8160 and st["pushed_bytes"] == 9 * 4080



# ------------------------------------------------------------------ two-sweep heat (NEXT-3, 3-D)
@pytest.mark.parametrize("d,h,w,zc", [(40, 36, 132, 8), (17, 9, 256, 4), (9, 70, 260, 3), (30, 50, 124, 128),
                                      (5, 3, 4, 2)])
def test_heat3d_tb2_oracle_and_bitwise(d, h, w, zc):
    u = synth.heat_grid(d, h, w)
    iters = 6
    ref = ok.heat3d(u, iters)
    g1, s1 = _heat_tb2(u, iters, 1, zc)
    ok_, err = rel_ok(g1, ref, 1e-5)
    assert ok_, err
    assert s1["kernel_launches"] == iters // 2
    for P in (2, 3, 5):
        gp, st = _heat_tb2(u, iters, P, zc)
        assert np.array_equal(g1, gp), P
        assert st["moved_bytes"] == st["stale_bytes"]


def _heat_tb2(u, iters, P, zc, mode=0):
    ctx = gpu_ctx(P, mode)
    pr = K.heat3d_setup(ctx, u, zc, kernel="heat3d_tb2")
    res = fetch(ctx, K.heat3d_iterate(pr, iters), u.shape)
    st = abi.pk_get_stats(ctx)
    abi.pk_finalize(ctx)
    return res, st


def test_heat3d_tb2_push_bitwise():
    u = synth.heat_grid(40, 36, 132)
    r1, _ = _heat_tb2(u, 8, 1, 8)
    rp, st = _heat_tb2(u, 8, 3, 8, abi.PK_MODE_PUSH)
    assert np.array_equal(r1, rp) and st["pushed_bytes"] > 0


# ------------------------------------------------------------------ K-sweep Jacobi (jacobi2d_tb)
def _jacobi_tb(u, iters, P, k, sequence=True, per_launch=False, mode=0):
    ctx = gpu_ctx(P, mode)
    pr, _ = K.jacobi2d_program(ctx, u, 0, kernel="jacobi2d_tb", sweeps=k)
    stale = []
    if per_launch:
        for _ in range(iters // k):
            abi.pk_reset_stats(ctx)
            out = K.jacobi2d_iterate(pr, k, sequence=False)
            stale.append(abi.pk_get_stats(ctx)["stale_bytes"])
    else:
        out = K.jacobi2d_iterate(pr, iters, sequence=sequence)
    res = fetch(ctx, out, u.shape)
    st = abi.pk_get_stats(ctx)
    abi.pk_finalize(ctx)
    return res, st, stale


@pytest.mark.parametrize("k", [1, 3, 10, 16])
@pytest.mark.parametrize("h,w", [(100, 130), (512, 512), (33, 7)])
def test_jacobi2d_tb_oracle_and_bitwise(h, w, k):
    """K sweeps per launch (ghost zones): within 1e-5 of the fp64 oracle, bit-identical to
    the one-sweep jacobi2d run, P-way bit-identical to 1-way with moved == stale, a
    remainder sweep count as one shorter launch."""
    u = synth.jacobi_grid(h, w)
    iters = 20
    g1, s1, _ = _jacobi_tb(u, iters, 1, k)
    ok_, err = rel_ok(g1, ok.jacobi2d(u, iters), 1e-5)
    assert ok_, err
    ref, _ = _jacobi(u, iters, 1)
    assert np.array_equal(g1, ref)
    assert s1["kernel_launches"] == -(-iters // k)
    for P in (2, 3):
        gp, st, _ = _jacobi_tb(u, iters, P, k)
        assert np.array_equal(g1, gp), P
        assert st["moved_bytes"] == st["stale_bytes"]


@pytest.mark.parametrize("P", [2, 3])
def test_jacobi2d_tb_push_bitwise(P):
    """The halo pushed by the producing jacobi2d_tb kernel (PK_MODE_PUSH) instead of pulled:
    bit-identical to 1-way, the pushed interior rows make later launches move nothing but
    the boundary columns' first copies."""
    u = synth.jacobi_grid(100, 130)
    g1, _, _ = _jacobi_tb(u, 20, 1, 5)
    gp, st, _ = _jacobi_tb(u, 20, P, 5, mode=abi.PK_MODE_PUSH)
    assert np.array_equal(g1, gp)
    assert st["pushed_bytes"] > 0 and st["moved_bytes"] == st["stale_bytes"]


@pytest.mark.parametrize("h,w", [(512, 512), (100, 130)])
def test_jacobi_bit_exact_vs_fp32_cpu_mirror(h, w):
    """SURVEY §8(c)'s optional strong pin: jacobi2d and jacobi2d_tb evaluate the C1 update with
    __fadd_rn / __fmul_rn in the oracle's order, so after 20 sweeps they equal the fp32 CPU
    mirror (oracle/kernels.c, -ffp-contract=off) bit for bit, at P = 1 and 2."""
    u = synth.jacobi_grid(h, w)
    ref = ok.jacobi2d_f32(u, 20)
    for P in (1, 2):
        g1, _ = _jacobi(u, 20, P)
        assert np.array_equal(g1, ref), P
        g5, _, _ = _jacobi_tb(u, 20, P, 5)
        assert np.array_equal(g5, ref), P


def test_jacobi2d_tb_stale_hand_derived_on_gpu():
    """tests/test_oracle_regions_shadow.py's hand count measured through the library: 64^2,
    P = 2, K = 3: 2 K 64 4 B for the first two launches (uploaded buffers, full rows), then
    2 K 62 4 B (the boundary columns are co-held after one copy)."""
    u = synth.jacobi_grid(64, 64)
    g, _, stale = _jacobi_tb(u, 15, 2, 3, per_launch=True)
    assert stale == [1536, 1536, 1488, 1488, 1488]
    ok_, err = rel_ok(g, ok.jacobi2d(u, 15), 1e-5)
    assert ok_, err


# ------------------------------------------------------------------ three-sweep heat (heat3d_tb3)
def _heat_tb3(u, iters, P, zc, mode=0):
    ctx = gpu_ctx(P, mode)
    pr = K.heat3d_setup(ctx, u, zc, kernel="heat3d_tb3")
    res = fetch(ctx, K.heat3d_iterate(pr, iters), u.shape)
    st = abi.pk_get_stats(ctx)
    abi.pk_finalize(ctx)
    return res, st


@pytest.mark.parametrize("d,h,w,zc", [(40, 36, 132, 8), (17, 9, 256, 4), (9, 70, 260, 3), (30, 50, 124, 128),
                                      (5, 3, 4, 2), (13, 22, 248, 1)])
def test_heat3d_tb3_oracle_and_bitwise(d, h, w, zc):
    """Three sweeps per launch: within 1e-5 of the fp64 oracle, P-way bit-identical to 1-way,
    moved == stale == three planes each way per z-cut and launch (closed form), and
    bit-identical to heat3d_tb2 (every cell is the same expression on the same inputs)."""
    u = synth.heat_grid(d, h, w)
    iters = 6
    ref = ok.heat3d(u, iters)
    g1, s1 = _heat_tb3(u, iters, 1, zc)
    ok_, err = rel_ok(g1, ref, 1e-5)
    assert ok_, err
    assert s1["kernel_launches"] == iters // 3
    g2, _ = _heat_tb2(u, iters, 1, max(2, zc))
    assert np.array_equal(g1, g2)
    for P in (2, 3, 5):
        gp, st = _heat_tb3(u, iters, P, zc)
        assert np.array_equal(g1, gp), P
        assert st["moved_bytes"] == st["stale_bytes"]
        nz = -(-d // zc)
        if nz % P == 0 and d % zc == 0 and d // P >= 3:
            assert st["stale_bytes"] == (iters // 3) * cf.heat3d_tb3_stale_per_launch(h, w, P)


@pytest.mark.parametrize("iters", [7, 8])
def test_heat3d_tb3_remainder_sweeps(iters):
    """C3's 50 sweeps = 16 three-sweep launches + a 2-sweep heat3d_tb2 launch: a remainder of
    1 or 2 sweeps runs on heat3d / heat3d_tb2 over the same buffers, bit-identical to
    heat3d_tb2 alone, and calls continue the ping-pong from the launch count."""
    u = synth.heat_grid(20, 34, 252)
    ctx = gpu_ctx(2)
    pr = K.heat3d_setup(ctx, u, 4, kernel="heat3d_tb3")
    K.heat3d_iterate(pr, iters)
    g = fetch(ctx, K.heat3d_iterate(pr, iters), u.shape)
    abi.pk_finalize(ctx)
    ok_, err = rel_ok(g, ok.heat3d(u, 2 * iters), 1e-5)
    assert ok_, err
    ctx = gpu_ctx(1)
    pr = K.heat3d_setup(ctx, u, 4, kernel="heat3d")
    ref = fetch(ctx, K.heat3d_iterate(pr, 2 * iters), u.shape)
    abi.pk_finalize(ctx)
    assert np.array_equal(g, ref)


def test_heat3d_tb3_push_bitwise():
    u = synth.heat_grid(40, 36, 132)
    r1, _ = _heat_tb3(u, 9, 1, 8)
    rp, st = _heat_tb3(u, 9, 3, 8, abi.PK_MODE_PUSH)
    assert np.array_equal(r1, rp) and st["pushed_bytes"] > 0


# ------------------------------------------------------------------ asynchronous host copies (pipelined steps)
@pytest.mark.parametrize("P", [1, 3])
def test_async_host_copies_pipelined_contexts(P):
    """bench.py's e2e pipeline: two contexts, every step = pk_copy_from_host_async of the inputs,
    the launches, pk_sync_to_host_async of the result, no synchronisation between steps; every
    step's result is bit-identical to the blocking path (and within 1e-5 of the oracle)."""
    import torch
    h, w, iters = 200, 1028, 12
    t, p = synth.hotspot_grids(h, w)
    ref, _ = _hotspot_k(t, p, iters, 1, 16, 4)
    ok_, err = rel_ok(ref, ok.hotspot2d(t, p, iters), 1e-5)
    assert ok_, err
    ctxs = [gpu_ctx(P), gpu_ctx(P)]
    zeros = np.zeros_like(t)
    prs = [K.hotspot2d_setup(c, zeros, zeros, ty=16, kernel="hotspot2d_tbk", sweeps=4) for c in ctxs]
    tp, pp = torch.from_numpy(t).pin_memory(), torch.from_numpy(p).pin_memory()
    outs = [torch.full((h, w), -1.0, dtype=torch.float32).pin_memory() for _ in range(5)]
    for s in range(5):
        c, pr = ctxs[s % 2], prs[s % 2]
        abi.pk_copy_from_host_async(c, pr.tb[0], tp)
        abi.pk_copy_from_host_async(c, pr.tb[2], pp)
        out = K.hotspot2d_iterate(pr, iters)
        abi.pk_sync_to_host_async(c, out, outs[s])
    for c in ctxs:
        abi.pk_synchronize(c)
    st = abi.pk_get_stats(ctxs[0])
    for c in ctxs:
        abi.pk_finalize(c)
    for s in range(5):
        assert np.array_equal(outs[s].numpy(), ref), s
    assert st["moved_bytes"] == st["stale_bytes"]


# ------------------------------------------------------------------ randomised launch programs
def _random_program(P, mode, seed, h=200, w=1028, tiles=None):
    """One context, two kernels (one-sweep hotspot2d and four-sweep hotspot2d_tbk) on the same
    ping-pong buffers, and a seeded random mix of launches, re-uploads of the current field and
    mid-program reads -- the hazards of the event DAG (RAW on copies' sources, WAR on both sides,
    pushed halos, graph replay vs eager) in orders no hand-written test has."""
    rng = np.random.default_rng(seed)
    t, p = synth.hotspot_grids(h, w)
    t2 = (t + np.float32(1.5)).astype(np.float32)
    ctx = gpu_ctx(P, mode)
    k1 = abi.pk_builtin_kernel(ctx, "hotspot2d")
    k4 = abi.pk_builtin_kernel(ctx, "hotspot2d_tbk")
    if tiles:   # NEXT-2 tile partitions: column cuts make strided halo copies
        abi.pk_set_partition_shape(ctx, k1, tiles)
        abi.pk_set_partition_shape(ctx, k4, tiles)
    b = [abi.pk_register_buffer(ctx, (h, w), 4, host_init=t), abi.pk_register_buffer(ctx, (h, w), 4)]
    pw = abi.pk_register_buffer(ctx, (h, w), 4, host_init=p)
    g1, bl1, s1 = K.hotspot2d_launch(h, w, 16, K.HOTSPOT_BDX)
    g4, bl4, s4 = K.hotspot2d_tbk_launch(h, w, 16, 4)
    cur, reads = 0, []
    for op in rng.choice(["s1", "s1", "s4", "s4", "s4", "up", "rd"], size=40):
        if op == "s1":
            abi.pk_launch_partitioned(ctx, k1, g1, bl1, [b[cur], pw, b[1 - cur], h, w, s1[2]], s1)
            cur = 1 - cur
        elif op == "s4":
            abi.pk_launch_partitioned(ctx, k4, g4, bl4, [b[cur], pw, b[1 - cur], h, w, s4[2]], s4)
            cur = 1 - cur
        elif op == "up":
            abi.pk_copy_from_host(ctx, b[cur], t2 if len(reads) % 2 else t)
        else:
            reads.append(fetch(ctx, b[cur], (h, w)))
    reads.append(fetch(ctx, b[cur], (h, w)))
    st = abi.pk_get_stats(ctx)
    abi.pk_finalize(ctx)
    return reads, st


@pytest.mark.parametrize("seed", [0, 1, 2, 3, 4])
@pytest.mark.parametrize("P,mode", [(3, 0), (5, 0), (5, abi.PK_MODE_PUSH), (4, abi.PK_MODE_NO_GRAPHS),
                                    (3, abi.PK_MODE_GLOBAL_BARRIER), (5, abi.PK_MODE_SINGLE_OWNER)])
def test_random_launch_programs_bitwise(seed, P, mode):
    ref, _ = _random_program(1, 0, seed)
    got, st = _random_program(P, mode, seed)
    assert len(got) == len(ref)
    for r, g in zip(ref, got):
        assert np.array_equal(r, g)
    assert st["moved_bytes"] == st["stale_bytes"] or mode == abi.PK_MODE_PUSH


@pytest.mark.parametrize("seed", [0, 1, 2])
@pytest.mark.parametrize("tiles,mode", [((2, 2, 1), 0), ((3, 2, 1), 0), ((2, 3, 1), abi.PK_MODE_NO_GRAPHS),
                                        ((3, 1, 1), abi.PK_MODE_SINGLE_OWNER)])
def test_random_launch_programs_tiles_bitwise(seed, tiles, mode):
    """The random programs on tile partitions (2-D and 3-D strided halo copies, the SM
    strided-copy kernel for narrow column halos)."""
    ref, _ = _random_program(1, 0, seed)
    got, st = _random_program(tiles[0] * tiles[1] * tiles[2], mode, seed, tiles=tiles)
    for r, g in zip(ref, got):
        assert np.array_equal(r, g)
    assert st["moved_bytes"] == st["stale_bytes"] and st["strided_copies"] + st["copy_kernels"] > 0
