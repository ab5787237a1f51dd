"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Tolerances (BASELINE.json north star, reading R8): max relative
error <= 1e-5 (f32) / 1e-12 (f64) after 10 iterations on positive fields;
bit-exact (shell included) on integer-valued fields whose every partial sum is
exactly representable.  Where several correct results exist (the summation
order, reading R7) the tests compare against the oracle within tolerance and
check that all CUDA configurations agree bit-for-bit with each other.
"""
import numpy as np
import pytest

import oracle
import stencil_inputs as si

pytestmark = pytest.mark.gpu

TOL = {"f32": 1e-5, "f64": 1e-12}


@pytest.fixture(scope="module")
def S():
    import torch  # noqa: F401
    import paper_conf_ipps_tangtkwkgtw13_b200 as pkg
    return pkg


def run_gpu(S, u, r, coeffs, dtype, iters, cfg=None):
    nz, ny, nx = (d - 2 * r for d in u.shape)
    with S.Plan(nx, ny, nz, r, coeffs, dtype) as p:
        if cfg:
            p.set_config(**cfg)
        a = p.upload(u)
        b = p.alloc()
        p.run(a, b, iters)
        out = p.download(b)
        back = p.download(a)
    assert np.array_equal(back, u.astype(back.dtype)), "stencil_run must not modify its input"
    return out


def rel_err(g, o, r):
    gi = g[r:-r, r:-r, r:-r].astype(np.float64)
    oi = o[r:-r, r:-r, r:-r]
    den = np.maximum(np.abs(oi), 1e-6 * np.max(np.abs(oi)))
    return float(np.max(np.abs(gi - oi) / den))


def shell_equal(g, u, r):
    m = np.ones(u.shape, dtype=bool)
    m[r:-r, r:-r, r:-r] = False
    return np.array_equal(g[m], u[m])


def ws_cfgs(dtype, r):
    """Warp-specialized in-plane configurations (kernel "inplane_ws", inplane_ws.cuh): compute threads a
    multiple of 32, tiles of the registered register shapes, planes per TMA box 1, 2 and 4."""
    vec = 4 if dtype == "f32" else 2
    ry = 2 if r >= 5 else 4
    return [dict(kernel="inplane_ws", tx=16, ty=4, rx=vec, ry=2, stages=3, zsegs=2, zbox=2),
            dict(kernel="inplane_ws", tx=32, ty=4, rx=vec, ry=ry, stages=4, zsegs=3, zbox=1),
            dict(kernel="inplane_ws", tx=16, ty=8, rx=vec, ry=ry, stages=3, zsegs=1, zbox=4, ytiles=5)]


def cfgs(kernel, dtype, r=1):
    vec = 4 if dtype == "f32" else 2
    if kernel == "inplane":
        return cfgs_ip(dtype, r) + ws_cfgs(dtype, r)
    if kernel == "forward":
        return [dict(kernel="forward", tx=32, ty=8, rx=1, ry=1, stages=1, zsegs=1),
                dict(kernel="forward", tx=16, ty=4, rx=1, ry=1, stages=1, zsegs=1)]
    raise ValueError(kernel)


def cfgs_ip(dtype, r):
    vec = 4 if dtype == "f32" else 2
    if r >= 5:  # 2r = 10, 12 accumulator slots per point: smaller register tiles (kern_inst.cuh)
        return [dict(kernel="inplane", tx=32, ty=4, rx=vec, ry=2, stages=3, zsegs=3, zbox=2),
                dict(kernel="inplane", tx=16, ty=2, rx=vec, ry=1, stages=2, zsegs=1, zbox=3),
                dict(kernel="inplane", tx=32, ty=2, rx=vec, ry=2, stages=4, zsegs=2, zbox=1),
                dict(kernel="inplane", tx=16, ty=3, rx=vec, ry=2, stages=3, zsegs=2, zbox=2, ytiles=5)]
    return [dict(kernel="inplane", tx=32, ty=4, rx=vec, ry=2, stages=3, zsegs=3, zbox=2),
            dict(kernel="inplane", tx=16, ty=2, rx=2 * vec, ry=1, stages=2, zsegs=1, zbox=3),
            dict(kernel="inplane", tx=16, ty=4, rx=vec, ry=4, stages=4, zsegs=2, zbox=1),
            dict(kernel="inplane", tx=16, ty=3, rx=vec, ry=2, stages=3, zsegs=2, zbox=2, ytiles=5)]


R_ALL = [1, 2, 3, 4, 5, 6]   # orders 2..12 (Table IV)


@pytest.mark.parametrize("dtype", ["f32", "f64"])
@pytest.mark.parametrize("r", R_ALL)
@pytest.mark.parametrize("kernel", ["inplane", "forward"])
def test_random_field_10_iterations(S, kernel, r, dtype):
    nx, ny, nz = 37, 23, 19 + 2 * r     # ragged: no tile divides it
    u = si.uniform(nx, ny, nz, r, seed=10 * r + len(dtype), dtype=dtype)
    c = si.coeffs_as("heat", r, dtype)
    o = oracle.sweep(u, r, c, 10)
    outs = []
    for cfg in cfgs(kernel, dtype, r):
        if cfg["kernel"] == "forward" and cfg["ty"] < r:
            continue
        g = run_gpu(S, u, r, c, dtype, 10, cfg)
        assert shell_equal(g, u, r)
        assert rel_err(g, o, r) <= TOL[dtype]
        outs.append(g)
    for g in outs[1:]:
        assert np.array_equal(g, outs[0]), "configurations must agree bit-for-bit (reading R7)"


@pytest.mark.parametrize("dtype", ["f32", "f64"])
@pytest.mark.parametrize("r", [1, 4])
def test_c1_64cubed(S, r, dtype):
    cfg = si.CONFIGS["c1"]
    u = si.uniform(64, 64, 64, r, seed=cfg["seed"], dtype=dtype)
    c = si.coeffs_as("heat", r, dtype)
    o = oracle.sweep(u, r, c, 10)
    g_ip = run_gpu(S, u, r, c, dtype, 10)                               # default (model-chosen) config
    g_fp = run_gpu(S, u, r, c, dtype, 10, dict(kernel="forward", tx=32, ty=8, rx=1, ry=1, stages=1, zsegs=1))
    assert rel_err(g_ip, o, r) <= TOL[dtype]
    assert np.array_equal(g_ip, g_fp), "in-plane and forward-plane use the same per-point order"


# integer fields: W = |c0| + 6 sum|c_m|, exact while 8 W^T < 2^24 (f32) / 2^53 (f64)
INT_COEFFS = {1: [-6, 1], 2: [-3, 1, 1], 3: [2, -1, 1, 1], 4: [1, 1, -1, 1, 1], 5: [1, 1, -1, 1, 1, -1],
              6: [1, -1, 1, 1, -1, 1, 1]}


@pytest.mark.parametrize("kernel", ["inplane", "forward"])
@pytest.mark.parametrize("r", R_ALL)
@pytest.mark.parametrize("dtype,iters", [("f32", 2), ("f64", 5)])
def test_integer_field_bit_exact(S, kernel, r, dtype, iters):
    c = INT_COEFFS[r]
    W = abs(c[0]) + 6 * sum(abs(x) for x in c[1:])
    assert 8 * W ** iters < (2 ** 24 if dtype == "f32" else 2 ** 53)
    nx, ny, nz = 41, 29, 13 + 2 * r
    u = si.integers(nx, ny, nz, r, seed=5 + r, dtype=dtype)
    o = oracle.sweep(u, r, [float(x) for x in c], iters)
    for cfg in cfgs(kernel, dtype, r):
        if cfg["kernel"] == "forward" and cfg["ty"] < r:
            continue
        g = run_gpu(S, u, r, c, dtype, iters, cfg)
        assert np.array_equal(g.astype(np.float64), o), cfg


@pytest.mark.parametrize("shape", [(1, 1, 1), (1, 9, 7), (9, 1, 7), (9, 7, 1), (3, 2, 5), (130, 3, 2)])
@pytest.mark.parametrize("r", [1, 4, 6])
def test_degenerate_shapes(S, shape, r):
    nx, ny, nz = shape
    c = INT_COEFFS[r]
    u = si.integers(nx, ny, nz, r, seed=3, dtype="f64")
    o = oracle.sweep(u, r, [float(x) for x in c], 3)
    for kernel in ["inplane", "forward"]:
        with S.Plan(nx, ny, nz, r, c, "f64") as p:
            if kernel == "forward":
                p.set_config(kernel="forward", tx=32, ty=max(4, r), rx=1, ry=1, stages=1, zsegs=1)
            a, b = p.upload(u), p.alloc()
            p.run(a, b, 3)
            assert np.array_equal(p.download(b), o), (kernel, shape)


def test_iters_zero_and_one(S):
    r = 2
    u = si.uniform(20, 17, 11, r, seed=9, dtype="f32")
    c = si.coeffs_as("heat", r, "f32")
    g0 = run_gpu(S, u, r, c, "f32", 0)
    assert np.array_equal(g0, u)
    g1 = run_gpu(S, u, r, c, "f32", 1)
    assert rel_err(g1, oracle.sweep(u, r, c, 1), r) <= 1e-6


def test_every_config_of_the_tuning_space_agrees(S):
    """All tunable configurations give bit-identical output (reading R7)."""
    import torch
    r, dtype = 4, "f32"
    nx, ny, nz = 70, 45, 40
    u = si.uniform(nx, ny, nz, r, seed=21, dtype=dtype)
    c = si.coeffs_as("heat", r, dtype)
    o = oracle.sweep(u, r, c, 3)
    with S.Plan(nx, ny, nz, r, c, dtype) as p:
        a = p.upload(u)
        s0, s1 = p.upload(u), p.upload(u)
        p.tune(kernel="inplane", beta=100, iters_per_rep=1, reps=1, scratch=(s0, s1))
        configs = [e["cfg"] for e in p.tune_results()]
        assert len(configs) > 20
        ref = None
        for cfg in configs[:: max(1, len(configs) // 60)]:
            cfg = dict(cfg)
            cfg["kernel"] = "inplane"
            p.set_config(**cfg)
            b = p.alloc()
            p.run(a, b, 3)
            g = p.download(b)
            if ref is None:
                ref = g
                assert rel_err(g, o, r) <= TOL[dtype]
            assert np.array_equal(g, ref), cfg
        torch.cuda.synchronize()


def test_tune_beta_and_exhaustive(S):
    r, dtype = 4, "f32"
    n = 128
    u = si.uniform(n, n, n, r, seed=4, dtype=dtype)
    c = si.coeffs_as("heat", r, dtype)
    with S.Plan(n, n, n, r, c, dtype) as p:
        s0, s1 = p.upload(u), p.upload(u)
        rep5 = p.tune(kernel="inplane", model="b200", beta=5, iters_per_rep=2, reps=3, scratch=(s0, s1))
        assert rep5["timed"] == max(1, -(-rep5["space_size"] * 5 // 100))
        assert rep5["best_measured_gpts"] > 0
        rep_fp = p.tune(kernel="forward", model="paper", beta=0, iters_per_rep=2, reps=3, scratch=(s0, s1))
        assert rep_fp["timed"] == rep_fp["space_size"]
        assert p.config["kernel"] == "forward"


def test_fill_counter_matches_inputs_module(S):
    import torch
    for dtype in ["f32", "f64"]:
        r, nx, ny, nz = 3, 33, 20, 9
        with S.Plan(nx, ny, nz, r, [0.5, 0.1, 0.1, 0.1], dtype) as p:
            t = p.alloc()
            p.fill_counter(t, seed=5)
            torch.cuda.synchronize()
            g = p.download(t)
            assert np.array_equal(g, si.counter(nx, ny, nz, r, 5, dtype))


def test_error_paths(S):
    import torch
    with S.Plan(16, 16, 16, 1, [0.5, 0.1], "f32") as p:
        a, b = p.alloc(), p.alloc()
        with pytest.raises(S.StencilError) as e:
            p.run(a, b, -1)
        assert e.value.status == 1
        with pytest.raises(S.StencilError) as e:
            p.run_raw(a.data_ptr() + 4, b.data_ptr(), 1, torch.cuda.current_stream().cuda_stream)
        assert e.value.status == 3
        with pytest.raises(S.StencilError) as e:
            p.run(a, a, 1)
        assert e.value.status == 1
        with pytest.raises(S.StencilError):
            p.set_config(kernel="inplane", tx=20, ty=4)       # not a half-warp multiple (constraint (i))
        with pytest.raises(S.StencilError):
            p.set_config(kernel="inplane", tx=64, ty=8, rx=8, ry=1)  # 512 threads; box 264 > 256


@pytest.mark.slow
def test_c2_full_size_sampled(S):
    """512^3 r=4 f32 (BASELINE configs[1]) in the bench's launch configuration,
    10 iterations, sampled against the oracle point by point."""
    import torch
    cfgd = si.CONFIGS["c2"]
    n, r, dtype = 512, 4, "f32"
    u = si.uniform(n, n, n, r, seed=cfgd["seed"], dtype=dtype)
    c = si.coeffs_as("heat", r, dtype)
    with S.Plan(n, n, n, r, c, dtype) as p:
        a = p.upload(u)
        s0, s1 = p.upload(u), p.upload(u)
        p.tune(kernel="inplane", beta=5, iters_per_rep=3, reps=3, scratch=(s0, s1))   # as bench.py does
        del s0, s1
        b = p.alloc()
        p.run(a, b, 10)
        torch.cuda.synchronize()
        g = p.outer_view(b)
        rng = np.random.default_rng(0)
        pts = [(0, 0, 0), (n - 1, n - 1, n - 1), (0, n - 1, 255), (n - 1, 0, 0), (127, 128, 129), (511, 300, 1)]
        pts += [tuple(int(x) for x in rng.integers(0, n, 3)) for _ in range(10)]
        for (i, j, k) in pts:
            o = oracle.point(u, r, c, 10, i, j, k)
            v = float(g[k + r, j + r, i + r])
            assert abs(v - o) <= TOL[dtype] * abs(o), (i, j, k, v, o)


def test_dist_plan_single_rank_matches_plan(S):
    """A distributed plan of one rank (no communicator) is the single-GPU plan."""
    import torch
    r, nx, ny, nz = 4, 40, 24, 30
    c = si.coeffs_as("heat", r, "f32")
    cfg = dict(kernel="inplane", tx=16, ty=2, rx=4, ry=2, stages=3, zsegs=3, zbox=2)
    with S.Plan(nx, ny, nz, r, c, "f32") as p, S.DistPlan(nx, ny, nz, r, c, "f32", bytes(128), 0, 1) as d:
        assert (d.z0, d.nz_local) == (0, nz)
        for q in (p, d):
            q.set_config(**cfg)
        a, b = p.alloc(), p.alloc()
        p.fill_counter(a, 11)
        ad, bd = d.alloc(), d.alloc()
        d.fill_counter(ad, 11)
        p.run(a, b, 5)
        d.run(ad, bd, 5)
        torch.cuda.synchronize()
        assert torch.equal(a, ad)
        assert torch.equal(b, bd)
        o = oracle.sweep(p.download(a), r, c, 5)
        assert rel_err(p.download(b), o, r) <= TOL["f32"]


def test_sweep_timing_modes(S):
    """Timing mode 1 accumulates run spans, mode 2 per-sweep events; results unchanged."""
    import torch
    r, n = 2, 48
    c = si.coeffs_as("heat", r, "f32")
    with S.Plan(n, n, n, r, c, "f32") as p:
        a, b = p.alloc(), p.alloc()
        p.fill_counter(a, 3)
        p.run(a, b, 3)
        ref = b.clone()
        for mode in (1, 2):
            p.set_timing(mode)
            for iters in (3, 2, 1):
                p.run(a, b, iters)
            torch.cuda.synchronize()
            s = p.stats()
            assert s["timing_enabled"] == mode
            assert s["timed_sweeps"] == 6 and s["timed_sweep_ms"] > 0
            assert s["last_run_sweeps"] == 1 and 0 < s["last_run_sweep_ms"] <= s["timed_sweep_ms"]
            if mode == 2:
                assert 0 < s["sweep_ms_min"] <= s["sweep_ms_max"]
            else:
                assert s["sweep_ms_min"] == -1.0
            p.set_timing(0)
        p.run(a, b, 3)
        torch.cuda.synchronize()
        assert torch.equal(b, ref)
        with pytest.raises(S.StencilError):
            p.set_timing(3)


def wide_cfgs(dtype, r):
    """Tiles narrower than the 150 x 70 grid below, so every in-plane store mode runs: interior tiles
    (mode 0: no checks), full-width tiles with a partial row range (mode 1) and the ragged x tile (mode 2)."""
    vec = 4 if dtype == "f32" else 2
    ry = 2 if r >= 5 else 4
    return [dict(kernel="inplane", tx=16, ty=4, rx=vec, ry=ry, stages=4, zsegs=2, zbox=2),        # W=64|32, H=16|8
            dict(kernel="inplane", tx=16, ty=15, rx=vec, ry=ry, stages=6, zsegs=2, zbox=1),       # the bench's shape
            dict(kernel="inplane", tx=32, ty=4, rx=vec, ry=2, stages=3, zsegs=3, zbox=2),
            dict(kernel="inplane", tx=16, ty=8, rx=vec, ry=ry, stages=3, zsegs=1, zbox=4, ytiles=5)] + ws_cfgs(dtype, r)


WIDE = (150, 70)


@pytest.mark.parametrize("dtype", ["f32", "f64"])
@pytest.mark.parametrize("r", [1, 2, 4, 6])
def test_random_wide_all_store_modes(S, r, dtype):
    nx, ny = WIDE
    nz = 19 + 2 * r
    u = si.uniform(nx, ny, nz, r, seed=300 + r, dtype=dtype)
    c = si.coeffs_as("heat", r, dtype)
    o = oracle.sweep(u, r, c, 10)
    outs = []
    for cfg in wide_cfgs(dtype, r) + [dict(kernel="forward", tx=32, ty=8, rx=1, ry=1, stages=1, zsegs=1)]:
        g = run_gpu(S, u, r, c, dtype, 10, cfg)
        assert shell_equal(g, u, r), cfg
        assert rel_err(g, o, r) <= TOL[dtype], cfg
        outs.append(g)
    for g in outs[1:]:
        assert np.array_equal(g, outs[0]), "configurations must agree bit-for-bit (reading R7)"


@pytest.mark.parametrize("dtype,iters", [("f32", 2), ("f64", 5)])
@pytest.mark.parametrize("r", [1, 3, 4, 5, 6])   # r >= 5 and fp64: the 16-byte store path of K-IP/WS
def test_integer_wide_all_store_modes(S, r, dtype, iters):
    nx, ny = WIDE
    c = INT_COEFFS[r]
    u = si.integers(nx, ny, 13 + 2 * r, r, seed=400 + r, dtype=dtype)
    o = oracle.sweep(u, r, [float(x) for x in c], iters)
    for cfg in wide_cfgs(dtype, r):
        g = run_gpu(S, u, r, c, dtype, iters, cfg)
        assert np.array_equal(g.astype(np.float64), o), cfg


@pytest.mark.slow
def test_c2_full_grid_bench_config(S):
    """512^3 r=4 f32 (BASELINE configs[1]) in the launch configuration bench.py times (the committed
    tuned configuration), 10 iterations, compared with the oracle at EVERY point: max relative error
    <= 1e-5, shell bit-exact ("verified ... consistent with the CPU"; R8)."""
    import torch
    import bench
    cfgd = si.CONFIGS["c2"]
    n, r, dtype = 512, 4, "f32"
    u = si.uniform(n, n, n, r, seed=cfgd["seed"], dtype=dtype)
    c = si.coeffs_as("heat", r, dtype)
    cfg = bench.pinned_config("c2")
    assert cfg is not None, "bench.py has no pinned configuration for c2"
    g = run_gpu(S, u, r, c, dtype, 10, cfg)
    torch.cuda.empty_cache()
    o = oracle.sweep(u, r, c, 10)
    assert shell_equal(g, u, r)
    err = rel_err(g, o, r)
    assert err <= TOL[dtype], err


ABLATION = ["ip_classic", "ip_vertical", "ip_horizontal", "ip_fullslice", "ip_fullslice_v"]


@pytest.mark.parametrize("dtype", ["f32", "f64"])
@pytest.mark.parametrize("r", [1, 2, 4, 6])
def test_loading_variants_and_forward_rb_bit_identical(S, r, dtype):
    """The paper's in-plane loading variants (Fig. 6 a-d) with per-thread loads, with and
    without register rows, and the forward-plane baseline with register rows (Fig. 10 case (i)) compute
    the same per-point order as K-IP: bit-identical outputs, and the oracle within tolerance."""
    nx, ny, nz = 53, 29, 17 + 2 * r       # ragged in x, y and z
    u = si.uniform(nx, ny, nz, r, seed=500 + r, dtype=dtype)
    c = si.coeffs_as("heat", r, dtype)
    ref = run_gpu(S, u, r, c, dtype, 5)   # the plan's default in-plane configuration
    assert rel_err(ref, oracle.sweep(u, r, c, 5), r) <= TOL[dtype]
    ty = max(4, r)
    for kern in ABLATION:
        for ry in (1, 2, 4):
            for zsegs in (1, 3):
                cfg = dict(kernel=kern, tx=16, ty=ty, rx=1, ry=ry, stages=1, zsegs=zsegs, zbox=1)
                g = run_gpu(S, u, r, c, dtype, 5, cfg)
                assert np.array_equal(g, ref), cfg
    for ry in (1, 2, 4):
        cfg = dict(kernel="forward", tx=32, ty=ty, rx=1, ry=ry, stages=1, zsegs=1, zbox=1)
        assert np.array_equal(run_gpu(S, u, r, c, dtype, 5, cfg), ref), cfg


@pytest.mark.parametrize("kern", ABLATION + ["forward"])
def test_loading_variants_integer_bit_exact(S, kern):
    r, dtype, iters = 3, "f32", 2
    c = INT_COEFFS[r]
    nx, ny, nz = 70, 37, 15
    u = si.integers(nx, ny, nz, r, seed=66, dtype=dtype)
    o = oracle.sweep(u, r, [float(x) for x in c], iters)
    for ry in (1, 4):
        cfg = dict(kernel=kern, tx=32, ty=4, rx=1, ry=ry, stages=1, zsegs=2 if kern != "forward" else 1, zbox=1)
        g = run_gpu(S, u, r, c, dtype, iters, cfg)
        assert np.array_equal(g.astype(np.float64), o), cfg


def fp_tma_cfgs(r, dtype):
    """Forward-plane + TMA (fp_tma.cuh): stages at and above the minimum ceil(r/zbox) + 2, box depths 1, 2
    and 4, register rows 1, 2 and 4, z segments, a balanced y partition."""
    vec = 4 if dtype == "f32" else 2
    out = []
    for zb, ry, zsegs, extra, ytiles in ((1, 1, 1, 0, 0), (2, 2, 3, 1, 0), (4, 4, 2, 0, 3), (2, 1, 1, 2, 0)):
        st = (r + zb - 1) // zb + 2 + extra
        out.append(dict(kernel="fp_tma", tx=16, ty=4, rx=vec, ry=ry, stages=st, zsegs=zsegs, zbox=zb, ytiles=ytiles))
    return out


@pytest.mark.parametrize("dtype", ["f32", "f64"])
@pytest.mark.parametrize("r", [1, 2, 3, 4, 6])
def test_fp_tma_bit_identical(S, r, dtype):
    """The forward-plane method with K-IP's TMA loads computes the fixed per-point order: bit-identical to
    K-IP on a grid ragged in x, y and z, over an odd and an even number of sweeps (both stream
    directions), and within tolerance of the oracle."""
    nx, ny, nz = 75, 29, 19 + 2 * r
    u = si.uniform(nx, ny, nz, r, seed=700 + r, dtype=dtype)
    c = si.coeffs_as("heat", r, dtype)
    for iters in (3, 4):
        ref = run_gpu(S, u, r, c, dtype, iters)
        assert rel_err(ref, oracle.sweep(u, r, c, iters), r) <= TOL[dtype]
        for cfg in fp_tma_cfgs(r, dtype):
            try:
                g = run_gpu(S, u, r, c, dtype, iters, cfg)
            except S.StencilError as e:   # a register tile not instantiated for this radius
                assert "instantiation" in str(e) or "exceeds" in str(e), (cfg, e)
                continue
            assert np.array_equal(g, ref), (iters, cfg)


def test_fp_tma_integer_bit_exact_and_stage_floor(S):
    r, dtype, iters = 3, "f32", 2
    c = INT_COEFFS[r]
    u = si.integers(70, 37, 15, r, seed=67, dtype=dtype)
    o = oracle.sweep(u, r, [float(x) for x in c], iters)
    cfg = dict(kernel="fp_tma", tx=16, ty=4, rx=4, ry=2, stages=5, zsegs=2, zbox=1)
    assert np.array_equal(run_gpu(S, u, r, c, dtype, iters, cfg).astype(np.float64), o)
    with pytest.raises(S.StencilError, match="stages"):   # ring too shallow: refused, never launched
        run_gpu(S, u, r, c, dtype, iters, dict(cfg, stages=4))
