"""GPU parity of the application stencils (Table V; BASELINE config 3
"3D wave") through the C ABI against oracle.source / oracle.wave.

Tolerances as tests/test_parity_gpu.py (R8; the leapfrog wave, a signed field
that cancels, is gated by the forward-error bound of reading R8b); integer-valued fields
with integer coefficients are compared bit for bit (every partial sum exact).
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


def wave_coeffs(r, dtype):
    """u_tt = Lap u, leapfrog with k = (c dt/h)^2 = 1/16: c0 = 2 + k 3a_0, c_m = k a_m, d = -1."""
    a = si.fd_weights(r)
    k = 1 / 16
    c = [2 + k * 3 * float(a[0])] + [k * float(a[m]) for m in range(1, r + 1)]
    return np.array(c, dtype=si.DTYPES[dtype]).astype(np.float64)


def cfgs(kernel, dtype, r):
    vec = 4 if dtype == "f32" else 2
    if kernel == "forward":
        return [dict(kernel="forward", tx=32, ty=8, rx=1, ry=1, stages=1, zsegs=1)]
    ry = 2 if r >= 5 else 4
    return [dict(kernel="inplane", tx=32, ty=4, rx=vec, ry=2, stages=3, zsegs=3, zbox=2),
            dict(kernel="inplane", tx=16, ty=4, rx=vec, ry=ry, stages=2, zsegs=2, zbox=1),
            dict(kernel="inplane", tx=16, ty=3, rx=vec, ry=2, stages=3, zsegs=2, zbox=2, ytiles=5)]


def norm_err(g, o, r):
    """Normwise max|g - o| / max|o| over the interior (reported beside the bound gate below)."""
    gi = g[r:-r, r:-r, r:-r].astype(np.float64)
    oi = o[r:-r, r:-r, r:-r]
    return float(np.max(np.abs(gi - oi)) / np.max(np.abs(oi)))


def abs_stencil(X, c, r):
    """|S|(X): Eq. (1) with |c_m| on a non-negative outer array (interior only, shell 0)."""
    out = np.zeros_like(X)
    nz, ny, nx = X.shape
    I = (slice(r, -r),) * 3
    out[I] = abs(c[0]) * X[I]
    for m in range(1, r + 1):
        out[I] += abs(c[m]) * (X[r:-r, r:-r, r - m:nx - r - m] + X[r:-r, r:-r, r + m:nx - r + m]
                               + X[r:-r, r - m:ny - r - m, r:-r] + X[r:-r, r + m:ny - r + m, r:-r]
                               + X[r - m:nz - r - m, r:-r, r:-r] + X[r + m:nz - r + m, r:-r, r:-r])
    return out


def wave_error_bound(u0, u1, c, d, r, steps, dtype):
    """Forward-error bound for `steps` leapfrog steps u+ = S(u) + d u- (reading R8b).

    Local rounding: each output point is a (6r+2)-term sum c0 u + sum_m c_m (6 neighbours) + d u-
    evaluated in the fixed order with one extra pair add, so |fl - exact| <= gamma_n (|S|(|u_t|) +
    |d||u_{t-1}|) with gamma_n = n eps / (1 - n eps), n = 6r+3 (the standard bound for an n-term sum of
    products in any order).  Propagation: an error injected at step t reaches step T through the linear
    leapfrog map, whose infinity norm rho_k is the l1 norm of its k-step impulse response (computed with
    the oracle, free space; x2 for the frozen-shell restriction).  Bound = 2 sum_t rho_{T-t} max D_t,
    for the plan's rounding plus the fp64 oracle's own."""
    eps = {"f32": 2.0 ** -24, "f64": 2.0 ** -53}[dtype]
    n = 6 * r + 3
    gam = n * eps / (1 - n * eps) + n * 2.0 ** -53 / (1 - n * 2.0 ** -53)
    I = (slice(r, -r),) * 3
    D = []
    p_, u_ = u0.astype(np.float64), u1.astype(np.float64)
    for t in range(1, steps + 1):
        D.append(float((gam * (abs_stencil(np.abs(u_), c, r) + abs(d) * np.abs(p_)))[I].max()))
        p_, u_ = oracle.wave(p_, u_, d, r, c, 1)
    m = 2 * r * steps + 3
    z = np.zeros((m + 2 * r,) * 3)
    ip, iu = z.copy(), z.copy()
    iu[(m + 2 * r) // 2, (m + 2 * r) // 2, (m + 2 * r) // 2] = 1.0
    rho = [1.0]
    for k in range(1, steps):
        ip, iu = oracle.wave(ip, iu, d, r, c, 1)
        rho.append(float(np.abs(iu).sum()))
    return 2.0 * sum(rho[steps - t] * D[t - 1] for t in range(1, steps + 1))


def rel_err(g, o, r):
    gi = g[r:-r, r:-r, r:-r].astype(np.float64)
    oi = o[r:-r, r:-r, r:-r]
    den = np.maximum(np.abs(oi), 1e-6 * np.max(np.abs(oi)))
    return float(np.max(np.abs(gi - oi) / den))


@pytest.mark.parametrize("dtype", ["f32", "f64"])
@pytest.mark.parametrize("r", [1, 2, 4, 6])
@pytest.mark.parametrize("kernel", ["inplane", "forward"])
def test_source_random(S, kernel, r, dtype):
    nx, ny, nz = 37, 23, 19 + 2 * r
    u = si.uniform(nx, ny, nz, r, seed=20 + r, dtype=dtype)
    f = si.uniform(nx, ny, nz, r, seed=40 + r, dtype=dtype)
    c = si.coeffs_as("heat", r, dtype)
    d = float(np.array(0.0625, dtype=si.DTYPES[dtype]))
    o = oracle.source(u, f, d, r, c, 10)
    outs = []
    for cfg in cfgs(kernel, dtype, r):
        if cfg["kernel"] == "forward" and cfg["ty"] < r:
            continue
        with S.Plan(nx, ny, nz, r, c, dtype, app="source", d=d) as p:
            p.set_config(**cfg)
            a, fg, b = p.upload(u), p.upload(f), p.alloc()
            p.run_source(a, fg, b, 10)
            g = p.download(b)
            assert np.array_equal(p.download(a), u.astype(g.dtype))   # in preserved
        assert rel_err(g, o, r) <= TOL[dtype], cfg
        outs.append(g)
    for g in outs[1:]:
        assert np.array_equal(g, outs[0]), "configurations must agree bit-for-bit (reading R7)"


@pytest.mark.parametrize("dtype", ["f32", "f64"])
@pytest.mark.parametrize("r", [1, 3, 4, 5])
@pytest.mark.parametrize("steps", [1, 2, 3, 10])
def test_wave_random(S, r, dtype, steps):
    nx, ny, nz = 33, 21, 17 + 2 * r
    u1 = si.uniform(nx, ny, nz, r, seed=60 + r, dtype=dtype)
    u0 = si.uniform(nx, ny, nz, r, seed=80 + r, dtype=dtype)
    c = wave_coeffs(r, dtype)
    op, ou = oracle.wave(u0, u1, -1.0, r, c, steps)
    bound = wave_error_bound(u0, u1, c, -1.0, r, steps, dtype)
    bound_prev = wave_error_bound(u0, u1, c, -1.0, r, steps - 1, dtype) if steps > 1 else 0.0
    res = []
    for kernel in ["inplane", "forward"]:
        for cfg in cfgs(kernel, dtype, r)[:2]:
            if cfg["kernel"] == "forward" and cfg["ty"] < r:
                continue
            with S.Plan(nx, ny, nz, r, c, dtype, app="wave", d=-1.0) as p:
                p.set_config(**cfg)
                a, b = p.upload(u0), p.upload(u1)
                p.run_wave(a, b, steps)
                gp, gu = p.download(a), p.download(b)
            eu = float(np.max(np.abs(gu.astype(np.float64) - ou)))
            ep = float(np.max(np.abs(gp.astype(np.float64) - op)))
            assert eu <= bound, (cfg, steps, eu, bound, norm_err(gu, ou, r), rel_err(gu, ou, r))
            assert ep <= bound_prev, (cfg, steps, ep, bound_prev, norm_err(gp, op, r))
            if steps == 1:   # one step: the north-star tolerance, normwise (R8b)
                assert norm_err(gu, ou, r) <= TOL[dtype], (cfg, norm_err(gu, ou, r))
            res.append((gp, gu))
    for gp, gu in res[1:]:
        assert np.array_equal(gu, res[0][1]) and np.array_equal(gp, res[0][0])


@pytest.mark.parametrize("kernel", ["inplane", "forward"])
@pytest.mark.parametrize("r", [1, 2, 4, 6])
def test_integer_fields_bit_exact(S, kernel, r):
    # integer coefficients, d = -1: W = |c0| + 6 sum|c_m| + 1, exact while 8 W^T < 2^24 (f32)
    c = {1: [2, 1], 2: [2, 1, -1], 4: [2, 1, -1, 1, 1], 6: [1, -1, 1, 1, -1, 1, 1]}[r]
    nx, ny, nz = 29, 18, 11 + 2 * r
    u0 = si.integers(nx, ny, nz, r, seed=7, dtype="f32")
    u1 = si.integers(nx, ny, nz, r, seed=8, dtype="f32")
    f = si.integers(nx, ny, nz, r, seed=9, dtype="f32")
    cfg = cfgs(kernel, "f32", r)[0] if kernel == "inplane" else dict(kernel="forward", tx=32, ty=8, rx=1, ry=1,
                                                                      stages=1, zsegs=1)
    with S.Plan(nx, ny, nz, r, c, "f32", app="wave", d=-1.0) as p:
        p.set_config(**cfg)
        a, b = p.upload(u0), p.upload(u1)
        p.run_wave(a, b, 2)
        op, ou = oracle.wave(u0, u1, -1.0, r, [float(x) for x in c], 2)
        assert np.array_equal(p.download(b).astype(np.float64), ou)
        assert np.array_equal(p.download(a).astype(np.float64), op)
    with S.Plan(nx, ny, nz, r, c, "f32", app="source", d=-1.0) as p:
        p.set_config(**cfg)
        a, fg, b = p.upload(u1), p.upload(f), p.alloc()
        p.run_source(a, fg, b, 2)
        assert np.array_equal(p.download(b).astype(np.float64), oracle.source(u1, f, -1.0, r, [float(x) for x in c], 2))


def test_poisson_jacobi_converges_on_gpu(S):
    # Jacobi iteration of the r = 1 FD Poisson problem (diagonally dominant; for r >= 2 the
    # order-2r FD Laplacian is not, and Jacobi diverges): converges to the polynomial solution
    import torch
    r, n = 1, 12
    a = si.fd_weights(r)
    w0 = 3 * a[0]
    c = [0.0] + [float(-a[m] / w0) for m in range(1, r + 1)]
    d = float(1 / w0)
    K, J, I = np.meshgrid(*(np.arange(n + 2 * r),) * 3, indexing="ij")
    p = 0.01 * (I * I + 2 * J * J - K * K) + 0.05 * I * K
    lap = np.full(p.shape, 0.01 * (2 + 4 - 2))   # Lap p, exact for the r = 1 FD Laplacian (degree 2)
    u0 = p.copy()
    u0[r:-r, r:-r, r:-r] = 0.0
    with S.Plan(n, n, n, r, c, "f64", app="source", d=d) as pl:
        x, fg, y = pl.upload(u0), pl.upload(lap), pl.alloc()
        pl.run_source(x, fg, y, 1500)
        torch.cuda.synchronize()
        g = pl.download(y)
    assert np.max(np.abs(g - p)) < 1e-9
    assert np.max(np.abs(g - oracle.source(u0, lap, d, r, c, 1500))) < 1e-12


def test_app_plan_kind_errors(S):
    import torch
    c = si.coeffs_as("heat", 1, "f32")
    with S.Plan(8, 8, 8, 1, c, "f32", app="wave", d=-1.0) as p:
        a, b = p.alloc(), p.alloc()
        with pytest.raises(S.StencilError):
            p.run(a, b, 1)                 # a WAVE plan has no plain run
        with pytest.raises(S.StencilError):
            p.run_source(a, a, b, 1)
        with pytest.raises(S.StencilError):
            p.run_wave(a, a, 1)            # u_prev and u overlap
        p.run_wave(a, b, 0)
        torch.cuda.synchronize()
    with S.Plan(8, 8, 8, 1, c, "f32") as p:
        a, b = p.alloc(), p.alloc()
        with pytest.raises(S.StencilError):
            p.run_wave(a, b, 1)
    with pytest.raises(S.StencilError):
        S.Plan(8, 8, 8, 1, c, "f32", app="source", d=float("nan"))


def test_app_tuning(S):
    import torch
    r, n = 2, 64
    c = si.coeffs_as("heat", r, "f32")
    with S.Plan(n, n, n, r, c, "f32", app="wave", d=-1.0) as p:
        s0, s1 = p.alloc(), p.alloc()
        p.fill_counter(s0, 1)
        s1.copy_(s0)
        rep = p.tune(kernel="inplane", model="b200", beta=5, iters_per_rep=2, reps=1, scratch=(s0, s1))
        assert rep["timed"] >= 1 and rep["best_measured_gpts"] > 0
        u0, u1 = p.alloc(), p.alloc()
        p.fill_counter(u0, 2)
        p.fill_counter(u1, 3)
        h0, h1 = p.download(u0), p.download(u1)
        p.run_wave(u0, u1, 4)
        torch.cuda.synchronize()
        op, ou = oracle.wave(h0, h1, -1.0, r, c, 4)
        assert norm_err(p.download(u1), ou, r) <= 4 * TOL["f32"]
