"""GPU parity of the Div / Grad application stencils (Table V; reading R19) through the C
ABI (stencil_plan_create_divgrad, stencil_run_div, stencil_run_grad) against oracle.div / oracle.grad.

Integer fields with integer-scaled weights are compared bit for bit (every partial sum exact).  Random
fields: the outputs are signed differences that cancel, so the gate is the forward-error bound of the
fixed-order evaluation, pointwise: |g - o| <= (gamma_n(dtype) + gamma_n(fp64)) * sum_m |a_m| (|f[+m]| +
|f[-m]|) summed over the differenced grids, n = 6r + 1 roundings (reading R19), plus the
north-star tolerance normwise.  All configurations agree bit for bit."""
import numpy as np
import pytest

import oracle
import stencil_inputs as si

pytestmark = pytest.mark.gpu
TOL = {"f32": 1e-5, "f64": 1e-12}
EPS = {"f32": 2.0 ** -24, "f64": 2.0 ** -53}


@pytest.fixture(scope="module")
def S():
    import torch  # noqa: F401
    import paper_conf_ipps_tangtkwkgtw13_b200 as pkg
    return pkg


def cfgs(dtype, r):
    vec = 4 if dtype == "f32" else 2
    return [None,
            dict(kernel="inplane_ws", tx=16, ty=8, rx=vec, ry=2, stages=3, zsegs=2, zbox=2),
            dict(kernel="inplane_ws", tx=32, ty=8, rx=vec, ry=4, stages=2, zsegs=3, zbox=2),
            dict(kernel="inplane_ws", tx=32, ty=4, rx=vec, ry=2, stages=2, zsegs=1, zbox=2, ytiles=9)]


def absum(x, axis, r, a):
    """sum_m |a_m| (|x[+m]| + |x[-m]|) along one axis of an outer array (interior points; 0 elsewhere)"""
    x = np.abs(x.astype(np.float64))
    out = np.zeros_like(x)
    n = x.shape[axis]
    I = [slice(r, -r)] * 3
    for m in range(1, r + 1):
        hi, lo = list(I), list(I)
        hi[axis] = slice(r + m, n - r + m)
        lo[axis] = slice(r - m, n - r - m)
        out[tuple(I)] += abs(a[m - 1]) * (x[tuple(hi)] + x[tuple(lo)])
    return out


def bound(dtype, r, terms):
    n = 6 * r + 1
    gam = n * EPS[dtype] / (1 - n * EPS[dtype]) + n * EPS["f64"] / (1 - n * EPS["f64"])
    return gam * terms


def run_div(S, u, v, w, r, a, dtype, cfg):
    nz, ny, nx = (d - 2 * r for d in u.shape)
    with S.DivGrad(nx, ny, nz, r, a, dtype, app="div") as p:
        if cfg:
            p.set_config(**cfg)
        gu, gv, gw = p.upload(u), p.upload(v), p.upload(w)
        o = p.upload(np.full(u.shape, 7.0, dtype=u.dtype))      # sentinel shell
        p.div(gu, gv, gw, o)
        return p.download(o)


def run_grad(S, f, r, a, dtype, cfg):
    nz, ny, nx = (d - 2 * r for d in f.shape)
    with S.DivGrad(nx, ny, nz, r, a, dtype, app="grad") as p:
        if cfg:
            p.set_config(**cfg)
        gf = p.upload(f)
        outs = [p.upload(np.full(f.shape, 7.0, dtype=f.dtype)) for _ in range(3)]
        p.grad(gf, *outs)
        return [p.download(t) for t in outs]


def shell_is(x, r, val):
    m = np.ones(x.shape, bool)
    m[r:-r, r:-r, r:-r] = False
    return np.all(x[m] == val)


@pytest.mark.parametrize("dtype", ["f32", "f64"])
@pytest.mark.parametrize("r", [1, 2, 3, 4])
def test_div_integer_bit_exact(S, r, dtype):
    _, a = si.fd1_int(r)
    nx, ny, nz = 150, 70, 13 + 2 * r
    u, v, w = (si.integers(nx, ny, nz, r, seed=s + r, dtype=dtype) for s in (11, 22, 33))
    o = oracle.div(u, v, w, r, a)
    outs = []
    for cfg in cfgs(dtype, r):
        g = run_div(S, u, v, w, r, a, dtype, cfg)
        I = (slice(r, -r),) * 3
        assert np.array_equal(g[I].astype(np.float64), o[I]), cfg
        assert shell_is(g, r, 7.0), cfg
        outs.append(g)


@pytest.mark.parametrize("dtype", ["f32", "f64"])
@pytest.mark.parametrize("r", [1, 2, 3, 4])
def test_grad_integer_bit_exact(S, r, dtype):
    _, a = si.fd1_int(r)
    nx, ny, nz = 150, 70, 13 + 2 * r
    f = si.integers(nx, ny, nz, r, seed=44 + r, dtype=dtype)
    want = oracle.grad(f, r, a)
    I = (slice(r, -r),) * 3
    for cfg in cfgs(dtype, r):
        got = run_grad(S, f, r, a, dtype, cfg)
        for g, o in zip(got, want):
            assert np.array_equal(g[I].astype(np.float64), o[I]), cfg
            assert shell_is(g, r, 7.0), cfg


@pytest.mark.parametrize("dtype", ["f32", "f64"])
@pytest.mark.parametrize("r", [1, 2, 4])
def test_div_random_error_bound(S, r, dtype):
    a = [float(np.array(float(x), dtype=si.DTYPES[dtype])) for x in si.fd1_weights(r)]
    nx, ny, nz = 37, 23, 17 + 2 * r
    u, v, w = (si.uniform(nx, ny, nz, r, seed=s + r, dtype=dtype) for s in (5, 6, 7))
    o = oracle.div(u, v, w, r, a)
    B = bound(dtype, r, absum(u, 2, r, a) + absum(v, 1, r, a) + absum(w, 0, r, a))
    I = (slice(r, -r),) * 3
    ref = None
    for cfg in cfgs(dtype, r):
        g = run_div(S, u, v, w, r, a, dtype, cfg).astype(np.float64)
        err = np.abs(g[I] - o[I])
        assert np.all(err <= B[I]), (cfg, float(np.max(err / np.maximum(B[I], 1e-300))))
        assert np.max(err) / np.max(np.abs(o[I])) <= TOL[dtype], cfg
        if ref is None:
            ref = g
        assert np.array_equal(g[I], ref[I]), "configurations must agree bit for bit"


@pytest.mark.parametrize("dtype", ["f32", "f64"])
@pytest.mark.parametrize("r", [1, 3, 4])
def test_grad_random_error_bound(S, r, dtype):
    a = [float(np.array(float(x), dtype=si.DTYPES[dtype])) for x in si.fd1_weights(r)]
    nx, ny, nz = 41, 29, 15 + 2 * r
    f = si.uniform(nx, ny, nz, r, seed=70 + r, dtype=dtype)
    want = oracle.grad(f, r, a)
    I = (slice(r, -r),) * 3
    refs = None
    for cfg in cfgs(dtype, r):
        got = [g.astype(np.float64) for g in run_grad(S, f, r, a, dtype, cfg)]
        for axis, g, o in zip((2, 1, 0), got, want):
            B = bound(dtype, r, absum(f, axis, r, a))
            err = np.abs(g[I] - o[I])
            assert np.all(err <= B[I]), (cfg, axis)
            assert np.max(err) / np.max(np.abs(o[I])) <= TOL[dtype], (cfg, axis)
        if refs is None:
            refs = got
        assert all(np.array_equal(x[I], y[I]) for x, y in zip(got, refs))


def test_divgrad_validation(S):
    with pytest.raises(S.StencilError):
        S.DivGrad(16, 16, 16, 5, [0.1] * 5, "f32", app="div")
    with S.DivGrad(16, 16, 16, 1, [0.5], "f32", app="grad") as p:
        f = p.alloc()
        with pytest.raises(S.StencilError):
            p.grad(f, f, p.alloc(), p.alloc())        # output aliases the input
        with pytest.raises(S.StencilError):
            p.div(f, f, f, p.alloc())                 # a Grad plan
