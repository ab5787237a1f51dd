"""GPU parity of the per-axis symmetric stencil (stencil_plan_create_axes,
reading R3b) against ``oracle.sweep_axes``: ragged grids, every radius, both
dtypes, in-plane and forward-plane kernels; bit-exact on integer fields; all
configurations bit-identical to each other (one fixed order, common.cuh)."""
import numpy as np
import pytest

import oracle
import stencil_inputs as si
from test_parity_gpu import TOL, rel_err, shell_equal

pytestmark = pytest.mark.gpu

R_ALL = [1, 2, 3, 4, 5, 6]


@pytest.fixture(scope="module")
def S():
    import torch  # noqa: F401
    import paper_conf_ipps_tangtkwkgtw13_b200 as pkg
    return pkg


def run(S, u, r, c, dtype, iters, cfg=None):
    nz, ny, nx = (d - 2 * r for d in u.shape)
    with S.Plan(nx, ny, nz, r, c, dtype) as p:
        assert p.axes
        if cfg:
            p.set_config(**cfg)
        a = p.upload(u)
        b = p.alloc()
        p.run(a, b, iters)
        out = p.download(b)
    return out


def cfgs(dtype, r):
    vec = 4 if dtype == "f32" else 2
    ry = 1 if (dtype == "f64" and r >= 5) else 2   # register budget of the per-axis tiles (kern_inst.cuh)
    out = [dict(kernel="inplane", tx=16, ty=4, rx=vec, ry=ry, stages=3, zsegs=2, zbox=2),
           dict(kernel="inplane", tx=32, ty=2, rx=vec, ry=1, stages=4, zsegs=1, zbox=1),
           dict(kernel="inplane", tx=16, ty=3, rx=vec, ry=ry, stages=3, zsegs=3, zbox=2, ytiles=5 if ry == 2 else 8),
           dict(kernel="forward", tx=32, ty=8, rx=1, ry=1, stages=1, zsegs=1)]
    if r <= 4:
        out.append(dict(kernel="inplane", tx=16, ty=2, rx=2 * vec, ry=1, stages=2, zsegs=1, zbox=3))
    return out


@pytest.mark.parametrize("dtype", ["f32", "f64"])
@pytest.mark.parametrize("r", R_ALL)
def test_axes_random_field_10_iterations(S, r, dtype):
    nx, ny, nz = 37, 23, 19 + 2 * r
    u = si.uniform(nx, ny, nz, r, seed=100 + r, dtype=dtype)
    c = si.coeffs_axes("heat_axes", r, dtype)
    o = oracle.sweep_axes(u, r, c, 10)
    outs = []
    for cfg in cfgs(dtype, r):
        g = run(S, u, r, c, dtype, 10, cfg)
        assert shell_equal(g, u, r)
        assert rel_err(g, o, r) <= TOL[dtype], cfg
        outs.append(g)
    for g in outs[1:]:
        assert np.array_equal(g, outs[0])   # one fixed per-point order for every kernel / tile


@pytest.mark.parametrize("dtype", ["f32", "f64"])
@pytest.mark.parametrize("r", [1, 2, 4, 6])
def test_axes_integer_field_bit_exact(S, r, dtype):
    nx, ny, nz = 29, 18, 13 + 2 * r
    u = si.integers(nx, ny, nz, r, seed=7 * r, lo=-8, hi=8, dtype=dtype)
    c = si.coeffs_axes("int_axes", r, dtype)
    o = oracle.sweep_axes(u, r, c, 2)
    assert np.max(np.abs(o)) < 2 ** 24   # every partial sum exact in fp32
    for cfg in cfgs(dtype, r):
        g = run(S, u, r, c, dtype, 2, cfg)
        assert np.array_equal(g.astype(np.float64), o), cfg


def test_axes_tune_and_default_config(S):
    r, dtype = 4, "f32"
    nx, ny, nz = 96, 80, 40
    u = si.uniform(nx, ny, nz, r, seed=5, dtype=dtype)
    c = si.coeffs_axes("heat_axes", r, dtype)
    o = oracle.sweep_axes(u, r, c, 3)
    with S.Plan(nx, ny, nz, r, c, dtype) as p:
        a = p.upload(u)
        b = p.alloc()
        p.run(a, b, 3)                      # default (model-chosen) configuration
        assert rel_err(p.download(b), o, r) <= TOL[dtype]
        s0, s1 = p.alloc(), p.alloc()
        p.tune(kernel="inplane", model="b200", beta=10, iters_per_rep=2, reps=2, scratch=(s0, s1))
        a = p.upload(u)
        p.run(a, b, 3)
        assert rel_err(p.download(b), o, r) <= TOL[dtype]


def test_axes_rejects_wrong_coefficient_count(S):
    with pytest.raises(ValueError):
        S.Plan(16, 16, 16, 2, [0.5, 0.1, 0.1, 0.1], "f32")   # neither r+1 nor 1+3r
