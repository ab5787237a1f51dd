"""GPU parity of the Fig. 1 stop criterion (stencil_run_until, reading R5b)
against ``oracle.run_until``.  The stop sweep T is an integer decided by a
floating-point comparison; the tolerance is placed (geometric mean) between
two consecutive oracle check residuals that differ by a factor >= 1.2, far
outside the dtype's rounding of the residual, so both sides must stop at the
same sweep; the field then matches within the north-star tolerance."""
import math

import numpy as np
import pytest

import oracle
import stencil_inputs as si
from test_parity_gpu import TOL, rel_err, shell_equal

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def S():
    import torch  # noqa: F401
    import paper_conf_ipps_tangtkwkgtw13_b200 as pkg
    return pkg


def checks(u, r, c, every, n):
    """oracle residuals at the first n checks"""
    out = []
    for k in range(1, n + 1):
        _, T, res = oracle.run_until(u, r, c, k * every, 0.0, every)
        out.append(res)
    return out


@pytest.mark.parametrize("dtype", ["f32", "f64"])
@pytest.mark.parametrize("r,every,axes", [(1, 3, False), (2, 1, False), (4, 2, False), (2, 3, True)])
def test_run_until_matches_oracle(S, r, every, axes, dtype):
    nx, ny, nz = 21, 14, 11 + 2 * r
    u = si.uniform(nx, ny, nz, r, seed=40 + r, dtype=dtype)
    c = si.coeffs_axes("heat_axes", r, dtype) if axes else si.coeffs_as("heat", r, dtype)
    rho = checks(u, r, c, every, 5)
    assert rho[2] / rho[3] >= 1.2 and rho[3] > 1e-4
    tol = math.sqrt(rho[2] * rho[3])
    want_u, want_T, want_res = oracle.run_until(u, r, c, 1000, tol, every)
    assert want_T == 4 * every
    with S.Plan(nx, ny, nz, r, c, dtype) as p:
        a = p.upload(u)
        b = p.alloc()
        T, res = p.run_until(a, b, 1000, tol, every)
        g = p.download(b)
        assert np.array_equal(p.download(a), u.astype(g.dtype))   # input untouched
    assert T == want_T
    assert abs(res - want_res) <= 1e-3 * want_res
    assert shell_equal(g, u, r)
    assert rel_err(g, want_u, r) <= TOL[dtype]


def test_run_until_caps_and_validates(S):
    r, dtype = 2, "f32"
    nx, ny, nz = 18, 12, 10
    u = si.uniform(nx, ny, nz, r, seed=3, dtype=dtype)
    c = si.coeffs_as("heat", r, dtype)
    want = oracle.sweep(u, r, c, 7)
    with S.Plan(nx, ny, nz, r, c, dtype) as p:
        a, b = p.upload(u), p.alloc()
        T, res = p.run_until(a, b, 7, 0.0, 100)     # tol 0 never met: capped, the last sweep is checked
        assert T == 7 and res > 0
        assert rel_err(p.download(b), want, r) <= TOL[dtype]
        T, res = p.run_until(a, b, 8, 0.0, 4)       # even count: result moved from the scratch grid
        assert T == 8
        assert rel_err(p.download(b), oracle.sweep(u, r, c, 8), r) <= TOL[dtype]
        with pytest.raises(S.StencilError):
            p.run_until(a, b, 0, 1e-3, 1)
        with pytest.raises(S.StencilError):
            p.run_until(a, b, 5, -1.0, 1)


def test_residual_between_grids(S):
    r, dtype = 3, "f64"
    nx, ny, nz = 23, 17, 15
    u = si.uniform(nx, ny, nz, r, seed=8, dtype=dtype)
    v = u.copy()
    v[r + 4, r + 5, r + 6] += 0.75          # interior difference
    v[0, 0, 0] += 100.0                     # shell differences are ignored
    c = si.coeffs_as("heat", r, dtype)
    with S.Plan(nx, ny, nz, r, c, dtype) as p:
        a, b = p.upload(u), p.upload(v)
        assert p.residual_between(a, b) == abs(np.float64(v[r + 4, r + 5, r + 6]) - np.float64(u[r + 4, r + 5, r + 6]))
        assert p.residual_between(a, a) == 0.0
