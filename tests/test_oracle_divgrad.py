"""Pins of oracle.div / oracle.grad (Table V Div 3 -> 1 and Grad 1 -> 3; definitions of
reading R19: order-2r central first derivatives, coefficient a_m on f[+m] - f[-m]) -- CPU only.

Each pin fails for a plausible slip: a swapped axis (sine modes with distinct frequencies per axis), a
sign (impulse response, odd symmetry), a dropped term (polynomial exactness up to degree 2r, failure at
2r+1), a wrong weight (hand-computed points)."""
import json
import os
from fractions import Fraction

import numpy as np
import pytest

import oracle
import stencil_inputs as si

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def coords(n, r):
    """centred integer coordinates of an outer axis of n interior points"""
    return np.arange(n + 2 * r, dtype=np.float64) - (n + 2 * r - 1) // 2


def grid3(f, nx, ny, nz, r):
    z, y, x = np.meshgrid(coords(nz, r), coords(ny, r), coords(nx, r), indexing="ij")
    return f(x, y, z)


@pytest.mark.parametrize("r", [1, 2, 3, 4])
def test_grad_polynomial_exact_to_degree_2r(r):
    S, a = si.fd1_int(r)                      # integer-scaled weights: every value exact in fp64
    n = 9
    I = (slice(r, -r),) * 3
    for d in range(1, 2 * r + 2):
        f = grid3(lambda x, y, z: x ** d + 2 * y ** d + 3 * z ** d, n, n, n, r)
        gx, gy, gz = oracle.grad(f, r, a)
        z, y, x = np.meshgrid(coords(n, r), coords(n, r), coords(n, r), indexing="ij")
        exact = (S * d * x ** (d - 1), S * 2 * d * y ** (d - 1), S * 3 * d * z ** (d - 1))
        ok = all(np.array_equal(g[I], e[I]) for g, e in zip((gx, gy, gz), exact))
        assert ok == (d <= 2 * r), (r, d)


@pytest.mark.parametrize("r", [1, 2, 4])
def test_div_polynomial_exact_to_degree_2r(r):
    S, a = si.fd1_int(r)
    n = 8
    I = (slice(r, -r),) * 3
    for d in range(1, 2 * r + 2):
        u = grid3(lambda x, y, z: x ** d + y * z, n, n, n, r)          # y*z: no x-derivative
        v = grid3(lambda x, y, z: 2 * y ** d + x * z, n, n, n, r)
        w = grid3(lambda x, y, z: 3 * z ** d + x * y, n, n, n, r)
        out = oracle.div(u, v, w, r, a)
        z, y, x = np.meshgrid(coords(n, r), coords(n, r), coords(n, r), indexing="ij")
        exact = S * d * (x ** (d - 1) + 2 * y ** (d - 1) + 3 * z ** (d - 1))
        assert np.array_equal(out[I], exact[I]) == (d <= 2 * r), (r, d)


@pytest.mark.parametrize("r", [1, 3, 4])
def test_grad_sine_modes_per_axis(r):
    """sin(a x) sin(b y) sin(c z), distinct a, b, c: gx = sigma(a) cos(a x) sin(b y) sin(c z) with
    sigma(t) = 2 sum_m a_m sin(m t) (sin(t(x+m)) - sin(t(x-m)) = 2 cos(t x) sin(m t))."""
    a = [float(x) for x in si.fd1_weights(r)]
    sig = lambda t: 2 * sum(am * np.sin((m + 1) * t) for m, am in enumerate(a))
    A, B, C = 0.31, 0.53, 0.77
    n = 11
    f = grid3(lambda x, y, z: np.sin(A * x) * np.sin(B * y) * np.sin(C * z), n, n, n, r)
    gx, gy, gz = oracle.grad(f, r, a)
    I = (slice(r, -r),) * 3
    z, y, x = np.meshgrid(coords(n, r), coords(n, r), coords(n, r), indexing="ij")
    ex = sig(A) * np.cos(A * x) * np.sin(B * y) * np.sin(C * z)
    ey = sig(B) * np.sin(A * x) * np.cos(B * y) * np.sin(C * z)
    ez = sig(C) * np.sin(A * x) * np.sin(B * y) * np.cos(C * z)
    for g, e in ((gx, ex), (gy, ey), (gz, ez)):
        assert np.max(np.abs(g[I] - e[I])) < 1e-13


@pytest.mark.parametrize("r", [1, 2, 4])
def test_div_grad_sine_mode(r):
    """div(grad f) = -(sigma(a)^2 + sigma(b)^2 + sigma(c)^2) f for a sine mode, away from the boundary
    (the oracle's outputs carry a zero shell, so points within 2r of it are excluded)."""
    a = [float(x) for x in si.fd1_weights(r)]
    sig = lambda t: 2 * sum(am * np.sin((m + 1) * t) for m, am in enumerate(a))
    A, B, C = 0.41, 0.23, 0.67
    n = 6 * r + 3
    f = grid3(lambda x, y, z: np.sin(A * x) * np.sin(B * y) * np.sin(C * z), n, n, n, r)
    gx, gy, gz = oracle.grad(f, r, a)
    dd = oracle.div(gx, gy, gz, r, a)
    J = (slice(2 * r, -2 * r),) * 3
    lam = -(sig(A) ** 2 + sig(B) ** 2 + sig(C) ** 2)
    assert np.max(np.abs(dd[J] - lam * f[J])) < 1e-12


def test_grad_impulse_response_and_shell():
    r = 3
    a = [0.7, -0.2, 0.05]
    n = 9
    f = np.zeros((n + 2 * r,) * 3)
    p = (r + 4, r + 4, r + 4)                  # (k, j, i)
    f[p] = 1.0
    gx, gy, gz = oracle.grad(f, r, a)
    for m in range(1, r + 1):
        # gx at q = p + m e_x sees f[q - m] = 1 with weight -a_m; at p - m e_x, f[q + m] with +a_m
        assert gx[p[0], p[1], p[2] + m] == -a[m - 1] and gx[p[0], p[1], p[2] - m] == a[m - 1]
        assert gy[p[0], p[1] + m, p[2]] == -a[m - 1] and gy[p[0], p[1] - m, p[2]] == a[m - 1]
        assert gz[p[0] + m, p[1], p[2]] == -a[m - 1] and gz[p[0] - m, p[1], p[2]] == a[m - 1]
    assert np.count_nonzero(gx) == np.count_nonzero(gy) == np.count_nonzero(gz) == 2 * r
    shell = np.ones(f.shape, bool)
    shell[r:-r, r:-r, r:-r] = False
    assert not gx[shell].any()


def test_divgrad_hand_points():
    with open(os.path.join(GOLDEN, "divgrad_hand.json")) as fh:
        g = json.load(fh)
    for case in g["cases"]:
        r, n = case["r"], case["n"]
        z, y, x = np.meshgrid(*(np.arange(n + 2 * r, dtype=np.float64),) * 3, indexing="ij")
        env = {"i": x, "j": y, "k": z}
        fields = [eval(e, {"np": np}, env) for e in case["fields"]]
        if case["op"] == "grad":
            outs = oracle.grad(fields[0], r, case["a"])
            for (comp, (i, j, k)), v in zip(case["points"], case["values"]):
                assert outs["xyz".index(comp)][k, j, i] == v, (case["name"], comp, (i, j, k))
        else:
            out = oracle.div(*fields, r, case["a"])
            for (i, j, k), v in zip(case["points"], case["values"]):
                assert out[k, j, i] == v, (case["name"], (i, j, k))
