"""Pins for the per-axis oracle ``oracle.sweep_axes`` (reading R3b: "symmetric
per-axis coefficients" of the BASELINE north star, the axis-wise generalisation
of Eq. (1)) -- CPU only.  Each test fixes the result by something other
than the oracle's own formula:

  * impulse response       -> cx_m / cy_m / cz_m land at +-m on THEIR axis only
  * sine-mode eigenvalue   -> lambda = c0 + 2 sum_m (cx_m cos ma + cy_m cos mb + cz_m cos mc),
                              distinct wave numbers and distinct axis sets, so any
                              axis permutation or sign error changes lambda
  * separable product field-> an x-only stencil (cy = cz = 0, c0 = 0) acts on
                              f(x) g(y) h(z) as the 1-D convolution of f, computed by numpy.convolve
  * isotropic special case -> cx = cy = cz reproduces Eq. (1) as oracle.sweep (its own pins)
  * anisotropic diffusion  -> with c0 = 1 - 2 sum(cx+cy+cz) the constant field is
                              exact and a linear ramp along any axis is preserved
"""
import itertools
import math

import numpy as np
import pytest

import oracle

R_ALL = [1, 2, 3, 4, 5, 6]


def axes_coeffs(r):
    c0 = 0.31
    cx = [0.113, -0.041, 0.0217, -0.0093, 0.0051, -0.0027][:r]
    cy = [0.077, 0.0333, -0.0149, 0.0071, -0.0039, 0.0013][:r]
    cz = [-0.059, 0.0251, 0.0117, -0.0063, 0.0029, 0.0017][:r]
    return c0, cx, cy, cz


def pack(c0, cx, cy, cz):
    return [c0, *cx, *cy, *cz]


@pytest.mark.parametrize("r", R_ALL)
def test_axes_impulse_response(r):
    n = 4 * r + 3
    u = np.zeros((n + 2 * r,) * 3)
    p = r + n // 2
    u[p, p, p] = 1.0
    c0, cx, cy, cz = axes_coeffs(r)
    out = oracle.sweep_axes(u, r, pack(c0, cx, cy, cz), 1)
    want = np.zeros_like(u)
    want[p, p, p] = c0
    for m in range(1, r + 1):
        for s in (-1, 1):
            want[p, p, p + s * m] = cx[m - 1]      # x is the last (fastest) array axis
            want[p, p + s * m, p] = cy[m - 1]
            want[p + s * m, p, p] = cz[m - 1]
    assert np.array_equal(out, want)


@pytest.mark.parametrize("r", R_ALL)
def test_axes_sine_mode_eigenvalue(r):
    nx, ny, nz = 13, 11, 9
    a, b, c = 0.31, 0.57, 0.83
    K, J, I = np.meshgrid(np.arange(nz + 2 * r), np.arange(ny + 2 * r), np.arange(nx + 2 * r), indexing="ij")
    f = np.sin(a * I + 0.2) * np.sin(b * J + 0.9) * np.sin(c * K + 1.7)
    c0, cx, cy, cz = axes_coeffs(r)
    lam = c0 + 2 * sum(cx[m - 1] * math.cos(m * a) + cy[m - 1] * math.cos(m * b) + cz[m - 1] * math.cos(m * c)
                       for m in range(1, r + 1))
    out = oracle.sweep_axes(f, r, pack(c0, cx, cy, cz), 1)
    inner = (slice(r, -r),) * 3
    assert np.max(np.abs(out[inner] - lam * f[inner])) < 1e-14
    # a permuted axis assignment gives a different eigenvalue (so the test can fail)
    for perm in itertools.permutations((a, b, c)):
        if perm == (a, b, c):
            continue
        lam_p = c0 + 2 * sum(cx[m - 1] * math.cos(m * perm[0]) + cy[m - 1] * math.cos(m * perm[1])
                             + cz[m - 1] * math.cos(m * perm[2]) for m in range(1, r + 1))
        assert abs(lam_p - lam) > 1e-6


@pytest.mark.parametrize("r", [1, 3, 6])
def test_axes_x_only_is_1d_convolution(r):
    nx, ny, nz = 17, 6, 5
    rng = np.random.default_rng(7 + r)
    fx = rng.standard_normal(nx + 2 * r)
    gy = rng.standard_normal(ny + 2 * r)
    hz = rng.standard_normal(nz + 2 * r)
    u = hz[:, None, None] * gy[None, :, None] * fx[None, None, :]
    cx = list(rng.uniform(-1, 1, r))
    kern = np.array(cx[::-1] + [0.0] + cx)                  # symmetric taps, centre 0
    conv = np.convolve(fx, kern, mode="valid")              # length nx
    out = oracle.sweep_axes(u, r, pack(0.0, cx, [0.0] * r, [0.0] * r), 1)
    want = hz[r:-r, None, None] * gy[None, r:-r, None] * conv[None, None, :]
    assert np.max(np.abs(out[r:-r, r:-r, r:-r] - want)) < 1e-12


@pytest.mark.parametrize("r", [1, 2, 4])
def test_axes_isotropic_special_case(r):
    rng = np.random.default_rng(r)
    u = rng.uniform(0, 1, (9 + 2 * r, 8 + 2 * r, 11 + 2 * r))
    c = [0.4] + list(rng.uniform(0, 0.1, r))
    iso = oracle.sweep(u, r, c, 3)
    ax = oracle.sweep_axes(u, r, [c[0]] + c[1:] * 3, 3)
    assert np.max(np.abs(iso - ax)) < 1e-13   # same sum, different association (rounding only)


@pytest.mark.parametrize("r", [1, 4])
def test_axes_constant_and_ramps(r):
    _, cx, cy, cz = axes_coeffs(r)
    c0 = 1.0 - 2.0 * (sum(cx) + sum(cy) + sum(cz))
    c = pack(c0, cx, cy, cz)
    shape = (7 + 2 * r, 8 + 2 * r, 9 + 2 * r)
    out = oracle.sweep_axes(np.full(shape, 2.5), r, c, 4)
    assert np.max(np.abs(out - 2.5)) < 1e-13
    K, J, I = np.meshgrid(*(np.arange(s, dtype=float) for s in shape), indexing="ij")
    for ramp in (I, J, K, 0.5 * I - 2 * J + 3 * K):
        out = oracle.sweep_axes(ramp, r, c, 2)
        assert np.max(np.abs(out - ramp)) < 1e-11


def test_axes_rejects_bad_coefficients():
    with pytest.raises(ValueError):
        oracle.sweep_axes(np.zeros((5, 5, 5)), 1, [1.0, 0.1], 1)
