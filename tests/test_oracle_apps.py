"""Pins for the application-stencil oracles (oracle.source, oracle.wave) -- CPU only.

Sec. V / Table V names the application stencils and their grid
counts ("Poisson": 2 inputs, 1 output) and BASELINE config 3 asks for a "3D
wave" kernel; the paper prints no formulas, so the oracle states the plain
definitions (reading R19):

    source:  u_{t+1} = S(u_t) + d f        (Jacobi iteration of the FD Poisson equation)
    wave:    u_{n+1} = S(u_n) + d u_{n-1}  (leapfrog; d = -1)

Pinned here by what the mathematics fixes:
  * the exact FD Poisson solution is a fixed point of one sweep, and the
    iteration converges to it from zero (c, d and f placement; the loop);
  * impulses in f give d at the point, then c_m d around it (term placement);
  * leapfrog on a Dirichlet eigenvector follows the scalar three-term
    recurrence a_{n+1} = (2 + k lam) a_n - a_{n-1}, i.e. cos(n phi) (loop,
    rotation, sign of d), for 1..7 steps;
  * one leapfrog step of a sine mode gives (lam_S cos(phi) - 1) f for r = 1..6.
"""
import math
from fractions import Fraction

import numpy as np
import pytest

import oracle
import stencil_inputs as si

R_ALL = [1, 2, 3, 4, 5, 6]


def grid(n, r):
    return np.meshgrid(np.arange(n[2] + 2 * r), np.arange(n[1] + 2 * r), np.arange(n[0] + 2 * r), indexing="ij")


def jacobi_coeffs(r):
    """Jacobi for Lap_h u = f with the order-2r FD Laplacian (h = 1):
    u = (f - sum_m a_m (six neighbours)) / (3 a_0)  ->  c0 = 0, c_m = -a_m/(3a_0), d = 1/(3a_0)."""
    a = si.fd_weights(r)
    w0 = 3 * a[0]
    return [0.0] + [float(-a[m] / w0) for m in range(1, r + 1)], float(1 / w0)


@pytest.mark.parametrize("r", R_ALL)
def test_poisson_exact_solution_is_a_fixed_point(r):
    # p of degree <= 2r+1 is differentiated exactly by the order-2r FD Laplacian, so u* = p solves
    # Lap_h u = Lap p with u* on the shell, and one Jacobi sweep must return it
    n = (7, 6, 5)
    K, J, I = grid(n, r)
    X, Y, Z = (I - 3.5) / 4, (J - 2.0) / 4, (K - 2.5) / 4
    d3 = min(3, 2 * r + 1)
    p = X ** d3 + 2 * Y ** 2 - 3 * Z ** d3 + X * Y
    # Lap p in grid units (h = 1): x = (i - 3.5)/4 -> d2/di2 = (1/16) d2/dx2
    lap = (d3 * (d3 - 1) * X ** (d3 - 2) + 4 - 3 * d3 * (d3 - 1) * Z ** (d3 - 2)) / 16.0
    c, d = jacobi_coeffs(r)
    out = oracle.source(p, lap, d, r, c, 1)
    assert np.max(np.abs(out - p)) < 1e-13 * max(1.0, np.max(np.abs(p)))
    # a wrong sign of d, or f ignored, breaks the fixed point
    bad = oracle.source(p, lap, -d, r, c, 1)
    assert np.max(np.abs(bad - p)) > 1e-4


def test_poisson_iteration_converges_to_solution():
    r, n = 1, (6, 5, 7)
    K, J, I = grid(n, r)
    p = 0.3 * I * I - 0.2 * J * K + 0.1 * K
    lap = np.full(p.shape, 0.6)     # Lap p = 2 * 0.3
    c, d = jacobi_coeffs(r)
    u0 = p.copy()
    u0[r:-r, r:-r, r:-r] = 0.0      # boundary values only
    out = oracle.source(u0, lap, d, r, c, 400)
    assert np.max(np.abs(out - p)) < 1e-8
    # the Jacobi error contracts monotonically in this case
    e = [np.max(np.abs(oracle.source(u0, lap, d, r, c, t) - p)) for t in (10, 20, 40)]
    assert e[0] > e[1] > e[2]


@pytest.mark.parametrize("r", [1, 3, 6])
def test_source_impulse(r):
    n = (4 * r + 3,) * 3
    u = np.zeros(si.outer_shape(*n, r))
    f = np.zeros_like(u)
    p = (r + n[2] // 2, r + n[1] // 2, r + n[0] // 2)
    f[p] = 1.0
    c = [Fraction(1, 4)] + [Fraction(1, 2 ** (m + 3)) for m in range(1, r + 1)]
    cf = [float(x) for x in c]
    d = 0.75
    one = oracle.source(u, f, d, r, cf, 1)
    exp = np.zeros_like(u)
    exp[p] = d
    assert np.array_equal(one, exp)
    two = oracle.source(u, f, d, r, cf, 2)   # S(d delta) + d delta
    exp2 = np.zeros_like(u)
    exp2[p] = float(c[0]) * d + d
    k, j, i = p
    for m in range(1, r + 1):
        for dk, dj, di in [(m, 0, 0), (-m, 0, 0), (0, m, 0), (0, -m, 0), (0, 0, m), (0, 0, -m)]:
            exp2[k + dk, j + dj, i + di] = float(c[m]) * d
    assert np.array_equal(two, exp2)


@pytest.mark.parametrize("steps", [1, 2, 3, 7])
def test_wave_dirichlet_mode_follows_recurrence(steps):
    r, n = 1, (12, 10, 14)
    modes = (2, 3, 1)
    K, J, I = grid(n, r)
    f = (np.sin(math.pi * modes[0] * I / (n[0] + 1)) * np.sin(math.pi * modes[1] * J / (n[1] + 1))
         * np.sin(math.pi * modes[2] * K / (n[2] + 1)))
    f[0], f[-1], f[:, 0], f[:, -1], f[:, :, 0], f[:, :, -1] = 0, 0, 0, 0, 0, 0
    kap = 0.1
    lam = -6 + 2 * sum(math.cos(math.pi * m / (nn + 1)) for m, nn in zip(modes, n))   # r=1 Lap_h eigenvalue
    c = [2 + kap * (-6.0), kap]
    phi = math.acos(1 + kap * lam / 2)
    up, u = oracle.wave(f, math.cos(phi) * f, -1.0, r, c, steps)
    assert np.max(np.abs(u - math.cos((steps + 1) * phi) * f)) < 1e-13
    assert np.max(np.abs(up - math.cos(steps * phi) * f)) < 1e-13


@pytest.mark.parametrize("r", R_ALL)
def test_wave_one_step_sine_mode(r):
    n = (13, 11, 9)
    a, b, cz = 0.31, 0.57, 0.83
    K, J, I = grid(n, r)
    f = np.sin(a * I + 0.2) * np.sin(b * J + 0.9) * np.sin(cz * K + 1.7)
    c = [0.37, 0.11, -0.053, 0.029, -0.0171, 0.0093, -0.0047][: r + 1]
    lam = c[0] + 2 * sum(c[m] * (math.cos(m * a) + math.cos(m * b) + math.cos(m * cz)) for m in range(1, r + 1))
    cphi = 0.7
    up, u = oracle.wave(f, cphi * f, -1.0, r, c, 1)
    inner = (slice(r, -r),) * 3
    assert np.max(np.abs(u[inner] - (lam * cphi - 1.0) * f[inner])) < 1e-14
    assert np.array_equal(up, cphi * f)          # the previous state is the old u
    mask = np.ones(f.shape, dtype=bool)
    mask[inner] = False
    assert np.array_equal(u[mask], (cphi * f)[mask])   # frozen shell = u's shell


def test_wave_zero_steps_and_errors():
    u = np.random.default_rng(1).random((7, 7, 7))
    up, uu = oracle.wave(u * 0.5, u, -1.0, 1, [1.0, 0.1], 0)
    assert np.array_equal(up, u * 0.5) and np.array_equal(uu, u)
    with pytest.raises(ValueError):
        oracle.wave(u, u[:-1], -1.0, 1, [1.0, 0.1], 1)
    with pytest.raises(ValueError):
        oracle.source(u, u, 1.0, 1, [1.0, 0.1], -1)
