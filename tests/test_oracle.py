"""Pins for the CPU oracle (oracle/stencil_oracle.c) -- CPU only.

Each test checks the oracle against something the paper or mathematics fixes,
not against a retyped copy of its own formula (PAPER.md = P:L<n>):

  * impulse response            -> coefficient placement per axis and offset (Eq. 1)
  * sine-mode eigenvalues       -> per-axis neighbour handling, signs, offsets
  * Dirichlet eigenvectors      -> iteration loop, ping-pong and frozen shell (Fig. 1)
  * constant / linear fields    -> weight handling, shell semantics
  * FD polynomial reproduction  -> order-2r accuracy of the Laplacian weights; fails at 2r+2
  * in-plane schedule simulator -> the paper's Eqs. (3)-(5) steps 1-6 == Eq. (1)
  * golden hand-computed points -> tests/golden/hand_points.json
"""
import json
import math
import os
from fractions import Fraction

import numpy as np
import pytest

import oracle
from oracle.inplane_sim import inplane_sweeps
import stencil_inputs as si

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def distinct_coeffs(r):
    # distinct, non-dyadic-related values so that a misplaced term shows up
    return [0.37, 0.11, -0.053, 0.029, -0.0171, 0.0093, -0.0047][: r + 1]


R_ALL = [1, 2, 3, 4, 5, 6]   # orders 2..12 (Table I / Table IV)


@pytest.mark.parametrize("r", R_ALL)
def test_impulse_one_iteration(r):
    nx, ny, nz = 3 * r + 5, 3 * r + 4, 3 * r + 6
    u = np.zeros(si.outer_shape(nx, ny, nz, r))
    p = (r + nz // 2, r + ny // 2, r + nx // 2)  # outer (k, j, i)
    u[p] = 1.0
    c = distinct_coeffs(r)
    out = oracle.sweep(u, r, c, 1)
    exp = np.zeros_like(u)
    exp[p] = c[0]
    k, j, i = p
    for m in range(1, r + 1):
        for dk, dj, di in [(m, 0, 0), (-m, 0, 0), (0, m, 0), (0, -m, 0), (0, 0, m), (0, 0, -m)]:
            exp[k + dk, j + dj, i + di] = c[m]
    # interior cells only get values; the shell (zero here) stays zero
    assert np.array_equal(out, exp)


@pytest.mark.parametrize("r", R_ALL)
def test_impulse_two_iterations_centre(r):
    nx = ny = nz = 4 * r + 3
    u = np.zeros(si.outer_shape(nx, ny, nz, r))
    p = (r + nz // 2, r + ny // 2, r + nx // 2)
    u[p] = 1.0
    c = [Fraction(1, 4)] + [Fraction(1, 2 ** (m + 3)) for m in range(1, r + 1)]  # dyadic: exact
    out = oracle.sweep(u, r, [float(x) for x in c], 2)
    # (S^2 delta)(p) = c0^2 + sum over the 6r neighbours of c_m^2
    exp = c[0] ** 2 + 6 * sum(x * x for x in c[1:])
    assert out[p] == float(exp)


@pytest.mark.parametrize("r", R_ALL)
def test_sine_mode_eigenvalue(r):
    nx, ny, nz = 13, 11, 9
    a, b, cz = 0.31, 0.57, 0.83
    ph = (0.2, 0.9, 1.7)
    K, J, I = np.meshgrid(np.arange(nz + 2 * r), np.arange(ny + 2 * r), np.arange(nx + 2 * r), indexing="ij")
    f = np.sin(a * I + ph[0]) * np.sin(b * J + ph[1]) * np.sin(cz * K + ph[2])
    c = distinct_coeffs(r)
    lam = c[0] + 2 * sum(c[m] * (math.cos(m * a) + math.cos(m * b) + math.cos(m * cz)) for m in range(1, r + 1))
    out = oracle.sweep(f, r, c, 1)
    inner = (slice(r, -r),) * 3
    assert np.max(np.abs(out[inner] - lam * f[inner])) < 1e-14
    # the shell is frozen
    mask = np.ones_like(f, dtype=bool)
    mask[inner] = False
    assert np.array_equal(out[mask], f[mask])


def test_sine_mode_detects_axis_swap():
    # guard: the per-axis frequencies make a different eigenvalue for a stencil
    # that weights axes differently -- the test above would catch it
    r = 1
    a, b, cz = 0.31, 0.57, 0.83
    lam = 0.37 + 2 * 0.11 * (math.cos(a) + math.cos(b) + math.cos(cz))
    lam_bad = 0.37 + 2 * 0.11 * (2 * math.cos(a) + math.cos(cz))
    assert abs(lam - lam_bad) > 1e-3


@pytest.mark.parametrize("iters", [1, 2, 10])
def test_dirichlet_eigenvector_iterated(iters):
    # r = 1 with a zero shell: f = prod sin(pi p_d x_d / (n_d + 1)) vanishes on
    # the shell and is an eigenvector of the sweep with eigenvalue lam
    r, nx, ny, nz = 1, 12, 10, 14
    p = (2, 3, 1)
    c = [0.4, 0.1]
    K, J, I = np.meshgrid(np.arange(nz + 2), np.arange(ny + 2), np.arange(nx + 2), indexing="ij")
    f = (np.sin(math.pi * p[0] * I / (nx + 1)) * np.sin(math.pi * p[1] * J / (ny + 1))
         * np.sin(math.pi * p[2] * K / (nz + 1)))
    f[0, :, :] = f[-1, :, :] = 0
    f[:, 0, :] = f[:, -1, :] = 0
    f[:, :, 0] = f[:, :, -1] = 0
    lam = c[0] + 2 * c[1] * sum(math.cos(math.pi * pd / (n + 1)) for pd, n in zip(p, (nx, ny, nz)))
    out = oracle.sweep(f, r, c, iters)
    assert np.max(np.abs(out - lam ** iters * f)) < 1e-14 * max(1, iters)


@pytest.mark.parametrize("r", R_ALL)
def test_constant_field_preserved_bitwise(r):
    c = [float(x) for x in si.coeffs("dyadic", r)]
    assert sum(si.coeffs("dyadic", r)[:1]) + 6 * sum(si.coeffs("dyadic", r)[1:]) == 1
    u = np.full(si.outer_shape(9, 7, 8, r), 0.71875)  # 23/32: few mantissa bits, all sums exact
    out = oracle.sweep(u, r, c, 7)
    assert np.array_equal(out, u)


@pytest.mark.parametrize("r", R_ALL)
def test_linear_field(r):
    # odd terms cancel: S(p) = (c0 + 6 sum c_m) * p for p affine
    nx, ny, nz = 7, 6, 5
    K, J, I = np.meshgrid(np.arange(nz + 2 * r), np.arange(ny + 2 * r), np.arange(nx + 2 * r), indexing="ij")
    p = 3.0 + 2.0 * I - 5.0 * J + 7.0 * K
    c = [2.0, 1.0, -3.0, 4.0, 1.0, -2.0, 3.0][: r + 1]
    w = c[0] + 6 * sum(c[1:])
    out = oracle.sweep(p, r, c, 1)
    inner = (slice(r, -r),) * 3
    assert np.array_equal(out[inner], w * p[inner])


@pytest.mark.parametrize("r", R_ALL)
def test_fd_polynomial_reproduction(r):
    # integer-scaled order-2r Laplacian reproduces S*Lap(p) exactly for
    # p = x^d + 2 y^d + 3 z^d, d <= 2r+1, and must fail at d = 2r+2.
    # r <= 4: every value is an integer below 2^53, so "exactly" is bitwise;
    # r = 5, 6: the top degrees exceed 2^53, so exact up to fp64 rounding
    # (1e-13 of the largest term) and the d = 2r+2 miss must be far larger.
    c = [float(x) for x in si.coeffs("laplace_int", r)]
    S = {1: 1, 2: 12, 3: 180, 4: 5040, 5: 25200, 6: 831600}[r]
    n = 5
    ctr = (n + 2 * r - 1) / 2.0
    K, J, I = np.meshgrid(np.arange(n + 2 * r), np.arange(n + 2 * r), np.arange(n + 2 * r), indexing="ij")
    X, Y, Z = I - ctr + 0.5, J - ctr, K - ctr - 0.5   # exact half-integers / integers
    for d in range(0, 2 * r + 3):
        p = X ** d + 2 * Y ** d + 3 * Z ** d
        out = oracle.sweep(p, r, c, 1)
        inner = (slice(r, -r),) * 3
        if d >= 2:
            lap = d * (d - 1) * (X ** (d - 2) + 2 * Y ** (d - 2) + 3 * Z ** (d - 2))
        else:
            lap = np.zeros_like(p)
        if r <= 4:
            ok = np.array_equal(out[inner], S * lap[inner])
        else:
            scale = max(1.0, float(np.max(np.abs(p))) * sum(abs(x) for x in c))
            miss = float(np.max(np.abs(out[inner] - S * lap[inner])))
            ok = miss <= 1e-13 * scale
            if d == 2 * r + 2:
                assert miss > 1e-8 * scale
        if d <= 2 * r + 1:
            assert ok, f"order-{2*r} FD must reproduce degree {d}"
        else:
            assert not ok, f"order-{2*r} FD must NOT reproduce degree {d}"


@pytest.mark.parametrize("r", R_ALL)
def test_inplane_schedule_equals_eq1_on_integers(r):
    # the paper's in-plane steps 1-6 (Eqs. 3-5) must give exactly Eq. (1)
    nx, ny, nz = 5, 4, 6
    u = si.integers(nx, ny, nz, r, seed=100 + r, dtype="f64")
    c = [-3, 1, 2, -1, 1, -2, 1][: r + 1]
    ui = u.astype(np.int64).astype(object)
    sim = inplane_sweeps(ui, r, c, 2)
    out = oracle.sweep(u, r, [float(x) for x in c], 2)
    assert np.array_equal(out, sim.astype(np.float64))


def test_golden_hand_points():
    with open(os.path.join(GOLDEN, "hand_points.json")) as f:
        cases = json.load(f)["cases"]
    assert cases
    for cs in cases:
        r, n = cs["r"], cs["n"]
        K, J, I = np.meshgrid(np.arange(n + 2 * r), np.arange(n + 2 * r), np.arange(n + 2 * r), indexing="ij")
        u = eval(cs["field"], {"i": I, "j": J, "k": K, "np": np})  # noqa: S307 (trusted fixture)
        u = np.asarray(u, dtype=np.float64)
        out = oracle.sweep(u, r, cs["coeffs"], cs["iters"])
        for (i, j, k), v in zip(cs["points_outer_ijk"], cs["values"]):
            assert out[k, j, i] == v, cs["name"]


@pytest.mark.parametrize("iters", [0, 1, 3])
def test_point_matches_sweep(iters):
    r, nx, ny, nz = 2, 11, 9, 13
    u = si.uniform(nx, ny, nz, r, seed=7, dtype="f64")
    c = [float(x) for x in si.coeffs("heat", r)]
    full = oracle.sweep(u, r, c, iters)
    for (i, j, k) in [(0, 0, 0), (nx - 1, ny - 1, nz - 1), (5, 4, 6), (0, 8, 3), (10, 0, 12)]:
        v = oracle.point(u, r, c, iters, i, j, k)
        assert v == full[k + r, j + r, i + r]


def test_iters_zero_and_shell():
    r = 3
    u = si.uniform(6, 5, 7, r, seed=3, dtype="f64")
    c = [float(x) for x in si.coeffs("avg", r)]
    assert np.array_equal(oracle.sweep(u, r, c, 0), u)
    out = oracle.sweep(u, r, c, 4)
    mask = np.ones_like(u, dtype=bool)
    mask[r:-r, r:-r, r:-r] = False
    assert np.array_equal(out[mask], u[mask])


def test_rejects_bad_arguments():
    u = np.zeros((5, 5, 5))
    with pytest.raises(ValueError):
        oracle.sweep(u, 1, [1.0], 1)          # wrong coefficient count
    with pytest.raises(ValueError):
        oracle.sweep(u, 1, [1.0, 0.0], -1)    # negative iterations
    with pytest.raises(ValueError):
        oracle.sweep(np.zeros((2, 2, 2)), 1, [1.0, 0.0], 1)  # smaller than the shell


def test_openmp_threads_do_not_change_result():
    r = 4
    u = si.uniform(20, 18, 22, r, seed=11, dtype="f64")
    c = [float(x) for x in si.coeffs("heat", r)]
    a = oracle.sweep(u, r, c, 3, nthreads=1)
    b = oracle.sweep(u, r, c, 3, nthreads=4)
    assert np.array_equal(a, b)


@pytest.mark.parametrize("check_every", [1, 3, 7])
def test_run_until_closed_form(check_every):
    """Fig. 1 stop criterion (reading R5b) pinned by the Dirichlet eigenvector:
    u_t = lam^t f, so rho_t = |lam|^(t-1) |lam - 1| max|f| and the stop sweep is
    the first check t with rho_t <= tol -- computed here in closed form."""
    r, nx, ny, nz = 1, 10, 9, 11
    c = [0.5, 0.07]
    K, J, I = np.meshgrid(np.arange(nz + 2), np.arange(ny + 2), np.arange(nx + 2), indexing="ij")
    f = np.sin(np.pi * I / (nx + 1)) * np.sin(np.pi * J / (ny + 1)) * np.sin(np.pi * K / (nz + 1))
    f[0, :, :] = f[-1, :, :] = 0
    f[:, 0, :] = f[:, -1, :] = 0
    f[:, :, 0] = f[:, :, -1] = 0
    lam = c[0] + 2 * c[1] * sum(math.cos(math.pi / (n + 1)) for n in (nx, ny, nz))
    M = float(np.max(np.abs(f)))
    tol = 2.5e-3
    t = check_every
    while abs(lam) ** (t - 1) * abs(lam - 1) * M > tol:
        t += check_every
    u, T, res = oracle.run_until(f, r, c, 10_000, tol, check_every)
    assert T == t
    assert abs(res - abs(lam) ** (T - 1) * abs(lam - 1) * M) < 1e-12
    assert np.max(np.abs(u - lam ** T * f)) < 1e-12
    # max_iters caps the loop and the last sweep is always checked
    u, T, res = oracle.run_until(f, r, c, 5, 0.0, 100)
    assert T == 5 and abs(res - abs(lam) ** 4 * abs(lam - 1) * M) < 1e-12


@pytest.mark.parametrize("dtype", ["f32", "f64"])
def test_counter_block_is_a_window_of_counter(dtype):
    """stencil_inputs.counter_block (used for the sampled BASELINE configs[4] checks) returns exactly the
    window of the global counter field, including windows of a slab (z0 > 0)."""
    nx, ny, nz, r, seed = 21, 13, 9, 2, 5
    u = si.counter(nx, ny, nz, r, seed, dtype)
    b = si.counter_block(nx, ny, r, seed, dtype, (3, 8), (2, 10), (5, 19))
    assert np.array_equal(u[3:8, 2:10, 5:19], b)
    s = si.counter(nx, ny, 4, r, seed, dtype, z0=3)
    assert np.array_equal(s, u[3:3 + 4 + 2 * r])


def test_cone_block_reproduces_the_full_grid():
    """The dependency-cone argument of tests/test_c5_gpu.py: the oracle on a block of half-width
    iters * r + r around a point (clipped at the real shell) equals the full-grid oracle there."""
    nx, ny, nz, r, seed, it = 40, 30, 50, 2, 5, 3
    u = si.counter(nx, ny, nz, r, seed, "f32")
    c = si.coeffs_as("heat", r, "f32")
    full = oracle.sweep(u, r, c, it)
    L = it * r
    for (i, j, k) in [(0, 0, 0), (39, 29, 49), (20, 15, 25), (5, 28, 10)]:
        rng_ = [(max(0, q - L), min(n + 2 * r, q + 2 * r + L + 1)) for q, n in ((k, nz), (j, ny), (i, nx))]
        blk = si.counter_block(nx, ny, r, seed, "f32", *rng_)
        o = oracle.point(blk, r, c, it, i - rng_[2][0], j - rng_[1][0], k - rng_[0][0])
        assert o == full[k + r, j + r, i + r]
