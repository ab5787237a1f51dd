"""Seeded synthetic inputs shared by the oracle tests and the CUDA path.

This module holds NO stencil arithmetic: it only draws fields and names
coefficient sets.  Both sides (``oracle/`` and the CUDA library) consume what
it returns; neither side's results ever flow back into it.

Input recipe:
  * fields live on the OUTER grid (nz+2r, ny+2r, nx+2r), x fastest, shell
    included (the shell is the frozen Dirichlet boundary);
  * ``uniform``  : i.i.d. U[0,1) drawn with numpy PCG64(seed) in float64, then
                   rounded once to the target dtype (the paper is silent on the
                   data; SURVEY reading 9);
  * ``integers`` : i.i.d. integers in [lo, hi] (bit-exactness fields);
  * ``counter``  : splitmix64(seed, global linear index) -> U[0,1) with 24
                   (f32) / 53 (f64) random bits, so any z-slab decomposition sees
                   the same global field;
  * coefficient sets c0..cr (isotropic, Eq. 1): "avg", "heat", "dyadic",
    "laplace_int", "fd" (see ``coeffs``).
"""
from __future__ import annotations

from fractions import Fraction
from math import factorial

import numpy as np

DTYPES = {"f32": np.float32, "f64": np.float64}


def outer_shape(nx: int, ny: int, nz: int, r: int):
    return (nz + 2 * r, ny + 2 * r, nx + 2 * r)


def uniform(nx: int, ny: int, nz: int, r: int, seed: int, dtype="f32") -> np.ndarray:
    """U[0,1) on the outer grid (PCG64), rounded to ``dtype``."""
    g = np.random.Generator(np.random.PCG64(seed))
    a = g.random(outer_shape(nx, ny, nz, r), dtype=np.float64)
    return a.astype(DTYPES[dtype])


def integers(nx: int, ny: int, nz: int, r: int, seed: int, lo=-8, hi=8, dtype="f32") -> np.ndarray:
    """Integer-valued field in [lo, hi] on the outer grid."""
    g = np.random.Generator(np.random.PCG64(seed))
    a = g.integers(lo, hi + 1, size=outer_shape(nx, ny, nz, r))
    return a.astype(DTYPES[dtype])


_M64 = (1 << 64) - 1


def splitmix64(x: np.ndarray) -> np.ndarray:
    """splitmix64 finaliser on uint64 arrays (wrapping arithmetic)."""
    x = (x + np.uint64(0x9E3779B97F4A7C15)) & np.uint64(_M64)
    x = ((x ^ (x >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)) & np.uint64(_M64)
    x = ((x ^ (x >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)) & np.uint64(_M64)
    return x ^ (x >> np.uint64(31))


def counter(nx: int, ny: int, nz: int, r: int, seed: int, dtype="f32", z0: int = 0, nz_global: int | None = None) -> np.ndarray:
    """Counter-based U[0,1) field.

    The value at GLOBAL outer point (i, j, kg) is
    ``splitmix64(seed * 2**40 + (kg*(ny+2r) + j)*(nx+2r) + i)`` keeping the top
    24 (f32) or 53 (f64) bits.  ``z0`` selects outer planes [z0, z0+nz+2r) of a
    global grid (for slab decompositions); the default is the whole grid.
    """
    return counter_block(nx, ny, r, seed, dtype, (z0, z0 + nz + 2 * r), (0, ny + 2 * r), (0, nx + 2 * r))


def counter_block(nx: int, ny: int, r: int, seed: int, dtype, ks, js, is_) -> np.ndarray:
    """The block [ks[0], ks[1]) x [js[0], js[1]) x [is_[0], is_[1]) of GLOBAL outer indices of the
    counter field of an nx x ny (x any nz) grid -- the same values ``counter`` gives there, without
    materialising the whole grid (sampled checks at BASELINE configs[4] size)."""
    with np.errstate(over="ignore"):
        px, py = nx + 2 * r, ny + 2 * r
        k = np.arange(ks[0], ks[1], dtype=np.uint64)[:, None, None]
        j = np.arange(js[0], js[1], dtype=np.uint64)[None, :, None]
        i = np.arange(is_[0], is_[1], dtype=np.uint64)[None, None, :]
        lin = (k * np.uint64(py) + j) * np.uint64(px) + i
        h = splitmix64(lin + np.uint64((seed << 40) & _M64))
        if dtype == "f32":
            return ((h >> np.uint64(40)).astype(np.float64) * 2.0 ** -24).astype(np.float32)
        return (h >> np.uint64(11)).astype(np.float64) * 2.0 ** -53


def fd_weights(r: int):
    """Central 1-D second-derivative weights of order 2r (exact Fractions).

    a_m = 2(-1)^(m+1) (r!)^2 / (m^2 (r-m)! (r+m)!),  a_0 = -2 sum a_m.
    """
    a = [Fraction(0)] * (r + 1)
    for m in range(1, r + 1):
        a[m] = Fraction(2 * (-1) ** (m + 1) * factorial(r) ** 2,
                        m * m * factorial(r - m) * factorial(r + m))
    a[0] = -2 * sum(a[1:])
    return a


def fd1_weights(r: int):
    """Central 1-D first-derivative weights of order 2r (exact Fractions), h = 1:
    f'(x) ~ sum_m a_m (f(x+m) - f(x-m)),  a_m = (-1)^(m+1) (r!)^2 / (m (r-m)! (r+m)!)
    (r = 1: 1/2; r = 2: 2/3, -1/12).  Returns [a_1, ..., a_r]."""
    return [Fraction((-1) ** (m + 1) * factorial(r) ** 2, m * factorial(r - m) * factorial(r + m))
            for m in range(1, r + 1)]


def fd1_int(r: int):
    """fd1_weights scaled to the smallest integers (scale, [a_1..a_r] * scale): exact in any FP format."""
    a = fd1_weights(r)
    from math import lcm
    s = 1
    for x in a:
        s = lcm(s, x.denominator)
    return s, [int(x * s) for x in a]


_INT_SCALE = {1: 1, 2: 12, 3: 180, 4: 5040, 5: 25200, 6: 831600}


def coeffs(kind: str, r: int):
    """Coefficient set c0..cr as a list of Fractions / ints.

    avg         c0 = 1/4, c_m = 1/(8r)          (weight sum 1)
    dyadic      c0 = 1/4, rest dyadic, weight sum 1 (exact in binary FP)
    heat        u + alpha*Lap_h u, alpha = 1/16  (weight sum 1; order-2r FD)
    laplace_int S * (3 a_0, a_1..a_r), S = 1,12,180,5040,25200,831600 (integer 3-D Laplacian)
    fd          (3 a_0, a_1..a_r) exactly (3-D Laplacian, Fractions)
    """
    if kind == "avg":
        return [Fraction(1, 4)] + [Fraction(1, 8 * r)] * r
    if kind == "dyadic":
        table = {
            1: [Fraction(1, 4), Fraction(1, 8)],
            2: [Fraction(1, 4), Fraction(1, 16), Fraction(1, 16)],
            3: [Fraction(1, 4), Fraction(1, 16), Fraction(1, 32), Fraction(1, 32)],
            4: [Fraction(1, 4), Fraction(1, 16), Fraction(1, 32), Fraction(1, 64), Fraction(1, 64)],
            5: [Fraction(1, 4), Fraction(1, 16), Fraction(1, 32), Fraction(1, 64), Fraction(1, 128), Fraction(1, 128)],
            6: [Fraction(1, 4), Fraction(1, 16), Fraction(1, 32), Fraction(1, 64), Fraction(1, 128), Fraction(1, 256),
                Fraction(1, 256)],
        }
        return table[r]
    a = fd_weights(r)
    if kind == "heat":
        al = Fraction(1, 16)
        return [1 + 3 * al * a[0]] + [al * a[m] for m in range(1, r + 1)]
    if kind == "fd":
        return [3 * a[0]] + a[1:]
    if kind == "laplace_int":
        S = _INT_SCALE[r]
        out = [3 * a[0] * S] + [a[m] * S for m in range(1, r + 1)]
        assert all(x.denominator == 1 for x in out)
        return [int(x) for x in out]
    raise ValueError(f"unknown coefficient set {kind!r}")


def coeffs_as(kind: str, r: int, dtype="f64") -> np.ndarray:
    """Coefficients rounded to ``dtype`` (what the GPU sees), returned as float64."""
    c = np.array([float(x) for x in coeffs(kind, r)], dtype=np.float64)
    return c.astype(DTYPES[dtype]).astype(np.float64)


def coeffs_axes(kind: str, r: int, dtype="f64") -> np.ndarray:
    """Per-axis coefficient set (1 + 3r values c0, cx_1..cx_r, cy_1..cy_r, cz_1..cz_r;
    DESIGN.md reading R3b), rounded to ``dtype`` and returned as float64.

    heat_axes  anisotropic diffusion u + sum_d alpha_d D2_d u with order-2r FD
               weights and alpha = (1/16, 1/24, 1/40) (weight sum 1)
    int_axes   small distinct integers per axis (exact integer arithmetic)
    """
    if kind == "heat_axes":
        a = fd_weights(r)
        al = (Fraction(1, 16), Fraction(1, 24), Fraction(1, 40))
        c = [1 + sum(al) * a[0]] + [al[d] * a[m] for d in range(3) for m in range(1, r + 1)]
    elif kind == "int_axes":
        tab = ((3, -2, 1, -1, 2, 1), (-1, 2, 2, 1, -1, -2), (2, 1, -3, 2, 1, -1))   # x, y, z; distinct at every m
        c = [-1] + [tab[d][m - 1] for d in range(3) for m in range(1, r + 1)]
    else:
        raise ValueError(f"unknown per-axis coefficient set {kind!r}")
    v = np.array([float(x) for x in c], dtype=np.float64)
    return v.astype(DTYPES[dtype]).astype(np.float64)


# BASELINE.json configs (shapes / recipes); the bench workload is C2.
CONFIGS = {
    "c1": dict(nx=64, ny=64, nz=64, r=1, dtype="f32", iters=10, coeffs="heat", seed=1),
    "c2": dict(nx=512, ny=512, nz=512, r=4, dtype="f32", iters=100, coeffs="heat", seed=2),
    "c3": dict(nx=512, ny=512, nz=512, r=4, dtype="f64", iters=100, coeffs="heat", seed=3),
    "c5": dict(nx=2048, ny=2048, nz=1024, r=4, dtype="f32", iters=100, coeffs="heat", seed=5),
}
