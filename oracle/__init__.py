"""CPU oracle for the iterative 3D star stencil -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline``
/ ``--impl reference`` legs may import this package.  It shares no code with the
CUDA product path (``paper_conf_ipps_tangtkwkgtw13_b200``) and never imports it.

Contents
  * ``stencil_oracle.c`` -- Eq. (1) + Fig. 1 of PAPER.md in plain fp64 C
    (Sec. III-A), and the Table V application stencils (Poisson-type
    source, leapfrog wave, Div, Grad); loaded here through ctypes.
  * ``model_p.py``       -- the paper's performance model, Eqs. (6)-(14)
    (Sec. VI), written out literally.
  * ``inplane_sim.py``   -- the paper's in-plane steps 1-6 (P:L168-173,
    Eqs. 3-5) as a scalar simulator (used to pin the oracle).

Array convention: dense *outer* grids as numpy float64 arrays of shape
``(nz+2r, ny+2r, nx+2r)`` (x fastest); the r-wide shell is a frozen Dirichlet
boundary (reading R1).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "stencil_oracle.c")
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile ``stencil_oracle.c`` with gcc (plain -O2, OpenMP, no FP contraction)."""
    if force or not os.path.exists(_LIB_PATH) or (
        os.path.getmtime(_LIB_PATH) < os.path.getmtime(_SRC)
    ):
        cmd = [
            "gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-fopenmp",
            "-ffp-contract=off", "-fno-fast-math", _SRC, "-o", _LIB_PATH + ".tmp",
        ]
        subprocess.run(cmd, check=True)
        os.replace(_LIB_PATH + ".tmp", _LIB_PATH)
    return _LIB_PATH


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        dp = ctypes.POINTER(ctypes.c_double)
        L, I = ctypes.c_long, ctypes.c_int
        lib.oracle_sweep.argtypes = [dp, dp, L, L, L, I, dp, I, I]
        lib.oracle_sweep.restype = I
        lib.oracle_sweep_axes.argtypes = [dp, dp, L, L, L, I, dp, I, I]
        lib.oracle_sweep_axes.restype = I
        lib.oracle_point.argtypes = [dp, L, L, L, I, dp, I, L, L, L, dp]
        lib.oracle_point.restype = I
        lib.oracle_time_sweep.argtypes = [dp, dp, L, L, L, I, dp, I, I]
        lib.oracle_time_sweep.restype = ctypes.c_double
        lib.oracle_source.argtypes = [dp, dp, ctypes.c_double, dp, L, L, L, I, dp, I, I]
        lib.oracle_source.restype = I
        lib.oracle_wave.argtypes = [dp, dp, ctypes.c_double, L, L, L, I, dp, I, I]
        lib.oracle_wave.restype = I
        lib.oracle_div.argtypes = [dp, dp, dp, dp, L, L, L, I, dp, I]
        lib.oracle_div.restype = I
        lib.oracle_grad.argtypes = [dp, dp, dp, dp, L, L, L, I, dp, I]
        lib.oracle_grad.restype = I
        lib.oracle_max_threads.argtypes = []
        lib.oracle_max_threads.restype = I
        _lib = lib
    return _lib


def _dptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_double))


def _check_outer(u: np.ndarray, r: int):
    if u.ndim != 3:
        raise ValueError("outer grid must be 3-D (nz+2r, ny+2r, nx+2r)")
    nz, ny, nx = (s - 2 * r for s in u.shape)
    if min(nx, ny, nz) < 1:
        raise ValueError("outer grid smaller than its shell")
    return nx, ny, nz


def sweep(u0: np.ndarray, r: int, coeffs, iters: int, nthreads: int = 1) -> np.ndarray:
    """ITERSTENCILLOOP (Fig. 1) of Eq. (1): ``iters`` Jacobi sweeps of ``u0``.

    ``u0``: outer grid (any real dtype; converted to float64 exactly).
    ``coeffs``: c0..cr.  Returns a new float64 outer grid (shell == u0's shell).
    """
    a = np.ascontiguousarray(u0, dtype=np.float64)
    nx, ny, nz = _check_outer(a, r)
    c = np.ascontiguousarray(coeffs, dtype=np.float64)
    if c.shape != (r + 1,):
        raise ValueError("need r+1 coefficients")
    out = np.empty_like(a)
    rc = _load().oracle_sweep(_dptr(a), _dptr(out), nx, ny, nz, r, _dptr(c), int(iters), int(nthreads))
    if rc != 0:
        raise ValueError(f"oracle_sweep failed with code {rc}")
    return out


def sweep_axes(u0: np.ndarray, r: int, coeffs, iters: int, nthreads: int = 1) -> np.ndarray:
    """Fig. 1 loop of the per-axis stencil (reading R3b): ``coeffs`` = 1 + 3r values
    c0, cx_1..cx_r, cy_1..cy_r, cz_1..cz_r.  Eq. (1) when the three axis sets agree."""
    a = np.ascontiguousarray(u0, dtype=np.float64)
    nx, ny, nz = _check_outer(a, r)
    c = np.ascontiguousarray(coeffs, dtype=np.float64)
    if c.shape != (1 + 3 * r,):
        raise ValueError("need 1 + 3r coefficients")
    out = np.empty_like(a)
    rc = _load().oracle_sweep_axes(_dptr(a), _dptr(out), nx, ny, nz, r, _dptr(c), int(iters), int(nthreads))
    if rc != 0:
        raise ValueError(f"oracle_sweep_axes failed with code {rc}")
    return out


def run_until(u0: np.ndarray, r: int, coeffs, max_iters: int, tol: float, check_every: int = 1):
    """Fig. 1 with its stop criterion (reading R5b): sweep (``sweep``, or
    ``sweep_axes`` for 1 + 3r coefficients) one step at a time; after every
    ``check_every``-th sweep and after sweep ``max_iters`` the residual is
    max over interior |u_t - u_{t-1}| (fp64); stop when it is <= ``tol``.
    Returns (u_T, T, residual_T)."""
    step = sweep_axes if len(coeffs) == 1 + 3 * r else sweep
    a = np.ascontiguousarray(u0, dtype=np.float64)
    inner = (slice(r, -r),) * 3
    res = -1.0
    t = 0
    while t < max_iters:
        t += 1
        b = step(a, r, coeffs, 1)
        if t % check_every == 0 or t == max_iters:
            res = float(np.max(np.abs(b[inner] - a[inner])))
            if res <= tol:
                a = b
                break
        a = b
    return a, t, res


def source(u0: np.ndarray, f: np.ndarray, d: float, r: int, coeffs, iters: int, nthreads: int = 1) -> np.ndarray:
    """Table V "Poisson"-type iteration: ``iters`` sweeps u <- S(u) + d f (Eq. 1 then + d f)."""
    a = np.ascontiguousarray(u0, dtype=np.float64)
    nx, ny, nz = _check_outer(a, r)
    g = np.ascontiguousarray(f, dtype=np.float64)
    if g.shape != a.shape:
        raise ValueError("f must have the outer shape of u0")
    c = np.ascontiguousarray(coeffs, dtype=np.float64)
    if c.shape != (r + 1,):
        raise ValueError("need r+1 coefficients")
    out = np.empty_like(a)
    rc = _load().oracle_source(_dptr(a), _dptr(g), float(d), _dptr(out), nx, ny, nz, r, _dptr(c), int(iters),
                               int(nthreads))
    if rc != 0:
        raise ValueError(f"oracle_source failed with code {rc}")
    return out


def wave(u_prev: np.ndarray, u: np.ndarray, d: float, r: int, coeffs, iters: int, nthreads: int = 1):
    """Leapfrog u_{n+1} = S(u_n) + d u_{n-1}; returns the new (u_prev, u) (states n+iters-1, n+iters)."""
    a = np.array(u_prev, dtype=np.float64, order="C", copy=True)
    b = np.array(u, dtype=np.float64, order="C", copy=True)
    nx, ny, nz = _check_outer(b, r)
    if a.shape != b.shape:
        raise ValueError("u_prev and u must have the same outer shape")
    c = np.ascontiguousarray(coeffs, dtype=np.float64)
    if c.shape != (r + 1,):
        raise ValueError("need r+1 coefficients")
    rc = _load().oracle_wave(_dptr(a), _dptr(b), float(d), nx, ny, nz, r, _dptr(c), int(iters), int(nthreads))
    if rc != 0:
        raise ValueError(f"oracle_wave failed with code {rc}")
    return a, b


def div(u: np.ndarray, v: np.ndarray, w: np.ndarray, r: int, a) -> np.ndarray:
    """Table V "Div" (3 grids -> 1, reading R19): sum_m a_m ((u[i+m]-u[i-m]) + (v[j+m]-v[j-m]) + (w[k+m]-w[k-m]))
    at every interior point; ``a`` = a_1..a_r; shell of the result 0."""
    g = [np.ascontiguousarray(x, dtype=np.float64) for x in (u, v, w)]
    nx, ny, nz = _check_outer(g[0], r)
    if any(x.shape != g[0].shape for x in g):
        raise ValueError("u, v, w must share the outer shape")
    c = np.ascontiguousarray(a, dtype=np.float64)
    if c.shape != (r,):
        raise ValueError("need r coefficients a_1..a_r")
    out = np.empty_like(g[0])
    rc = _load().oracle_div(_dptr(g[0]), _dptr(g[1]), _dptr(g[2]), _dptr(out), nx, ny, nz, r, _dptr(c), 1)
    if rc != 0:
        raise ValueError(f"oracle_div failed with code {rc}")
    return out


def grad(f: np.ndarray, r: int, a):
    """Table V "Grad" (1 grid -> 3, reading R19): (gx, gy, gz) = sum_m a_m (f[+m]-f[-m]) along x, y, z."""
    g = np.ascontiguousarray(f, dtype=np.float64)
    nx, ny, nz = _check_outer(g, r)
    c = np.ascontiguousarray(a, dtype=np.float64)
    if c.shape != (r,):
        raise ValueError("need r coefficients a_1..a_r")
    gx, gy, gz = np.empty_like(g), np.empty_like(g), np.empty_like(g)
    rc = _load().oracle_grad(_dptr(g), _dptr(gx), _dptr(gy), _dptr(gz), nx, ny, nz, r, _dptr(c), 1)
    if rc != 0:
        raise ValueError(f"oracle_grad failed with code {rc}")
    return gx, gy, gz


def point(u0: np.ndarray, r: int, coeffs, iters: int, i: int, j: int, k: int) -> float:
    """Value at INTERIOR point (i, j, k) after ``iters`` sweeps (dependency-cone evaluation)."""
    a = np.ascontiguousarray(u0, dtype=np.float64)
    nx, ny, nz = _check_outer(a, r)
    c = np.ascontiguousarray(coeffs, dtype=np.float64)
    v = ctypes.c_double(0.0)
    rc = _load().oracle_point(_dptr(a), nx, ny, nz, r, _dptr(c), int(iters), int(i), int(j), int(k), ctypes.byref(v))
    if rc != 0:
        raise ValueError(f"oracle_point failed with code {rc}")
    return v.value


def time_sweep(u0: np.ndarray, r: int, coeffs, iters: int, nthreads: int):
    """(seconds, result) of one oracle sweep; used by bench.py's cpu_baseline leg."""
    a = np.ascontiguousarray(u0, dtype=np.float64)
    nx, ny, nz = _check_outer(a, r)
    c = np.ascontiguousarray(coeffs, dtype=np.float64)
    out = np.empty_like(a)
    t = _load().oracle_time_sweep(_dptr(a), _dptr(out), nx, ny, nz, r, _dptr(c), int(iters), int(nthreads))
    if t < 0:
        raise ValueError("oracle_time_sweep failed")
    return t, out


def max_threads() -> int:
    return int(_load().oracle_max_threads())
