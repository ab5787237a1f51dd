"""BASELINE configs[4] at full size: 2048 x 2048 x 1024, r = 4 fp32, in the launch configurations bench.py
times -- the single-GPU grid of its `c5_1gpu` leg (plan default = the tune-cache tuple) and the z-slabs of
its N > 1 path (fused peer-store exchange, tune-cache tuple for the slab shape), here P slabs in one process
on one GPU -- 10 sweeps, sampled against the oracle point by point.

The field is the counter-based one bench.py fills on the device (`stencil_fill_counter`); the oracle gets
the same values from the seeded generator (`stencil_inputs.counter_block`), restricted to the dependency
cone of each sampled point: after `iters` sweeps a point depends on inputs within iters * r cells per axis,
so a block of half-width iters * r + r around it (clipped at the grid's real shell) has a frozen outer
layer no information from which reaches the point (R1).  Tolerance: north star 1e-5
relative (R8)."""
import numpy as np
import pytest

import oracle
import stencil_inputs as si
from test_parity_gpu import TOL

pytestmark = [pytest.mark.gpu, pytest.mark.slow]

NX, NY, NZ, R, DT, SEED, ITERS = 2048, 2048, 1024, 4, "f32", 5, 10


@pytest.fixture(scope="module")
def S():
    import torch  # noqa: F401
    import paper_conf_ipps_tangtkwkgtw13_b200 as pkg
    return pkg


def sample_points(extra_z=()):
    rng = np.random.default_rng(45)
    pts = [(0, 0, 0), (NX - 1, NY - 1, NZ - 1), (0, NY - 1, 511), (NX - 1, 0, 512), (1023, 1024, 1),
           (127, 128, 129), (128, 127, 1022), (2047, 1000, 700)]
    pts += [(int(rng.integers(0, NX)), int(rng.integers(0, NY)), int(z)) for z in extra_z]
    pts += [tuple(int(v) for v in (rng.integers(0, NX), rng.integers(0, NY), rng.integers(0, NZ))) for _ in range(6)]
    return pts


def oracle_at(coeffs, i, j, k):
    """oracle value at interior (i, j, k) after ITERS sweeps from the cone block of the counter field"""
    L = ITERS * R
    rng_ = []
    for c, n in ((k, NZ), (j, NY), (i, NX)):
        lo = max(0, c - L)                       # outer indices; the point is outer c + R
        hi = min(n + 2 * R, c + 2 * R + L + 1)
        rng_.append((lo, hi))
    blk = si.counter_block(NX, NY, R, SEED, DT, *rng_)
    (k0, _), (j0, _), (i0, _) = rng_
    return oracle.point(blk, R, coeffs, ITERS, i - i0, j - j0, k - k0)


def check(vals, coeffs):
    for (i, j, k), v in vals.items():
        o = oracle_at(coeffs, i, j, k)
        assert abs(v - o) <= TOL[DT] * abs(o), ((i, j, k), v, o)


def test_c5_single_gpu_sampled(S):
    """bench.py's c5_1gpu leg: one plan over the whole grid, plan default (tune-cache) configuration."""
    import torch
    c = si.coeffs_as("heat", R, DT)
    with S.Plan(NX, NY, NZ, R, c, DT) as p:
        a, b = p.alloc(), p.alloc()
        p.fill_counter(a, SEED)
        p.run(a, b, ITERS)
        torch.cuda.synchronize()
        g = p.outer_view(b)
        vals = {(i, j, k): float(g[k + R, j + R, i + R]) for (i, j, k) in sample_points()}
        cfg = p.config
    check(vals, c)
    assert cfg["kernel"] in ("inplane_ws", "inplane")


@pytest.mark.parametrize("P", [2, 4])
def test_c5_p2p_slabs_sampled(S, P):
    """bench.py's N > 1 path on one GPU: P fused peer-store slabs in one process (separate streams), each
    with the tune-cache tuple for its slab shape (as bench.py picks it), points on every slab interface."""
    import torch
    import bench
    c = si.coeffs_as("heat", R, DT)
    plans = [S.P2PSlab(NX, NY, NZ, R, c, DT, k, P) for k in range(P)]
    try:
        sm = torch.cuda.get_device_properties(0).multi_processor_count
        for k, p in enumerate(plans):
            p.connect(plans[k - 1] if k > 0 else None, plans[k + 1] if k < P - 1 else None)
            e = bench.cache_entry(NX, NY, p.nz_local, R, DT, 3, sm, None)
            if e is not None:
                d = e[1]
                p.set_config(kernel=e[0], tx=d["tx"], ty=d["ty"], rx=d["rx"], ry=d["ry"], stages=d["stages"],
                             zsegs=d["zsegs"], zbox=d["zbox"], ytiles=d["ytiles"])
            p.fill_counter(p.grid_tensor(0), SEED)
            p.fill_counter(p.grid_tensor(1), SEED)
        torch.cuda.synchronize()
        streams = [torch.cuda.Stream() for _ in plans]
        for p, s in zip(plans, streams):
            p.run(ITERS, stream=s)
        torch.cuda.synchronize()
        faces = []
        for p in plans[1:]:
            faces += [p.z0 - 1, p.z0, p.z0 + R - 1, p.z0 - R]
        vals = {}
        for (i, j, k) in sample_points(faces):
            p = next(q for q in plans if q.z0 <= k < q.z0 + q.nz_local)
            vals[(i, j, k)] = float(p.grid_view(p.current)[k - p.z0 + R, j + R, i + R])
    finally:
        for p in plans:
            p.close()
    check(vals, c)
