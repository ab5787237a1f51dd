"""The distributed plan's multi-rank logic on one GPU: every rank of a
z-slab decomposition in one process (stencil_plan_create_dist_local / stencil_run_dist_local) with the
DistPlan's partition, boundary-first split, events and exchange offsets; the transport is
cudaMemcpyAsync into the neighbour's buffer.  The assembled result must be BIT-IDENTICAL to the
single-GPU plan (one fixed per-point order, reading R7) and match the oracle."""
import numpy as np
import pytest

import oracle
import stencil_inputs as si
from test_parity_gpu import INT_COEFFS, TOL, rel_err

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def S():
    import torch  # noqa: F401
    import paper_conf_ipps_tangtkwkgtw13_b200 as pkg
    return pkg


def single(S, u, r, c, dtype, iters):
    nz, ny, nx = (d - 2 * r for d in u.shape)
    with S.Plan(nx, ny, nz, r, c, dtype) as p:
        a, b = p.upload(u), p.alloc()
        p.run(a, b, iters)
        return p.download(b)


def run_group(S, u, r, c, dtype, P, iters, cfg=None):
    import torch
    nz, ny, nx = (d - 2 * r for d in u.shape)
    out = u.astype(np.float64).copy()
    with S.LocalRankGroup(nx, ny, nz, r, c, dtype, P) as g:
        ins, outs = [], []
        for q in g.plans:
            if cfg:
                q.set_config(**cfg)
            ins.append(q.upload(np.ascontiguousarray(u[q.z0: q.z0 + q.nz_local + 2 * r])))
            outs.append(q.alloc())
        streams = [torch.cuda.Stream() for _ in g.plans]
        torch.cuda.synchronize()
        g.run(ins, outs, iters, streams)
        torch.cuda.synchronize()
        for q, t in zip(g.plans, outs):
            out[r + q.z0: r + q.z0 + q.nz_local] = q.download(t)[r:-r]
            assert np.array_equal(q.download(ins[g.plans.index(q)]),
                                  u[q.z0: q.z0 + q.nz_local + 2 * r].astype(out.dtype if dtype == "f64" else np.float32))
    return out


@pytest.mark.parametrize("dtype", ["f32", "f64"])
@pytest.mark.parametrize("r,P,zsegs", [(1, 2, 1), (2, 3, 3), (4, 4, 2), (4, 2, 4), (3, 3, 1)])
@pytest.mark.parametrize("iters", [1, 2, 7])
def test_group_matches_single_plan(S, r, P, zsegs, dtype, iters):
    vec = 4 if dtype == "f32" else 2
    nx, ny = 37, 23
    nz = 5 * P * r + 2                     # ragged partition; zsegs segments of >= r planes where asked
    u = si.uniform(nx, ny, nz, r, seed=90 + r + P, dtype=dtype)
    c = si.coeffs_as("heat", r, dtype)
    cfg = dict(kernel="inplane_ws", tx=16, ty=4, rx=vec, ry=2, stages=3, zsegs=zsegs, zbox=2)
    want = single(S, u, r, c, dtype, iters)
    got = run_group(S, u, r, c, dtype, P, iters, cfg)
    assert np.array_equal(got.astype(want.dtype), want)
    assert rel_err(got, oracle.sweep(u, r, c, iters), r) <= TOL[dtype]


def test_group_thin_segments_fall_back_to_sweep_then_exchange(S):
    """zsegs whose segments hold fewer than r planes: the exchange must follow the
    WHOLE sweep, not just the boundary segments -- still bit-identical."""
    r, P, dtype = 4, 3, "f32"
    nx, ny, nz = 30, 20, 3 * 12
    u = si.uniform(nx, ny, nz, r, seed=7, dtype=dtype)
    c = si.coeffs_as("heat", r, dtype)
    cfg = dict(kernel="inplane", tx=16, ty=2, rx=4, ry=2, stages=3, zsegs=6, zbox=1)   # 2-plane segments
    want = single(S, u, r, c, dtype, 5)
    got = run_group(S, u, r, c, dtype, P, 5, cfg)
    assert np.array_equal(got.astype(want.dtype), want)


def test_group_integer_field_bit_exact(S):
    r, P, dtype, iters = 3, 4, "f64", 5
    c = [float(x) for x in INT_COEFFS[r]]
    nx, ny, nz = 21, 19, 4 * 3 * r
    u = si.integers(nx, ny, nz, r, seed=12, dtype=dtype)
    got = run_group(S, u, r, c, dtype, P, iters)
    assert np.array_equal(got, oracle.sweep(u, r, c, iters))


def test_group_members_refuse_stencil_run(S):
    with S.LocalRankGroup(20, 10, 12, 1, [0.5, 0.1], "f32", 2) as g:
        q = g.plans[0]
        a, b = q.alloc(), q.alloc()
        with pytest.raises(S.StencilError):
            q.run(a, b, 2)
