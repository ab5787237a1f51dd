"""CUDA-graph replay of stencil_run (plan.cu run_jacobi_graph): the first run of
a (buffers, iters, configuration) key is captured, later runs replay it.  The
replayed result must equal the oracle and the un-captured path bit for bit,
for every key, including after a configuration change."""
import numpy as np
import pytest

import oracle
import stencil_inputs as si
from test_parity_gpu import TOL, rel_err

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def S():
    import torch  # noqa: F401
    import paper_conf_ipps_tangtkwkgtw13_b200 as pkg
    return pkg


def test_graph_replay_matches(S):
    r, dtype = 1, "f32"
    n = 64
    u = si.uniform(n, n, n, r, seed=1, dtype=dtype)
    c = si.coeffs_as("heat", r, dtype)
    with S.Plan(n, n, n, r, c, dtype) as p:
        a, b = p.upload(u), p.alloc()
        outs = []
        for iters in (10, 10, 3, 10, 3):            # capture, replay, new key, replay, replay
            p.run(a, b, iters)
            outs.append((iters, p.download(b)))
        s0 = p.stats()
        p.run(a, b, 10)
        s1 = p.stats()
        assert s1["launches"] - s0["launches"] == 10   # replays still count their sweep launches
        p.set_timing(True)                           # timing runs bypass graphs: reference result
        p.run(a, b, 10)
        ref10 = p.download(b)
        p.run(a, b, 3)
        ref3 = p.download(b)
        p.set_timing(False)
        for iters, g in outs:
            assert np.array_equal(g, ref10 if iters == 10 else ref3)
        assert rel_err(ref10, oracle.sweep(u, r, c, 10), r) <= TOL[dtype]
        # a configuration change is a new key
        p.set_config(kernel="inplane", tx=16, ty=4, rx=4, ry=2, stages=3, zsegs=2, zbox=2)
        p.run(a, b, 10)
        p.run(a, b, 10)
        assert np.array_equal(p.download(b), ref10)   # one fixed order for every configuration
        # a different output buffer is a new key
        b2 = p.alloc()
        p.run(a, b2, 10)
        assert np.array_equal(p.download(b2), ref10)


def test_run_host_pipelined(S):
    """stencil_run_host: several back-to-back host-to-host calls (upload / sweeps / download
    pipelined over two device slots) each give the oracle's result for their own input."""
    import torch
    r, dtype, iters = 2, "f32", 4
    nx, ny, nz = 40, 26, 22
    c = si.coeffs_as("heat", r, dtype)
    with S.Plan(nx, ny, nz, r, c, dtype) as p:
        n = p.alloc().numel()
        ins, outs, fields = [], [], []
        for k in range(5):
            u = si.uniform(nx, ny, nz, r, seed=200 + k, dtype=dtype)
            d = p.upload(u)
            h = torch.empty(n, dtype=d.dtype, pin_memory=True)
            h.copy_(d)
            ins.append(h)
            outs.append(torch.zeros(n, dtype=d.dtype, pin_memory=True))
            fields.append(u)
        torch.cuda.synchronize()
        s = torch.cuda.current_stream()
        for k in range(5):
            p.run_host(ins[k], outs[k], iters, stream=s)
        p.host_wait(stream=s)
        s.synchronize()
        for k in range(5):
            g = p.outer_view(outs[k].cuda()).cpu().numpy()
            assert rel_err(g, oracle.sweep(fields[k], r, c, iters), r) <= TOL[dtype]
