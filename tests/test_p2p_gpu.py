"""GPU tests of the fused peer-store slab decomposition (stencil_plan_create_p2p,
SURVEY NEXT-3): the halo exchange rides on the in-plane kernel's own stores
into the neighbours' grids, ordered by stream-side flags.

* several slab plans in ONE process on one GPU, each on its own stream, wired
  with stencil_p2p_connect (plain device pointers) -- the protocol runs
  concurrently exactly as across GPUs;
* two PROCESSES sharing the GPU, wired through CUDA IPC handles
  (stencil_p2p_export / stencil_p2p_import) -- the multi-process path.

The assembled result must be BIT-IDENTICAL to the single-GPU plan (one fixed
per-point order for every decomposition, reading R7) and match the oracle
within the north-star tolerance."""
import os
import socket

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


def single_gpu(S, u, r, c, dtype, iters):
    nz, ny, nx = (d - 2 * r for d in u.shape)
    with S.Plan(nx, ny, nz, r, c, dtype) as p:
        a, b = p.upload(u), p.alloc()
        p.run(a, b, iters)
        return p.download(b)


def run_slabs(S, u, r, c, dtype, P, chunks, cfg=None):
    import torch
    nz, ny, nx = (d - 2 * r for d in u.shape)
    plans = [S.P2PSlab(nx, ny, nz, r, c, dtype, k, P) for k in range(P)]
    for k, p in enumerate(plans):
        p.connect(plans[k - 1] if k > 0 else None, plans[k + 1] if k < P - 1 else None)
        if cfg:
            p.set_config(**cfg)
        p.fill_local(u)
    torch.cuda.synchronize()
    streams = [torch.cuda.Stream() for _ in range(P)]
    for n in chunks:                      # every rank issues its sweeps; the GPU orders them by flags
        for p, s in zip(plans, streams):
            p.run(n, stream=s)
    torch.cuda.synchronize()
    out = u.astype(np.float64).copy()
    for p in plans:
        loc = p.local_result()
        out[r + p.z0: r + p.z0 + p.nz_local] = loc[r:-r]
    for p in plans:
        p.close()
    return out


@pytest.mark.parametrize("dtype", ["f32", "f64"])
@pytest.mark.parametrize("r,P", [(1, 2), (2, 3), (4, 4), (4, 2), (6, 3)])
def test_p2p_slabs_one_process(S, r, P, dtype):
    nx, ny = 37, 23
    nz = 4 * P * r + 3                     # ragged partition
    u = si.uniform(nx, ny, nz, r, seed=60 + r + P, dtype=dtype)
    c = si.coeffs_as("heat", r, dtype)
    want = single_gpu(S, u, r, c, dtype, 10)
    got = run_slabs(S, u, r, c, dtype, P, [10])
    assert np.array_equal(got.astype(want.dtype), want)
    assert rel_err(got, oracle.sweep(u, r, c, 10), r) <= TOL[dtype]


def test_p2p_continuation_and_segments(S):
    r, P, dtype = 2, 3, "f32"
    nx, ny, nz = 40, 18, 30
    u = si.uniform(nx, ny, nz, r, seed=9, dtype=dtype)
    c = si.coeffs_as("heat", r, dtype)
    want = single_gpu(S, u, r, c, dtype, 9)
    vec = 4
    cfg = dict(kernel="inplane", tx=16, ty=2, rx=vec, ry=2, stages=3, zsegs=2, zbox=2)
    got = run_slabs(S, u, r, c, dtype, P, [4, 1, 4], cfg)   # runs continue from the current grid
    assert np.array_equal(got.astype(want.dtype), want)


def test_p2p_integer_field_bit_exact(S):
    # integer field and coefficients, every partial sum exact in fp32 (8 W^T < 2^24)
    r, P, dtype, iters = 3, 3, "f32", 2
    c = [2.0, -1.0, 1.0, 1.0]
    nx, ny, nz = 21, 19, 25
    u = si.integers(nx, ny, nz, r, seed=4, dtype=dtype)
    o = oracle.sweep(u, r, c, iters)
    got = run_slabs(S, u, r, c, dtype, P, [1, 1])
    assert np.array_equal(got, o)


def test_p2p_rejects_bad_wiring(S):
    r, dtype = 1, "f32"
    a = S.P2PSlab(16, 16, 20, r, [0.5, 0.05], dtype, 0, 2)
    b = S.P2PSlab(16, 16, 20, r, [0.5, 0.05], dtype, 1, 2)
    with pytest.raises(S.StencilError):
        a.connect(None, None)              # rank 0 of 2 needs its upper neighbour
    with pytest.raises(S.StencilError):
        a.run(1)                           # not connected
    with pytest.raises(S.StencilError):
        b.connect(None, a)                 # wrong side
    a.close()
    b.close()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _ipc_worker(rank, world, port, r, dtype, iters, q):
    import torch
    import torch.distributed as dist
    import paper_conf_ipps_tangtkwkgtw13_b200 as S2
    import stencil_inputs as si2
    try:
        os.environ["MASTER_ADDR"], os.environ["MASTER_PORT"] = "127.0.0.1", str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        torch.cuda.set_device(0)
        nx, ny, nz = 33, 20, 26
        u = si2.uniform(nx, ny, nz, r, seed=77, dtype=dtype)
        c = si2.coeffs_as("heat", r, dtype)
        p = S2.P2PSlab(nx, ny, nz, r, c, dtype, rank, world)
        handles = [None] * world
        dist.all_gather_object(handles, p.export_handles())
        p.import_handles(handles[rank - 1] if rank > 0 else None, handles[rank + 1] if rank < world - 1 else None)
        p.fill_local(u)
        torch.cuda.synchronize()
        dist.barrier()                     # every fill done before any sweep
        p.run(iters)
        torch.cuda.synchronize()
        dist.barrier()                     # neighbours' last peer stores are done too
        loc = p.local_result()
        parts = [None] * world
        dist.all_gather_object(parts, (p.z0, p.nz_local, loc))
        dist.barrier()
        p.close()
        dist.destroy_process_group()
        if rank == 0:
            q.put(("ok", parts))
    except Exception as e:  # pragma: no cover - reported to the parent
        q.put(("error", f"rank {rank}: {type(e).__name__}: {e}"))


@pytest.mark.parametrize("world", [2, 3])
def test_p2p_two_processes_ipc(S, world):
    import multiprocessing as mp
    r, dtype, iters = 2, "f32", 7
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_ipc_worker, args=(k, world, port, r, dtype, iters, q)) for k in range(world)]
    for pr in procs:
        pr.start()
    kind, payload = q.get(timeout=300)
    for pr in procs:
        pr.join(timeout=120)
    assert kind == "ok", payload
    nx, ny, nz = 33, 20, 26
    u = si.uniform(nx, ny, nz, r, seed=77, dtype=dtype)
    c = si.coeffs_as("heat", r, dtype)
    out = u.astype(np.float64).copy()
    for z0, nzl, loc in payload:
        out[r + z0: r + z0 + nzl] = loc[r:-r]
    want = single_gpu(S, u, r, c, dtype, iters)
    assert np.array_equal(out.astype(want.dtype), want)


def test_bench_two_ranks_p2p_on_one_gpu():
    """bench.py's N>1 path (torchrun, fused p2p exchange) end to end on one GPU
    (STENCIL_BENCH_SAME_DEVICE=1: both ranks on cuda:0, gloo process group)."""
    import json
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, STENCIL_BENCH_SAME_DEVICE="1")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(_free_port()), "bench.py", "--gpus", "2",
           "--steps", "2", "--warmup", "3", "--iters", "10", "--tune", "none", "--config", "32,8,4,4,4,2,2,0",
           "--no-cpu", "--workload", "c2"]
    p = subprocess.run(cmd, cwd=root, env=env, capture_output=True, text=True, timeout=600)
    assert p.returncode == 0, p.stderr[-3000:]
    lines = [ln for ln in p.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, p.stdout
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["value"] > 0 and d["config"]["exchange"].startswith("fused")
    assert d["e2e"]["value"] > 0 and d["gpu_launches"] > 0


def test_p2p_residual_matches_single_plan(S):
    """the slabs' local residuals max-reduce to the single-GPU stop-criterion residual, bit for bit"""
    import torch
    r, P, dtype, K = 2, 3, "f32", 5
    nx, ny, nz = 30, 17, 28
    u = si.uniform(nx, ny, nz, r, seed=21, dtype=dtype)
    c = si.coeffs_as("heat", r, dtype)
    with S.Plan(nx, ny, nz, r, c, dtype) as p:
        a, b = p.upload(u), p.alloc()
        T, res_single = p.run_until(a, b, K, 0.0, K)
        assert T == K
    plans = [S.P2PSlab(nx, ny, nz, r, c, dtype, k, P) for k in range(P)]
    for k, p in enumerate(plans):
        p.connect(plans[k - 1] if k > 0 else None, plans[k + 1] if k < P - 1 else None)
        p.fill_local(u)
    torch.cuda.synchronize()
    streams = [torch.cuda.Stream() for _ in range(P)]
    for p, s in zip(plans, streams):
        p.run(K, stream=s)
    res = max(p.residual(stream=s) for p, s in zip(plans, streams))
    assert res == res_single
    for p in plans:
        p.close()


def _ipc_until_worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    import paper_conf_ipps_tangtkwkgtw13_b200 as S2
    import stencil_inputs as si2
    try:
        os.environ["MASTER_ADDR"], os.environ["MASTER_PORT"] = "127.0.0.1", str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        torch.cuda.set_device(0)
        r, dtype = 1, "f32"
        nx, ny, nz = 21, 14, 13
        u = si2.uniform(nx, ny, nz, r, seed=41, dtype=dtype)
        c = si2.coeffs_as("heat", r, dtype)
        tol = float(os.environ["P2P_TEST_TOL"])
        p = S2.P2PSlab(nx, ny, nz, r, c, dtype, rank, world)
        handles = [None] * world
        dist.all_gather_object(handles, p.export_handles())
        p.import_handles(handles[rank - 1] if rank > 0 else None, handles[rank + 1] if rank < world - 1 else None)
        p.fill_local(u)
        torch.cuda.synchronize()
        dist.barrier()
        T, res = p.run_until(1000, tol, 3)
        torch.cuda.synchronize()
        dist.barrier()
        parts = [None] * world
        dist.all_gather_object(parts, (p.z0, p.nz_local, p.local_result(), T, res))
        dist.barrier()
        p.close()
        dist.destroy_process_group()
        if rank == 0:
            q.put(("ok", parts))
    except Exception as e:  # pragma: no cover
        q.put(("error", f"rank {rank}: {type(e).__name__}: {e}"))


def test_p2p_run_until_two_processes(S):
    """multi-rank Fig. 1 stop criterion: local residuals + one all-reduce per check (gloo here)"""
    import math
    import multiprocessing as mp
    r, dtype, every = 1, "f32", 3
    nx, ny, nz = 21, 14, 13
    u = si.uniform(nx, ny, nz, r, seed=41, dtype=dtype)
    c = si.coeffs_as("heat", r, dtype)
    rho = [oracle.run_until(u, r, c, k * every, 0.0, every)[2] for k in range(1, 6)]
    assert rho[2] / rho[3] >= 1.2
    tol = math.sqrt(rho[2] * rho[3])
    want_u, want_T, _ = oracle.run_until(u, r, c, 1000, tol, every)
    os.environ["P2P_TEST_TOL"] = repr(tol)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_ipc_until_worker, args=(k, 2, port, q)) for k in range(2)]
    for pr in procs:
        pr.start()
    kind, payload = q.get(timeout=300)
    for pr in procs:
        pr.join(timeout=120)
    assert kind == "ok", payload
    out = u.astype(np.float64).copy()
    for z0, nzl, loc, T, res in payload:
        assert T == want_T
        out[r + z0: r + z0 + nzl] = loc[r:-r]
    assert rel_err(out, want_u, r) <= TOL[dtype]



@pytest.mark.parametrize("r", [2, 3])
def test_p2p_thin_middle_slab(S, r):
    """A middle slab of exactly r planes (r <= nz_local < 2r): each of its planes is both among the
    first r (-> rank-1's halo) and the last r (-> rank+1's halo), so every completed plane goes to
    BOTH neighbours (the lower store used to be dropped)."""
    P, dtype = 3, "f64"
    nx, ny, nz = 23, 17, 3 * r            # every slab has exactly r planes
    c = [float(x) for x in [2, -1, 1, 1][: r + 1]]
    u = si.integers(nx, ny, nz, r, seed=31 + r, dtype=dtype)
    o = oracle.sweep(u, r, c, 4)
    got = run_slabs(S, u, r, c, dtype, P, [2, 2])
    assert np.array_equal(got, o)


def _ws_cfgs(dtype):
    vec = 4 if dtype == "f32" else 2
    return [dict(kernel="inplane_ws", tx=16, ty=4, rx=vec, ry=2, stages=3, zsegs=2, zbox=2),
            dict(kernel="inplane_ws", tx=32, ty=2, rx=vec, ry=4, stages=4, zsegs=1, zbox=1),
            dict(kernel="inplane_ws", tx=16, ty=8, rx=vec, ry=2, stages=3, zsegs=3, zbox=4, ytiles=3)]


@pytest.mark.parametrize("dtype", ["f32", "f64"])
@pytest.mark.parametrize("grid", ["ragged", "aligned"])
@pytest.mark.parametrize("r,P", [(1, 3), (2, 2), (4, 3)])
def test_p2p_warp_specialized_slabs(S, r, P, dtype, grid):
    """The warp-specialized kernel's fused peer-store variant (inplane_ws.cuh, PS): the peer stores sit in
    the head / tail blocks of U steps only; ragged tiles (element path) and whole interior tiles (8-byte
    path), both sweep directions (odd then even run lengths), z segments, box depths 1 / 2 / 4:
    bit-identical to the single plan."""
    vec = 4 if dtype == "f32" else 2
    nx, ny = (37, 23) if grid == "ragged" else (16 * vec, 16)
    nz = 4 * P * r + 5
    u = si.uniform(nx, ny, nz, r, seed=90 + r + P, dtype=dtype)
    c = si.coeffs_as("heat", r, dtype)
    want = single_gpu(S, u, r, c, dtype, 7)
    for cfg in _ws_cfgs(dtype):
        got = run_slabs(S, u, r, c, dtype, P, [3, 4], cfg)
        assert np.array_equal(got.astype(want.dtype), want), cfg


@pytest.mark.parametrize("r", [2, 3])
def test_p2p_warp_specialized_thin_middle_slab(S, r):
    """the warp-specialized PS kernel on slabs of exactly r planes (every plane to both neighbours)"""
    P, dtype = 3, "f32"
    nx, ny, nz = 64, 16, 3 * r
    c = [float(x) for x in [2, -1, 1, 1][: r + 1]]
    u = si.integers(nx, ny, nz, r, seed=41 + r, dtype=dtype)
    o = oracle.sweep(u, r, c, 3)
    for cfg in _ws_cfgs(dtype)[:2]:
        got = run_slabs(S, u, r, c, dtype, P, [1, 2], dict(cfg, zsegs=1))
        assert np.array_equal(got, o), cfg


def test_p2p_fill_counter_is_the_global_field(S):
    """stencil_fill_counter on a p2p slab fills global planes z0 .. z0 + nz_local + 2r (stencil.h); the
    slabs together equal the undecomposed counter field (every slab used to get rank 0's)."""
    import torch
    r, P, nx, ny, nz = 2, 3, 20, 11, 17
    c = si.coeffs_as("heat", r, "f32")
    plans = [S.P2PSlab(nx, ny, nz, r, c, "f32", k, P) for k in range(P)]
    try:
        for p in plans:
            g = p.grid_tensor(0)
            p.fill_counter(g, 13)
            torch.cuda.synchronize()
            got = p.grid_view(0).cpu().numpy()
            want = si.counter(nx, ny, p.nz_local, r, 13, "f32", z0=p.z0)
            assert np.array_equal(got, want), p.z0
    finally:
        for p in plans:
            p.close()


def test_p2p_run_until_threads_in_one_process(S):
    """stencil_p2p_run_until on three slabs of one process (a host thread per slab, as one process per
    GPU would): the device-side residual reduction gives every rank the same stop sweep and residual,
    equal to the single-GPU stop criterion."""
    import math
    import threading
    import torch
    r, P, dtype, every = 2, 3, "f32", 2
    nx, ny, nz = 25, 16, 21
    u = si.uniform(nx, ny, nz, r, seed=44, dtype=dtype)
    c = si.coeffs_as("heat", r, dtype)
    rho = [oracle.run_until(u, r, c, k * every, 0.0, every)[2] for k in range(1, 7)]
    k = next(i for i in range(2, 5) if rho[i] / rho[i + 1] >= 1.2)
    tol = math.sqrt(rho[k] * rho[k + 1])
    want_u, want_T, _ = oracle.run_until(u, r, c, 1000, tol, every)
    with S.Plan(nx, ny, nz, r, c, dtype) as p:
        a, b = p.upload(u), p.alloc()
        T1, res1 = p.run_until(a, b, 1000, tol, every)
    assert T1 == want_T
    plans = [S.P2PSlab(nx, ny, nz, r, c, dtype, q, P) for q in range(P)]
    for q, p in enumerate(plans):
        p.connect(plans[q - 1] if q > 0 else None, plans[q + 1] if q < P - 1 else None)
        p.fill_local(u)
    torch.cuda.synchronize()
    results = [None] * P

    def work(q):
        results[q] = plans[q].run_until(1000, tol, every, stream=torch.cuda.Stream())

    ths = [threading.Thread(target=work, args=(q,)) for q in range(P)]
    for t in ths:
        t.start()
    for t in ths:
        t.join(timeout=120)
    assert all(res == (T1, res1) for res in results), (results, T1, res1)
    torch.cuda.synchronize()
    out = u.astype(np.float64).copy()
    for p in plans:
        p.quiesce()
        torch.cuda.synchronize()
        out[r + p.z0: r + p.z0 + p.nz_local] = p.local_result()[r:-r]
        p.close()
    assert rel_err(out, want_u, r) <= TOL[dtype]
