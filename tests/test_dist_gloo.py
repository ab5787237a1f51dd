"""Multi-process test of the z-slab decomposition's host logic (CPU, gloo).

The C library's host-only functions decide the decomposition:
``stencil_slab_partition`` (which planes a rank owns) and
``stencil_exchange_plan`` (which byte ranges of the pitched local buffer are
sent to / received from the neighbours after every sweep).  Here world_size 2
and 3 processes use exactly those answers, move the bytes with gloo send/recv
on host buffers laid out as ``stencil_layout_compute`` says, and sweep each
slab with the CPU oracle; the gathered result must equal the oracle run on the
undecomposed grid BIT FOR BIT (same fp64 arithmetic per point).  No GPU, no
NCCL: the transport differs, the decomposition under test does not.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, nx, ny, nz, r, iters, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        import stencil_inputs as si
        import paper_conf_ipps_tangtkwkgtw13_b200 as S

        c = [float(x) for x in si.coeffs("heat", r)]
        g = si.counter(nx, ny, nz, r, seed=9, dtype="f64")            # the global outer field
        z0, nzl = S.slab_partition(nz, world, rank, r)
        lay = S.layout_compute(nx, ny, nzl, r, "f64")
        xp = S.exchange_plan(lay, world, rank)
        buf = np.zeros(lay.bytes, dtype=np.uint8)                      # pitched local grid
        grid = buf.view(np.float64).reshape(lay.planes_z, lay.rows_y, lay.pitch_x)
        outer = grid[:, :, lay.x_origin: lay.x_origin + nx + 2 * r]
        outer[...] = g[z0: z0 + nzl + 2 * r]                          # local planes incl. halos
        tb = torch.from_numpy(buf)
        for _ in range(iters):
            new = oracle.sweep(np.ascontiguousarray(outer), r, c, 1)   # one Jacobi sweep of the slab
            outer[r:-r, r:-r, r:-r] = new[r:-r, r:-r, r:-r]
            ops = []
            for peer, s_off, r_off in ((xp["peer_lo"], xp["send_lo_off"], xp["recv_lo_off"]),
                                       (xp["peer_hi"], xp["send_hi_off"], xp["recv_hi_off"])):
                if peer < 0:
                    continue
                n = xp["msg_bytes"]
                ops.append(dist.P2POp(dist.isend, tb[s_off: s_off + n].clone(), peer))
                ops.append(dist.P2POp(dist.irecv, tb[r_off: r_off + n], peer))
            for w in dist.batch_isend_irecv(ops) if ops else []:
                w.wait()
        interior = torch.from_numpy(np.ascontiguousarray(outer[r:-r, r:-r, r:-r]))
        sizes = [S.slab_partition(nz, world, k, r)[1] for k in range(world)]
        if rank == 0:
            parts = [interior] + [torch.empty((n, ny, nx), dtype=torch.float64) for n in sizes[1:]]
            for k in range(1, world):
                dist.recv(parts[k], k)
            got = torch.cat(parts).numpy()
            ref = oracle.sweep(g, r, c, iters)[r:-r, r:-r, r:-r]
            q.put(("ok", bool(np.array_equal(got, ref)), float(np.max(np.abs(got - ref)))))
        else:
            dist.send(interior, 0)
    except Exception as e:  # pragma: no cover - surfaced through the queue
        q.put(("error", repr(e), 0.0))
        raise
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,nz,r", [(2, 12, 2), (2, 9, 4), (3, 14, 3)])
def test_zslab_decomposition_matches_global_oracle(world, nz, r):
    from conftest import build_library
    build_library()
    import oracle
    oracle.build()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(k, world, port, 11, 7, nz, r, 3, q)) for k in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=240)
    assert all(p.exitcode == 0 for p in procs), [p.exitcode for p in procs]
    status, same, err = q.get(timeout=5)
    assert status == "ok", same
    assert same, f"decomposed result differs from the global oracle (max abs diff {err})"


def _p2p_worker(rank, world, port, nx, ny, nz, r, iters, q):
    """Emulates the fused peer-store exchange (stencil_plan_create_p2p): after each
    sweep the rank 'stores' its boundary output planes into the neighbours' flat
    grids at (own element index + delta) from stencil_p2p_targets -- here the
    (indices, values) travel over gloo and the receiver writes them where the
    SENDER's deltas say, so a wrong delta lands data in the wrong planes."""
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        import stencil_inputs as si
        import paper_conf_ipps_tangtkwkgtw13_b200 as S

        c = [float(x) for x in si.coeffs("heat", r)]
        g = si.counter(nx, ny, nz, r, seed=13, dtype="f64")
        z0, nzl = S.slab_partition(nz, world, rank, r)
        lay = S.layout_compute(nx, ny, nzl, r, "f64")
        tg = S.p2p_targets(lay, nz, world, rank)
        flat = np.zeros(lay.bytes // 8, dtype=np.float64)            # pitched local grid, flat
        grid = flat.reshape(lay.planes_z, lay.rows_y, lay.pitch_x)
        outer = grid[:, :, lay.x_origin: lay.x_origin + nx + 2 * r]
        outer[...] = g[z0: z0 + nzl + 2 * r]
        # element indices of our interior output planes z (interior rows / columns only)
        idx = np.arange(flat.size).reshape(grid.shape)[:, :, lay.x_origin: lay.x_origin + nx + 2 * r]
        for _ in range(iters):
            new = oracle.sweep(np.ascontiguousarray(outer), r, c, 1)
            outer[r:-r, r:-r, r:-r] = new[r:-r, r:-r, r:-r]
            ops, recvs = [], []
            for peer, lo_side in ((tg["lo_rank"], True), (tg["hi_rank"], False)):
                if peer < 0:
                    continue
                zs = slice(r, r + tg["planes"]) if lo_side else slice(r + nzl - tg["planes"], r + nzl)
                sel = (zs, slice(r, -r), slice(r, -r))
                dst = (idx[sel] + (tg["lo_delta"] if lo_side else tg["hi_delta"])).ravel().astype(np.int64)
                vals = outer[sel].ravel().copy()
                n = dst.size
                ops.append(dist.P2POp(dist.isend, torch.from_numpy(dst), peer))
                ops.append(dist.P2POp(dist.isend, torch.from_numpy(vals), peer))
                ri = torch.empty(n, dtype=torch.int64)
                rv = torch.empty(n, dtype=torch.float64)
                ops.append(dist.P2POp(dist.irecv, ri, peer))
                ops.append(dist.P2POp(dist.irecv, rv, peer))
                recvs.append((ri, rv))
            for w in dist.batch_isend_irecv(ops) if ops else []:
                w.wait()
            for ri, rv in recvs:                                      # the neighbour's "peer stores"
                flat[ri.numpy()] = rv.numpy()
        interior = torch.from_numpy(np.ascontiguousarray(outer[r:-r, r:-r, r:-r]))
        sizes = [S.slab_partition(nz, world, k, r)[1] for k in range(world)]
        if rank == 0:
            parts = [interior] + [torch.empty((n, ny, nx), dtype=torch.float64) for n in sizes[1:]]
            for k in range(1, world):
                dist.recv(parts[k], k)
            got = torch.cat(parts).numpy()
            ref = oracle.sweep(g, r, c, iters)[r:-r, r:-r, r:-r]
            q.put(("ok", bool(np.array_equal(got, ref)), float(np.max(np.abs(got - ref)))))
        else:
            dist.send(interior, 0)
    except Exception as e:  # pragma: no cover
        q.put(("error", repr(e), 0.0))
        raise
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,nz,r", [(2, 11, 2), (3, 16, 3), (3, 13, 4)])
def test_p2p_fused_store_offsets_match_global_oracle(world, nz, r):
    from conftest import build_library
    build_library()
    import oracle
    oracle.build()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_p2p_worker, args=(k, world, port, 10, 6, nz, r, 3, q)) for k in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=240)
    assert all(p.exitcode == 0 for p in procs), [p.exitcode for p in procs]
    status, same, err = q.get(timeout=5)
    assert status == "ok", same
    assert same, f"p2p-decomposed result differs from the global oracle (max abs diff {err})"
