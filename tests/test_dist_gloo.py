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
