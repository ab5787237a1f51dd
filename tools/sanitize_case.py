"""Small runs of every kernel family for compute-sanitizer (memcheck / racecheck / synccheck).

    compute-sanitizer --tool racecheck python tools/sanitize_case.py [case ...]
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import stencil_inputs as si  # noqa: E402
import paper_conf_ipps_tangtkwkgtw13_b200 as S  # noqa: E402

CASES = {
    "ip_f32_r4": ("f32", 4, (37, 21, 17), dict(kernel="inplane", tx=16, ty=2, rx=4, ry=2, stages=3, zsegs=2, zbox=2)),
    "ip_f32_r4_full": ("f32", 4, (64, 16, 17), dict(kernel="inplane", tx=16, ty=2, rx=4, ry=2, stages=3, zsegs=2, zbox=2)),
    "ip_f32_r4_z1": ("f32", 4, (37, 21, 17), dict(kernel="inplane", tx=16, ty=2, rx=4, ry=2, stages=3, zsegs=1, zbox=1)),
    "ip_f32_r1_yt": ("f32", 1, (37, 21, 17), dict(kernel="inplane", tx=16, ty=2, rx=8, ry=1, stages=2, zsegs=1, zbox=1, ytiles=11)),
    "ip_f64_r3": ("f64", 3, (37, 21, 17), dict(kernel="inplane", tx=16, ty=4, rx=2, ry=4, stages=4, zsegs=3, zbox=4)),
    "fp_f32_r4": ("f32", 4, (37, 21, 17), dict(kernel="forward", tx=16, ty=4, rx=1, ry=1, stages=1, zsegs=1)),
    # warp-specialized in-plane (producer warpgroup, full/empty ring as CUTLASS PipelineTmaAsync)
    "ws_f32_r4": ("f32", 4, (70, 41, 21), dict(kernel="inplane_ws", tx=16, ty=4, rx=4, ry=4, stages=3, zsegs=2, zbox=2)),
    "ws_f32_r4_full": ("f32", 4, (64, 32, 21), dict(kernel="inplane_ws", tx=16, ty=4, rx=4, ry=4, stages=3, zsegs=2, zbox=1)),
    "ws_f64_r2": ("f64", 2, (37, 21, 17), dict(kernel="inplane_ws", tx=32, ty=4, rx=2, ry=2, stages=4, zsegs=1, zbox=4)),
    # forward-plane with the in-plane kernel's TMA ring (two cursors, stages >= ceil(r/zbox) + 2)
    "fpt_f32_r4": ("f32", 4, (70, 41, 21), dict(kernel="fp_tma", tx=16, ty=4, rx=4, ry=2, stages=4, zsegs=2, zbox=2)),
    "fpt_f64_r3": ("f64", 3, (37, 21, 17), dict(kernel="fp_tma", tx=16, ty=4, rx=2, ry=1, stages=5, zsegs=1, zbox=1)),
}
# fused peer-store slabs, three in one process (warp-specialized and classic PS kernels)
P2P_CASES = {
    "ps_ws_f32_r2": ("f32", 2, (64, 16, 29), dict(kernel="inplane_ws", tx=16, ty=4, rx=4, ry=2, stages=3, zsegs=2, zbox=2)),
    "ps_ip_f32_r2": ("f32", 2, (37, 21, 29), dict(kernel="inplane", tx=16, ty=2, rx=4, ry=2, stages=3, zsegs=2, zbox=2)),
}


def run_p2p(dtype, r, shape, cfg, P=3):
    nx, ny, nz = shape
    u = si.uniform(nx, ny, nz, r, seed=2, dtype=dtype)
    c = si.coeffs_as("heat", r, dtype)
    plans = [S.P2PSlab(nx, ny, nz, r, c, dtype, k, P) for k in range(P)]
    for k, q in enumerate(plans):
        q.connect(plans[k - 1] if k > 0 else None, plans[k + 1] if k < P - 1 else None)
        q.set_config(**cfg)
        q.fill_local(u)
    torch.cuda.synchronize()
    streams = [torch.cuda.Stream() for _ in range(P)]
    for q, st in zip(plans, streams):
        q.run(3, stream=st)
    torch.cuda.synchronize()
    for q in plans:
        assert np.isfinite(q.local_result()).all()
        q.close()



names = sys.argv[1:] or list(CASES) + list(P2P_CASES)
for name in names:
    if name in P2P_CASES:
        run_p2p(*P2P_CASES[name])
        print("case done:", name, flush=True)
        continue
    dtype, r, (nx, ny, nz), cfg = CASES[name]
    u = si.uniform(nx, ny, nz, r, seed=1, dtype=dtype)
    with S.Plan(nx, ny, nz, r, si.coeffs_as("heat", r, dtype), dtype) as p:
        p.set_config(**cfg)
        a, b = p.upload(u), p.alloc()
        p.run(a, b, 3)
        torch.cuda.synchronize()
        assert np.isfinite(p.download(b)).all()
    print("case done:", name, flush=True)
