"""Small runs of the round-1 additions for compute-sanitizer memcheck:
per-axis (AX) kernels, fused peer-store slabs (PS, 3 slabs in one process),
the stop-criterion residual kernel, CUDA-graph replay and the pipelined
host-to-host path.

    compute-sanitizer --tool memcheck python tools/sanitize_new.py
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import stencil_inputs as si  # noqa: E402
import paper_conf_ipps_tangtkwkgtw13_b200 as S  # noqa: E402

r, dtype = 2, "f32"
nx, ny, nz = 37, 21, 19
u = si.uniform(nx, ny, nz, r, seed=1, dtype=dtype)
# per-axis kernels
with S.Plan(nx, ny, nz, r, si.coeffs_axes("heat_axes", r, dtype), dtype) as p:
    p.set_config(kernel="inplane", tx=16, ty=3, rx=4, ry=2, stages=3, zsegs=2, zbox=2, ytiles=5)
    a, b = p.upload(u), p.alloc()
    p.run(a, b, 3)
    p.set_config(kernel="forward", tx=32, ty=4, rx=1, ry=1, stages=1, zsegs=1)
    p.run(a, b, 2)
# stop criterion, graphs, host-to-host
c = si.coeffs_as("heat", r, dtype)
with S.Plan(nx, ny, nz, r, c, dtype) as p:
    a, b = p.upload(u), p.alloc()
    p.run_until(a, b, 7, 1e-3, 2)
    p.run(a, b, 4)
    p.run(a, b, 4)                          # graph replay
    h_in = torch.empty(a.numel(), dtype=a.dtype, pin_memory=True)
    h_in.copy_(a)
    h_out = torch.empty_like(h_in).pin_memory()
    s = torch.cuda.current_stream()
    for _ in range(3):
        p.run_host(h_in, h_out, 3, stream=s)
    p.host_wait(stream=s)
# fused peer-store slabs
P = 3
plans = [S.P2PSlab(nx, ny, 4 * P * r, r, c, dtype, k, P) for k in range(P)]
ug = si.uniform(nx, ny, 4 * P * r, r, seed=2, dtype=dtype)
for k, q in enumerate(plans):
    q.connect(plans[k - 1] if k > 0 else None, plans[k + 1] if k < P - 1 else None)
    q.fill_local(ug)
torch.cuda.synchronize()
streams = [torch.cuda.Stream() for _ in range(P)]
for q, st in zip(plans, streams):
    q.run(5, stream=st)
for q, st in zip(plans, streams):
    q.residual(stream=st)
torch.cuda.synchronize()
for q in plans:
    q.close()
print("sanitize_new done")
