"""Tune the per-rank slabs of BASELINE configs[4] (2048 x 2048 x 1024 f32 r=4, z-slabs over P = 2, 4, 8
GPUs) on one GPU and append the winners to tune_cache.txt (STENCIL_TUNE_CACHE), so that bench.py under
torchrun starts from tuned configurations:
  * plain slab extents (the NCCL-exchange DistPlan and rank-local plans, plan kind 0): both in-plane kernels;
  * the fused peer-store slab plan of rank 0 (plan kind 3, the PS variants of both in-plane kernels),
    unconnected -- tuning launches its sweeps with no peer stores.
    python tools/tune_c5_slabs.py [--beta 5]
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ.setdefault("STENCIL_TUNE_CACHE", os.path.join(ROOT, "tune_cache.txt"))

import torch  # noqa: E402

import stencil_inputs as si  # noqa: E402
import paper_conf_ipps_tangtkwkgtw13_b200 as S  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--beta", type=float, default=5.0)
ap.add_argument("--ranks", default="2,4,8")
a = ap.parse_args()
nx = ny = 2048
nz = 1024
c = si.coeffs_as("heat", 4, "f32")
for P in [int(x) for x in a.ranks.split(",")]:
    nzl = S.slab_partition(nz, P, 0, 4)[1]
    with S.Plan(nx, ny, nzl, 4, c, "f32") as p:
        s0, s1 = p.alloc(), p.alloc()
        p.fill_counter(s0, 5)
        s1.copy_(s0)
        for k in ("inplane_ws", "inplane"):
            rep = p.tune(kernel=k, beta=a.beta, iters_per_rep=2, reps=2, scratch=(s0, s1))
            print(f"P={P} plain {k}: {rep['best']} {rep['best_measured_gpts']:.1f} Gpts/s", flush=True)
    torch.cuda.empty_cache()
    q = S.P2PSlab(nx, ny, nz, 4, c, "f32", 0, P)
    try:
        s0, s1 = q.alloc(), q.alloc()
        q.fill_counter(s0, 5)
        s1.copy_(s0)
        for k in ("inplane_ws", "inplane"):
            rep = q.tune(kernel=k, beta=a.beta, iters_per_rep=2, reps=2, scratch=(s0, s1))
            print(f"P={P} p2p slab {k}: {rep['best']} {rep['best_measured_gpts']:.1f} Gpts/s", flush=True)
        del s0, s1
    finally:
        q.close()
    torch.cuda.empty_cache()
