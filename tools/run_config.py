"""Run `iters` sweeps of one configuration on a grid (for ncu captures).

    python tools/run_config.py --n 512 --nz 256 --r 4 --dtype f32 --iters 3 inplane_ws:16,16,4,4,4,2,2,0
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import stencil_inputs as si  # noqa: E402
import paper_conf_ipps_tangtkwkgtw13_b200 as S  # noqa: E402

KEYS = ["tx", "ty", "rx", "ry", "stages", "zsegs", "zbox", "ytiles"]
ap = argparse.ArgumentParser()
ap.add_argument("--n", type=int, default=512)
ap.add_argument("--nz", type=int, default=256)
ap.add_argument("--r", type=int, default=4)
ap.add_argument("--dtype", default="f32")
ap.add_argument("--iters", type=int, default=3)
ap.add_argument("cfg")
a = ap.parse_args()
k, v = a.cfg.split(":")
cfg = dict(zip(KEYS, [int(x) for x in v.split(",")]), kernel=k)
with S.Plan(a.n, a.n, a.nz, a.r, si.coeffs_as("heat", a.r, a.dtype), a.dtype) as p:
    p.set_config(**cfg)
    x, y = p.alloc(), p.alloc()
    p.fill_counter(x, 1)
    p.run(x, y, a.iters)
    torch.cuda.synchronize()
