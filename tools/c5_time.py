"""Time BASELINE configs[4] (2048^2 x 1024 r=4 f32) on one GPU at the plan default configuration, sustained
(~2 s warm-up, then `reps` 20-sweep runs); for library / environment A/B runs.

    STENCIL_L2_PROMO=128 python tools/c5_time.py
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import stencil_inputs as si  # noqa: E402
import paper_conf_ipps_tangtkwkgtw13_b200 as S  # noqa: E402

nx, ny, nz, r = 2048, 2048, 1024, 4
reps = int(sys.argv[1]) if len(sys.argv) > 1 else 8
with S.Plan(nx, ny, nz, r, si.coeffs_as("heat", r, "f32"), "f32") as p:
    a, b = p.alloc(), p.alloc()
    p.fill_counter(a, 5)
    for _ in range(15):
        p.run(a, b, 20)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        p.run(a, b, 20)
    e1.record()
    e1.synchronize()
    ms = e0.elapsed_time(e1)
    print(json.dumps({"promo": os.environ.get("STENCIL_L2_PROMO", "default"), "cfg": p.config,
                      "gpts": round(nx * ny * nz * 20 * reps / (ms * 1e-3) / 1e9, 1)}))
