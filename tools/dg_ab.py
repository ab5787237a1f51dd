"""Time Div / Grad (512^3) at fixed configurations, for library A/B runs (STENCIL_LIB=...).

    python tools/dg_ab.py grad f32 4 32,4,4,4,3,1,2 [reps]
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import stencil_inputs as si  # noqa: E402
import paper_conf_ipps_tangtkwkgtw13_b200 as S  # noqa: E402

app, dtype, r = sys.argv[1], sys.argv[2], int(sys.argv[3])
k = [int(x) for x in sys.argv[4].split(",")]
reps = int(sys.argv[5]) if len(sys.argv) > 5 else 200
cfg = dict(kernel="inplane_ws", tx=k[0], ty=k[1], rx=k[2], ry=k[3], stages=k[4], zsegs=k[5], zbox=k[6])
n = 512
with S.DivGrad(n, n, n, r, [float(x) for x in si.fd1_weights(r)], dtype, app=app) as p:
    bufs = [p.alloc() for _ in range(4)]
    for b in bufs:
        p.fill_counter(b, 3)
    p.set_config(**cfg)
    run = (lambda: p.div(*bufs)) if app == "div" else (lambda: p.grad(*bufs))
    for _ in range(20):
        run()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        run()
    e1.record()
    e1.synchronize()
    ms = e0.elapsed_time(e1) / reps
    print(json.dumps({"app": app, "dtype": dtype, "r": r, "cfg": sys.argv[4], "ms": round(ms, 5),
                      "gpts": round(n ** 3 / (ms * 1e-3) / 1e9, 1), "lib": os.environ.get("STENCIL_LIB", "")}))
