"""Div / Grad on 512^3 (Table V application stencils; BASELINE configs[2] style): every registered tile
shape at a few segment counts, best of them, for r = 1..4 in f32 and f64.  Algorithmic bytes per point:
4 s (three grids read + one written, or one read + three written).

    python tools/divgrad_bench.py > gpurun_out/divgrad.json
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import stencil_inputs as si  # noqa: E402
import paper_conf_ipps_tangtkwkgtw13_b200 as S  # noqa: E402


def timed(fn, reps=10):
    fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    e1.synchronize()
    return e0.elapsed_time(e1) / reps


peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"] if os.path.exists(
    os.path.join(ROOT, "MEASURED_PEAKS.json")) else 6650.0
n = 512
rows = []
for dtype in ("f32", "f64"):
    s = 4 if dtype == "f32" else 8
    vec = 16 // s
    for r in (1, 2, 3, 4):
        a = [float(x) for x in si.fd1_weights(r)]
        for app in ("div", "grad"):
            with S.DivGrad(n, n, n, r, a, dtype, app=app) as p:
                bufs = [p.alloc() for _ in range(4)]
                for b in bufs:
                    p.fill_counter(b, 3)
                run = (lambda: p.div(*bufs)) if app == "div" else (lambda: p.grad(*bufs))
                best = None
                for tx in (16, 32):
                    for ry in (2, 4):
                        for warps in (8, 4):
                            for stages in (2, 3, 4):
                                for zsegs in (1, 2, 3):
                                    cfg = dict(kernel="inplane_ws", tx=tx, ty=warps * 32 // tx, rx=vec, ry=ry,
                                               stages=stages, zsegs=zsegs, zbox=2)
                                    try:
                                        p.set_config(**cfg)
                                    except S.StencilError:
                                        continue
                                    ms = timed(run, 5)
                                    if best is None or ms < best[0]:
                                        best = (ms, cfg)
                p.set_config(**best[1])
                ms = timed(run, 20)
                gpts = n ** 3 / (ms * 1e-3) / 1e9
                row = {"app": app, "dtype": dtype, "r": r, "ms": round(ms, 4), "gpts": round(gpts, 1),
                       "alg_GBs": round(gpts * 4 * s, 1), "frac_of_copy": round(gpts * 4 * s / peak, 3),
                       "cfg": best[1]}
                print(row, file=sys.stderr, flush=True)
                rows.append(row)
print(json.dumps({"grid": [n, n, n], "peak_GBs": peak, "rows": rows}))
