#!/usr/bin/env python3
"""Speedup breakdown in the spirit of the paper's Fig. 7 / Fig. 10 (P:L216-226,
P:L272-282) on B200 -- SURVEY NEXT-2 (measurement only; no new kernels).

    python tools/ablation.py [--nz 256] > gpurun_out/ablation.json

On the paper's 512 x 512 x 256 grid, f32, r = 1..4 (Table IV orders 2..8):
  FP      forward-plane, SDK FDTD3d shape (K-FP), best of its block shapes
  IP-TB   in-plane full-slice with THREAD blocking only: one 16-byte vector of
          x-points and one row per thread (rx = vec, ry = 1; the smallest tile
          our TMA/vector design allows), best over block shapes / ring depth
  IP-RB   in-plane + register blocking: the auto-tuner's pick (beta = 5 %,
          model-B) over the whole space
  IP-AX   the per-axis-coefficient variant at the tuner's pick (cost of
          reading R3b)
speedups: IP-TB / FP (the in-plane schedule + TMA loading), IP-RB / IP-TB
(register blocking), as the paper's Fig. 10 splits its gain.
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def time_run(plan, a, b, iters, reps=3):
    import torch
    plan.run(a, b, iters)
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        plan.run(a, b, iters)
        e1.record()
        e1.synchronize()
        ts.append(e0.elapsed_time(e1))
    return sorted(ts)[len(ts) // 2]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--nz", type=int, default=256)
    ap.add_argument("--iters", type=int, default=10)
    args = ap.parse_args()
    import torch
    import paper_conf_ipps_tangtkwkgtw13_b200 as S
    import stencil_inputs as si

    nx = ny = 512
    nz = args.nz
    pts = nx * ny * nz * args.iters
    rows = []
    for r in (1, 2, 3, 4):
        c = si.coeffs_as("heat", r, "f32")
        row = {"r": r, "order": 2 * r}
        with S.Plan(nx, ny, nz, r, c, "f32") as p:
            a, b = p.alloc(), p.alloc()
            p.fill_counter(a, 11)
            s0, s1 = p.alloc(), p.alloc()
            s0.copy_(a)
            s1.copy_(a)
            # FP: SDK shape over its block dims
            p.tune(kernel="forward", beta=100, iters_per_rep=2, reps=2, scratch=(s0, s1))
            row["FP_cfg"] = p.config
            row["FP"] = pts / (time_run(p, a, b, args.iters) * 1e-3) / 1e9
            # IP-TB: thread blocking only
            best, best_cfg = 0.0, None
            for tx in (16, 32, 64):
                for ty in (2, 4, 8, 16):
                    if tx * ty > 256 or tx * ty < 64:
                        continue
                    for stages in (3, 4, 6):
                        for zbox in (2, 4):
                            for zsegs in (1, 2, 4):
                                try:
                                    p.set_config(kernel="inplane", tx=tx, ty=ty, rx=4, ry=1, stages=stages,
                                                 zsegs=zsegs, zbox=zbox)
                                except S.StencilError:
                                    continue
                                v = pts / (time_run(p, a, b, args.iters, reps=1) * 1e-3) / 1e9
                                if v > best:
                                    best, best_cfg = v, p.config
            p.set_config(**{k: best_cfg[k] for k in ("kernel", "tx", "ty", "rx", "ry", "stages", "zsegs", "zbox",
                                                      "ytiles")})
            row["IP_TB_cfg"] = best_cfg
            row["IP_TB"] = pts / (time_run(p, a, b, args.iters) * 1e-3) / 1e9
            # IP-RB: the tuner's pick
            s0.copy_(a)
            s1.copy_(a)
            p.tune(kernel="inplane", model="b200", beta=5, iters_per_rep=2, reps=2, scratch=(s0, s1))
            rb_cfg = p.config
            row["IP_RB_cfg"] = rb_cfg
            row["IP_RB"] = pts / (time_run(p, a, b, args.iters) * 1e-3) / 1e9
            del s0, s1
        # IP-AX: per-axis coefficients at the same configuration where it is instantiated
        cax = si.coeffs_axes("heat_axes", r, "f32")
        with S.Plan(nx, ny, nz, r, cax, "f32") as p:
            a, b = p.alloc(), p.alloc()
            p.fill_counter(a, 11)
            try:
                p.set_config(**{k: rb_cfg[k] for k in ("kernel", "tx", "ty", "rx", "ry", "stages", "zsegs", "zbox",
                                                        "ytiles")})
                row["IP_AX_cfg"] = "same as IP_RB"
            except S.StencilError:
                s0, s1 = p.alloc(), p.alloc()
                s0.copy_(a)
                s1.copy_(a)
                p.tune(kernel="inplane", model="b200", beta=5, iters_per_rep=2, reps=2, scratch=(s0, s1))
                row["IP_AX_cfg"] = p.config
                del s0, s1
            row["IP_AX"] = pts / (time_run(p, a, b, args.iters) * 1e-3) / 1e9
        row["speedup_TB_over_FP"] = row["IP_TB"] / row["FP"]
        row["speedup_RB_over_TB"] = row["IP_RB"] / row["IP_TB"]
        row["speedup_total"] = row["IP_RB"] / row["FP"]
        rows.append(row)
        print(json.dumps(row), file=sys.stderr, flush=True)
        torch.cuda.empty_cache()
    print(json.dumps({"grid": [nx, ny, nz], "iters": args.iters, "unit": "Gpoints/s", "rows": rows}))


if __name__ == "__main__":
    main()
