#!/usr/bin/env python3
"""BASELINE.json configs 1, 3 and 4 on one GPU (the bench.py line is config 2).

    python tools/configs_bench.py [--quick] > gpurun_out/configs.json

C1  64^3 r=1 f32, 10 iterations: time per stencil_run (launch-bound) + oracle parity
C3  512^3 heat stencils r = 1..6 (Table IV orders 2..12) and the leapfrog 3D wave
    (application stencil, 3 grids of traffic per point) in f32 and f64, 20-21
    iterations per run, in-plane (tuned, beta = 5 %, model-B) vs forward-plane
    (tuned over its block shapes)
C4  auto-tuning sweep r = 1, 2, 4 on 256^3, 512^3, 768^3 (f32): exhaustive search,
    then what beta = 5 % pruning with model-P (paper Eqs. 6-14) and model-B would
    have picked, and the Spearman rank correlation of each model with measurement
"""
from __future__ import annotations

import argparse
import json
import math
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def spearman(a, b):
    def ranks(x):
        order = sorted(range(len(x)), key=lambda i: x[i])
        r = [0.0] * len(x)
        for k, i in enumerate(order):
            r[i] = k
        return r
    ra, rb = ranks(a), ranks(b)
    n = len(a)
    ma, mb = sum(ra) / n, sum(rb) / n
    cov = sum((x - ma) * (y - mb) for x, y in zip(ra, rb))
    va = math.sqrt(sum((x - ma) ** 2 for x in ra))
    vb = math.sqrt(sum((y - mb) ** 2 for y in rb))
    return cov / (va * vb) if va and vb else float("nan")


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


def time_call(fn, reps=3):
    import torch
    fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        e1.synchronize()
        ts.append(e0.elapsed_time(e1))
    return sorted(ts)[len(ts) // 2]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--quick", action="store_true")
    ap.add_argument("--c4", action="store_true", help="also run the exhaustive C4 sweeps (~10 min)")
    ap.add_argument("--c4-only", action="store_true", help="only the C4 sweeps")
    args = ap.parse_args()
    import numpy as np
    import torch
    import oracle
    import stencil_inputs as si
    import paper_conf_ipps_tangtkwkgtw13_b200 as S

    out = {"device": torch.cuda.get_device_name(0)}
    if args.c4_only:
        args.c4 = True
        return c4_sweeps(args, out, S, si)
    # ---- C1
    n, r = 64, 1
    u = si.uniform(n, n, n, r, seed=1, dtype="f32")
    c = si.coeffs_as("heat", r, "f32")
    with S.Plan(n, n, n, r, c, "f32") as p:
        a, b = p.upload(u), p.alloc()
        ms = time_run(p, a, b, 10, reps=10)
        g = p.download(b).astype(np.float64)
    o = oracle.sweep(u, r, c, 10)
    err = float(np.max(np.abs(g[1:-1, 1:-1, 1:-1] - o[1:-1, 1:-1, 1:-1]) / np.abs(o[1:-1, 1:-1, 1:-1])))
    out["c1"] = {"ms_per_run_10_iters": ms, "gpts": n ** 3 * 10 / (ms * 1e-3) / 1e9, "max_rel_err": err}
    print(json.dumps({"c1": out["c1"]}), file=sys.stderr, flush=True)

    # ---- C3: heat stencils r = 1..6 (Table IV orders 2..12) and the application stencils
    c3 = []
    for app in ["jacobi", "wave"]:
        for dtype in ["f32", "f64"]:
            for r in ([1, 2, 3, 4, 5, 6] if app == "jacobi" else [1, 2, 4]):
                n = 512
                s = 4 if dtype == "f32" else 8
                if app == "jacobi":
                    coeffs = si.coeffs_as("heat", r, dtype)
                    kw = {}
                else:  # leapfrog u_tt = Lap u, k = 1/16: c0 = 2 + k 3a_0, c_m = k a_m, d = -1
                    a = si.fd_weights(r)
                    coeffs = np.array([2 + 3 * float(a[0]) / 16] + [float(a[m]) / 16 for m in range(1, r + 1)])
                    kw = dict(app="wave", d=-1.0)
                with S.Plan(n, n, n, r, coeffs, dtype, **kw) as p:
                    a0 = p.alloc()
                    p.fill_counter(a0, 3)
                    b0 = p.alloc()
                    s0, s1 = p.alloc(), p.alloc()
                    s0.copy_(a0)
                    s1.copy_(a0)
                    t0 = time.time()
                    run = (lambda: p.run(a0, b0, 20)) if app == "jacobi" else (lambda: p.run_wave(a0, b0, 21))
                    # the in-plane family: the classic kernel and (plain sweeps) the warp-specialized one
                    best_ip = None
                    for kern in (["inplane_ws", "inplane"] if app == "jacobi" else ["inplane"]):
                        rep = p.tune(kernel=kern, model="b200", beta=5, iters_per_rep=4, reps=3, scratch=(s0, s1))
                        ms = time_call(run)
                        if best_ip is None or ms < best_ip[0]:
                            best_ip = (ms, p.config, rep)
                    t_tune = time.time() - t0
                    ms_ip, cfg_ip, rep = best_ip
                    p.set_config(**cfg_ip)
                    p.tune(kernel="forward", model="b200", beta=0, iters_per_rep=2, reps=2, scratch=(s0, s1))
                    cfg_fp = p.config
                    ms_fp = time_call(run)
                    del s0, s1
                its = 20 if app == "jacobi" else 21
                grids = 2 if app == "jacobi" else 3
                row = {"app": app, "dtype": dtype, "r": r, "inplane_gpts": n ** 3 * its / (ms_ip * 1e-3) / 1e9,
                       "inplane_GBs": grids * s * n ** 3 * its / (ms_ip * 1e-3) / 1e9, "inplane_cfg": cfg_ip,
                       "forward_gpts": n ** 3 * its / (ms_fp * 1e-3) / 1e9, "forward_cfg": cfg_fp,
                       "speedup": ms_fp / ms_ip, "tune_M": rep["space_size"], "tune_N": rep["timed"],
                       "tune_seconds": t_tune}
                c3.append(row)
                print(json.dumps(row), file=sys.stderr, flush=True)
                torch.cuda.empty_cache()
    out["c3"] = c3
    if not args.c4:
        print(json.dumps(out))
        return

    c4_sweeps(args, out, S, si)


def c4_sweeps(args, out, S, si):
    import torch
    os.environ["STENCIL_TUNE_SUSTAIN_MS"] = "0"   # every candidate under the same short-run conditions
    # ---- C4: both in-plane kernels (classic and warp-specialized), each over its own space
    c4 = []
    shapes = [256, 512] if args.quick else [256, 512, 768]
    for n in shapes:
        for r, kern in [(r, k) for r in [1, 2, 4] for k in ("inplane", "inplane_ws")]:
            coeffs = si.coeffs_as("avg", r, "f32")
            with S.Plan(n, n, n, r, coeffs, "f32") as p:
                s0 = p.alloc()
                p.fill_counter(s0, 4)
                s1 = p.alloc()
                s1.copy_(s0)
                t0 = time.time()
                p.tune(kernel=kern, model="b200", beta=100, iters_per_rep=3, reps=2, scratch=(s0, s1))
                secs = time.time() - t0
                res = p.tune_results()
            meas = [e["measured_gpts"] for e in res]
            best = max(meas)
            nb = max(1, math.ceil(0.05 * len(res)))
            row = {"n": n, "r": r, "kernel": kern, "M": len(res), "N_beta5": nb, "exhaustive_best_gpts": best,
                   "exhaustive_seconds": secs}
            for key, name in (("pred_paper_gpts", "model_paper"), ("pred_b200_gpts", "model_b200")):
                order = sorted(res, key=lambda e: -e[key])
                pick = max(e["measured_gpts"] for e in order[:nb])
                row[f"{name}_beta5_frac"] = pick / best
                row[f"{name}_spearman"] = spearman([e[key] for e in res], meas)
            bestcfg = max(res, key=lambda e: e["measured_gpts"])["cfg"]
            row["best_cfg"] = bestcfg
            c4.append(row)
            print(json.dumps(row), file=sys.stderr, flush=True)
            torch.cuda.empty_cache()
    out["c4"] = c4
    print(json.dumps(out))


if __name__ == "__main__":
    main()
