#!/usr/bin/env python3
"""Exhaustive tuning of one (n, r, dtype) case; prints the top configurations.

    python tools/tune_one.py --n 512 --r 4 --dtype f64 [--top 20] [--kernel inplane]
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=512)
    ap.add_argument("--r", type=int, default=4)
    ap.add_argument("--dtype", default="f64")
    ap.add_argument("--top", type=int, default=20)
    ap.add_argument("--kernel", default="inplane")
    ap.add_argument("--beta", type=float, default=100.0)
    ap.add_argument("--dump", default=None, help="write every timed entry (cfg, measured, regs, occupancy) here")
    a = ap.parse_args()
    import torch
    import paper_conf_ipps_tangtkwkgtw13_b200 as S
    import stencil_inputs as si
    n = a.n
    with S.Plan(n, n, n, a.r, si.coeffs_as("heat", a.r, a.dtype), a.dtype) as p:
        s0 = p.alloc()
        p.fill_counter(s0, 3)
        s1 = p.alloc()
        s1.copy_(s0)
        t0 = time.time()
        rep = p.tune(kernel=a.kernel, model="b200", beta=a.beta, iters_per_rep=4, reps=3, scratch=(s0, s1))
        res = p.tune_results()
        timed = sorted([e for e in res if e["measured_gpts"] > 0], key=lambda e: -e["measured_gpts"])
        print(json.dumps({"n": n, "r": a.r, "dtype": a.dtype, "M": rep["space_size"], "timed": len(timed),
                          "seconds": round(time.time() - t0, 1)}))
        if a.dump:
            with open(a.dump, "w") as f:
                json.dump({"n": n, "r": a.r, "dtype": a.dtype, "kernel": a.kernel, "entries": timed}, f)
        for e in timed[:a.top]:
            print(json.dumps({k: e[k] for k in ("cfg", "measured_gpts", "regs_per_thread", "active_blocks",
                                                "pred_b200_gpts", "pred_paper_gpts") if k in e}))


if __name__ == "__main__":
    main()
