#!/usr/bin/env python3
"""BASELINE configs[0] (64^3, r = 1, f32, 10 iterations) -- a launch-bound run.

    python tools/c1_bench.py > gpurun_out/c1.json

Times stencil_run(in, out, 10) (median of 50, CUDA events on the caller's
stream) with the model's default configuration and with the exhaustively tuned
one, with CUDA-graph replay (default) and with STENCIL_GRAPHS=0 (one launch per
sweep), and checks the result against the oracle.
"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def leg():
    import numpy as np
    import torch
    import oracle
    import stencil_inputs as si
    import paper_conf_ipps_tangtkwkgtw13_b200 as S
    n, r, iters = 64, 1, 10
    u = si.uniform(n, n, n, r, seed=1, dtype="f32")
    c = si.coeffs_as("heat", r, "f32")
    res = {}
    with S.Plan(n, n, n, r, c, "f32") as p:
        a, b = p.upload(u), p.alloc()
        for name in ("default", "tuned"):
            if name == "tuned":
                s0, s1 = p.alloc(), p.alloc()
                s0.copy_(a)
                s1.copy_(a)
                p.tune(kernel="inplane", beta=100, iters_per_rep=10, reps=5, scratch=(s0, s1))
            for _ in range(3):
                p.run(a, b, iters)
            torch.cuda.synchronize()
            ts = []
            for _ in range(50):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                p.run(a, b, iters)
                e1.record()
                e1.synchronize()
                ts.append(e0.elapsed_time(e1))
            ms = sorted(ts)[len(ts) // 2]
            g = p.download(b).astype(np.float64)
            o = oracle.sweep(u, r, c, iters)
            err = float(np.max(np.abs(g[1:-1, 1:-1, 1:-1] - o[1:-1, 1:-1, 1:-1]) / np.abs(o[1:-1, 1:-1, 1:-1])))
            res[name] = {"config": p.config, "ms_per_run": round(ms, 4), "us_per_sweep": round(ms * 100, 2),
                         "gpts": round(n ** 3 * iters / (ms * 1e-3) / 1e9, 2), "max_rel_err": err}
    return res


def main():
    if len(sys.argv) > 1 and sys.argv[1] == "--leg":
        print(json.dumps(leg()))
        return
    out = {"workload": "c1: 64^3 r=1 f32 heat stencil, 10 iterations per stencil_run"}
    for graphs in ("1", "0"):
        env = dict(os.environ, STENCIL_GRAPHS=graphs)
        p = subprocess.run([sys.executable, __file__, "--leg"], env=env, capture_output=True, text=True, cwd=ROOT)
        out["graphs" if graphs == "1" else "no_graphs"] = json.loads(p.stdout) if p.returncode == 0 else p.stderr[-2000:]
    print(json.dumps(out))


if __name__ == "__main__":
    main()
