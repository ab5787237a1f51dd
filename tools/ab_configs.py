"""A/B of sweep configurations on one grid, interleaved so clock drift hits all alike.

    python tools/ab_configs.py [--n 512] [--r 4] [--dtype f32] [--iters 100] [--rounds 5] \
        inplane:16,16,4,4,4,2,2,0 inplane_ws:16,16,4,4,4,2,2,0 ...

Each round runs every configuration once (stencil_run of --iters sweeps, CUDA events on the
run stream); prints the median ms per sweep and Gpts/s per configuration as one JSON line.
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import stencil_inputs as si  # noqa: E402
import paper_conf_ipps_tangtkwkgtw13_b200 as S  # noqa: E402

KEYS = ["tx", "ty", "rx", "ry", "stages", "zsegs", "zbox", "ytiles"]


def parse(c):
    k, v = c.split(":")
    d = dict(zip(KEYS, [int(x) for x in v.split(",")]))
    d["kernel"] = k
    return d


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=512)
    ap.add_argument("--nz", type=int, default=0)
    ap.add_argument("--r", type=int, default=4)
    ap.add_argument("--dtype", default="f32")
    ap.add_argument("--iters", type=int, default=100)
    ap.add_argument("--rounds", type=int, default=5)
    ap.add_argument("cfgs", nargs="+")
    a = ap.parse_args()
    nz = a.nz or a.n
    cfgs = [parse(c) for c in a.cfgs]
    res = {c: [] for c in a.cfgs}
    with S.Plan(a.n, a.n, nz, a.r, si.coeffs_as("heat", a.r, a.dtype), a.dtype) as p:
        x, y = p.alloc(), p.alloc()
        p.fill_counter(x, 7)
        ref = None
        for name, c in zip(a.cfgs, cfgs):          # warm-up + agreement check
            p.set_config(**c)
            p.run(x, y, 2)
            torch.cuda.synchronize()
            if ref is None:
                ref = y.clone()
            elif not torch.equal(ref, y):
                print(f"MISMATCH {name}", file=sys.stderr)
        st = torch.cuda.current_stream()
        for _ in range(a.rounds):
            for name, c in zip(a.cfgs, cfgs):
                p.set_config(**c)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(st)
                p.run(x, y, a.iters)
                e1.record(st)
                e1.synchronize()
                res[name].append(e0.elapsed_time(e1) / a.iters)
    pts = a.n * a.n * nz
    out = {name: {"ms": round(statistics.median(v), 5), "gpts": round(pts / (statistics.median(v) * 1e-3) / 1e9, 1),
                  "min_ms": round(min(v), 5)} for name, v in res.items()}
    print(json.dumps({"n": a.n, "nz": nz, "r": a.r, "dtype": a.dtype, "iters": a.iters, "res": out}))


if __name__ == "__main__":
    main()
