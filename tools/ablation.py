#!/usr/bin/env python3
"""Speedup breakdown in the spirit of the paper's Fig. 7 and Fig. 10 on
B200 -- SURVEY.md NEXT-2.

    python tools/ablation.py [--nz 256] [--dtype f32] [--radii 1,2,3,4] > gpurun_out/ablation.json

On the paper's 512 x 512 x 256 grid.  Every kernel is auto-tuned exhaustively over its own space
(stencil_tune, beta = 100 %) and reported at its best configuration with thread blocking only
(one point per thread in y, "TB") and with register blocking ("RB", the best over the whole space):
  fp            forward-plane, the SDK FDTD3d shape (K-FP); RB = register rows, Fig. 10 case (i)
  ip_classic    in-plane schedule, interior + four separate halo loads (Fig. 6a), per-thread loads
  ip_vertical   columns loaded with their top/bottom halos (Fig. 6b)
  ip_horizontal rows loaded with their left/right halos (Fig. 6c)
  ip_fullslice  the full slice, corners included (Fig. 6d)
  ip_fullslice_v  the full slice in 16-byte vectors (memory-level parallelism)
  fp_tma        forward-plane with K-IP's loads: full-slice TMA boxes, 16-byte column loads, register rows
                (the loading held fixed, so the gap to K-IP is the method: Fig. 10 (i) "+ the same loads")
  inplane       K-IP: the full slice as ONE TMA box per ZB planes (TB = one 16-byte vector of x-points
                and one row per thread)
  inplane_ws    K-IP warp-specialized (producer warpgroup), RB only
All kernels compute the same per-point order (bit-identical outputs, tests/test_parity_gpu.py).  The
rates are the tuner's short-run (boost clock) measurements -- the same conditions for every kernel.
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

KERNELS = ["forward", "ip_classic", "ip_vertical", "ip_horizontal", "ip_fullslice", "ip_fullslice_v", "fp_tma",
           "inplane", "inplane_ws"]
KEYS = ["tx", "ty", "rx", "ry", "stages", "zsegs", "zbox", "ytiles"]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--nz", type=int, default=256)
    ap.add_argument("--dtype", default="f32")
    ap.add_argument("--radii", default="1,2,3,4")
    args = ap.parse_args()
    import paper_conf_ipps_tangtkwkgtw13_b200 as S
    import stencil_inputs as si
    os.environ.setdefault("STENCIL_TUNE_SUSTAIN_MS", "0")   # burst ranking only: same conditions for all
    n, nz = 512, args.nz
    vec = 4 if args.dtype == "f32" else 2
    rows = []
    for r in [int(x) for x in args.radii.split(",")]:
        c = si.coeffs_as("heat", r, args.dtype)
        row = {"r": r, "order": 2 * r, "kernels": {}}
        with S.Plan(n, n, nz, r, c, args.dtype) as p:
            s0, s1 = p.alloc(), p.alloc()
            p.fill_counter(s0, 3)
            s1.copy_(s0)
            for k in KERNELS:
                try:
                    p.tune(kernel=k, model="b200", beta=100, iters_per_rep=4, reps=3, scratch=(s0, s1))
                except S.StencilError as e:
                    row["kernels"][k] = {"error": str(e)}
                    continue
                res = [e for e in p.tune_results() if e["measured_gpts"] > 0]
                tb_ok = (lambda e: e["cfg"]["ry"] == 1 and e["cfg"]["rx"] == vec) if k in ("inplane", "fp_tma") else \
                        (lambda e: e["cfg"]["ry"] == 1)
                tb = [e for e in res if tb_ok(e)]
                best = max(res, key=lambda e: e["measured_gpts"])
                out = {"M": len(res), "rb_gpts": round(best["measured_gpts"], 2),
                       "rb_cfg": {kk: best["cfg"][kk] for kk in KEYS}, "rb_regs": best["regs_per_thread"]}
                if tb and k != "inplane_ws":
                    b = max(tb, key=lambda e: e["measured_gpts"])
                    out.update({"tb_gpts": round(b["measured_gpts"], 2), "tb_cfg": {kk: b["cfg"][kk] for kk in KEYS}})
                row["kernels"][k] = out
                print(f"r={r} {k}: {out}", file=sys.stderr, flush=True)
        fp = row["kernels"].get("forward", {})
        for k, v in row["kernels"].items():
            if "tb_gpts" in v and fp.get("tb_gpts"):
                v["tb_speedup_vs_fp_tb"] = round(v["tb_gpts"] / fp["tb_gpts"], 3)
            if "rb_gpts" in v and fp.get("tb_gpts"):
                v["rb_speedup_vs_fp_tb"] = round(v["rb_gpts"] / fp["tb_gpts"], 3)
        rows.append(row)
    print(json.dumps({"grid": [n, n, nz], "dtype": args.dtype, "rows": rows}))


if __name__ == "__main__":
    main()
