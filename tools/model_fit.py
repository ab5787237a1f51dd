#!/usr/bin/env python3
"""Evaluate the auto-tuner's performance models against exhaustive measurements.

    python tools/model_fit.py [profiles/tune_space/*.csv.gz]

Each file holds every configuration of one (n, r, dtype) search space timed on
a B200 (tools/tune_one.py --dump, compacted).  For model-P (Eqs. 6-14) and
model-B (csrc/tune.cu) the library's own implementations are called through
the C ABI, and the script reports what beta = 5 % pruning would have picked
(fraction of the exhaustive best, the P:L374 criterion) and the Spearman rank
correlation with the measurement.
"""
from __future__ import annotations

import csv
import ctypes
import glob
import gzip
import math
import os
import re
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def load(path):
    rows = list(csv.DictReader(gzip.open(path, "rt")))
    return [{k: float(v) for k, v in r.items()} for r in rows]


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


def b200_params(L):
    g = L.GpuParams()
    g.sm, g.bw, g.smem, g.reg, g.blk_sm, g.warp_sm = 148, 0.8 * 2 * 3.996e9 * 1024, 233472, 65536, 32, 64
    g.lat_cycles, g.clock_hz = 600.0, 1.965e9
    return g


def main():
    from paper_conf_ipps_tangtkwkgtw13_b200 import _lib as L
    files = sys.argv[1:] or sorted(glob.glob(os.path.join(ROOT, "profiles", "tune_space", "*.csv.gz")))
    gp = b200_params(L)
    print(f"{'case':<14}{'M':>7}{'best':>8}  {'P beta5':>8}{'P rho':>7}  {'B beta5':>8}{'B rho':>7}")
    tot = {"P": [], "B": []}
    for f in files:
        m = re.search(r"n(\d+)_r(\d+)_(f\d+)", os.path.basename(f))
        n, r, dt = int(m.group(1)), int(m.group(2)), m.group(3)
        s = 4 if dt == "f32" else 8
        rows = load(f)
        meas = [e["measured_gpts"] for e in rows]
        best = max(meas)
        preds = {"P": [], "B": []}
        for e in rows:
            k = L.ModelKernel()
            k.lx = k.ly = k.lz = n
            k.tx, k.ty, k.rx, k.ry = int(e["tx"]), int(e["ty"]), int(e["rx"]), int(e["ry"])
            k.radius, k.elem_size, k.regs_per_thread = r, s, int(e["regs"])
            k.smem_per_block = 0
            k.ops_per_point = 8 * r + 1
            k.stages, k.zbox, k.zsegs = int(e["stages"]), int(e["zbox"]), int(e["zsegs"])
            k.ytiles, k.active_blocks, k.inputs = int(e["ytiles"]), int(e["active_blocks"]), 1
            preds["B"].append(L.lib.stencil_model_b200(ctypes.byref(gp), ctypes.byref(k)))
            preds["P"].append(e["pred_paper"])
        nb = max(1, math.ceil(0.05 * len(rows)))
        out = []
        for key in ("P", "B"):
            order = sorted(range(len(rows)), key=lambda i: -preds[key][i])
            pick = max(meas[i] for i in order[:nb]) / best
            rho = spearman(preds[key], meas)
            tot[key].append(pick)
            out += [pick, rho]
        print(f"n{n} r{r} {dt:<6}{len(rows):>7}{best:>8.1f}  {out[0]:>8.3f}{out[1]:>7.2f}  {out[2]:>8.3f}{out[3]:>7.2f}")
    for key in ("P", "B"):
        v = tot[key]
        print(f"model-{key}: beta=5% pick / exhaustive best: mean {sum(v) / len(v):.3f}, worst {min(v):.3f}")


if __name__ == "__main__":
    main()
