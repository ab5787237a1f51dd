#!/usr/bin/env python3
"""Does the per-sweep time depend on the run length?  (diagnostic)

    python tools/drift.py [--config tx,ty,rx,ry,stages,zsegs,zbox,ytiles] > gpurun_out/drift.json

512^3 r=4 f32 (bench workload).  Runs of 1, 4, 20, 100 and 400 sweeps with
per-sweep CUDA events (timing mode 2), NVML power / SM clock sampled
throughout.  Prints one JSON line per run length.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


class Nvml:
    def __init__(self):
        import pynvml as nv
        nv.nvmlInit()
        self.nv, self.h = nv, nv.nvmlDeviceGetHandleByIndex(0)
        self.samples, self.stop = [], threading.Event()

    def _run(self):
        nv = self.nv
        while not self.stop.is_set():
            self.samples.append((nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM),
                                 nv.nvmlDeviceGetPowerUsage(self.h) / 1000.0,
                                 nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)))
            self.stop.wait(0.01)

    def __enter__(self):
        self.samples.clear()
        self.stop.clear()
        self.t = threading.Thread(target=self._run, daemon=True)
        self.t.start()
        return self

    def __exit__(self, *a):
        self.stop.set()
        self.t.join()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="32,8,4,4,4,2,2,18")
    ap.add_argument("--lengths", default="1,4,20,100,400")
    args = ap.parse_args()
    import torch
    import paper_conf_ipps_tangtkwkgtw13_b200 as S
    import stencil_inputs as si
    plan = S.Plan(512, 512, 512, 4, si.coeffs_as("heat", 4, "f32"), "f32")
    v = [int(x) for x in args.config.split(",")]
    plan.set_config(kernel="inplane", **dict(zip(["tx", "ty", "rx", "ry", "stages", "zsegs", "zbox", "ytiles"], v)))
    a, b = plan.alloc(), plan.alloc()
    plan.fill_counter(a, 2)
    plan.run(a, b, 10)
    torch.cuda.synchronize()
    mon = Nvml()
    for n in [int(x) for x in args.lengths.split(",")]:
        reps = max(1, 400 // n)
        plan.set_timing(2)
        with mon:
            for _ in range(reps):
                plan.run(a, b, n)
            torch.cuda.synchronize()
        st = plan.stats()
        plan.set_timing(0)
        clk = [c for c, _, _ in mon.samples]
        pw = [p for _, p, _ in mon.samples]
        reasons = 0
        for _, _, r in mon.samples:
            reasons |= r
        print(json.dumps({"sweeps_per_run": n, "runs": reps,
                          "avg_sweep_ms": round(st["timed_sweep_ms"] / st["timed_sweeps"], 5),
                          "min_sweep_ms": round(st["sweep_ms_min"], 5), "max_sweep_ms": round(st["sweep_ms_max"], 5),
                          "sm_mhz_median": statistics.median(clk) if clk else None, "sm_mhz_min": min(clk) if clk else None,
                          "power_w_median": statistics.median(pw) if pw else None, "power_w_max": max(pw) if pw else None,
                          "clock_event_reasons": hex(reasons)}), flush=True)
        torch.cuda.synchronize()
    plan.close()


if __name__ == "__main__":
    main()
