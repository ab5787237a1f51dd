"""Sustained-clock A/B of sweep configurations: after a warm-up that brings the GPU to its power-capped
steady state, each configuration runs ~`--seconds` of back-to-back 100-sweep stencil_run calls per round,
rounds interleaved; reports mean ms per sweep, Gpts/s, median SM clock and board power per configuration.

    python tools/sustained_ab.py [--seconds 1.0] [--rounds 3] inplane_ws:32,8,4,4,4,2,2,0 ...
"""
import argparse
import json
import os
import statistics
import sys
import threading

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import stencil_inputs as si  # noqa: E402
import paper_conf_ipps_tangtkwkgtw13_b200 as S  # noqa: E402

KEYS = ["tx", "ty", "rx", "ry", "stages", "zsegs", "zbox", "ytiles"]


class Sampler:
    def __init__(self):
        import pynvml
        pynvml.nvmlInit()
        self.nv, self.h = pynvml, pynvml.nvmlDeviceGetHandleByIndex(torch.cuda.current_device())
        self.clk, self.pw, self.stop = [], [], threading.Event()

    def run(self):
        while not self.stop.is_set():
            self.clk.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
            self.pw.append(self.nv.nvmlDeviceGetPowerUsage(self.h) / 1000.0)
            self.stop.wait(0.02)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=512)
    ap.add_argument("--r", type=int, default=4)
    ap.add_argument("--dtype", default="f32")
    ap.add_argument("--seconds", type=float, default=1.0)
    ap.add_argument("--rounds", type=int, default=3)
    ap.add_argument("cfgs", nargs="+")
    a = ap.parse_args()
    n = a.n
    res = {c: {"ms": [], "clk": [], "pw": []} for c in a.cfgs}
    with S.Plan(n, n, n, a.r, si.coeffs_as("heat", a.r, a.dtype), a.dtype) as p:
        x, y = p.alloc(), p.alloc()
        p.fill_counter(x, 2)
        cfgs = []
        for c in a.cfgs:
            k, v = c.split(":")
            cfgs.append(dict(zip(KEYS, [int(t) for t in v.split(",")]), kernel=k))
        # warm-up: 2 s of the first configuration
        p.set_config(**cfgs[0])
        p.run(x, y, 100)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        p.run(x, y, 100)
        e1.record()
        e1.synchronize()
        ms100 = e0.elapsed_time(e1)
        for _ in range(max(1, int(2000 / ms100))):
            p.run(x, y, 100)
        torch.cuda.synchronize()
        for rd in range(a.rounds):
            order = list(zip(a.cfgs, cfgs)) if rd % 2 == 0 else list(reversed(list(zip(a.cfgs, cfgs))))
            for name, c in order:
                p.set_config(**c)
                p.run(x, y, 100)
                torch.cuda.synchronize()
                reps = max(1, int(a.seconds * 1000 / ms100))
                smp = Sampler()
                th = threading.Thread(target=smp.run, daemon=True)
                th.start()
                e0.record()
                for _ in range(reps):
                    p.run(x, y, 100)
                e1.record()
                e1.synchronize()
                smp.stop.set()
                th.join()
                res[name]["ms"].append(e0.elapsed_time(e1) / (100 * reps))
                res[name]["clk"] += smp.clk
                res[name]["pw"] += smp.pw
    pts = n ** 3
    out = {name: {"ms_per_sweep": round(statistics.mean(v["ms"]), 5),
                  "gpts": round(pts / (statistics.mean(v["ms"]) * 1e-3) / 1e9, 1),
                  "sm_mhz": statistics.median(v["clk"]) if v["clk"] else None,
                  "power_w": round(statistics.median(v["pw"]), 1) if v["pw"] else None,
                  "rounds_ms": [round(t, 5) for t in v["ms"]]} for name, v in res.items()}
    print(json.dumps({"n": n, "r": a.r, "dtype": a.dtype, "seconds": a.seconds, "res": out}))


if __name__ == "__main__":
    main()
