"""Inter-sweep gaps and CTA tails from in-kernel %globaltimer stamps (a STENCIL_TIMESTAMPS variant library).

    python tools/variant_lib.py ab_variants/ts.so -D STENCIL_TIMESTAMPS kern_f32_r4_ws.cu
    STENCIL_LIB=$PWD/ab_variants/ts.so python tools/ts_gaps.py inplane_ws:32,8,4,4,4,2,2,0

Per launch of a 100-sweep run: first CTA start to last CTA end (the launch's span), the spread of CTA start
and end times, and the gap from the previous launch's last CTA end to this launch's first CTA start.
"""
import ctypes
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import stencil_inputs as si  # noqa: E402
import paper_conf_ipps_tangtkwkgtw13_b200 as S  # noqa: E402
from paper_conf_ipps_tangtkwkgtw13_b200 import _lib as L  # noqa: E402

KEYS = ["tx", "ty", "rx", "ry", "stages", "zsegs", "zbox", "ytiles"]


def main():
    k, v = sys.argv[1].split(":")
    cfg = dict(zip(KEYS, [int(t) for t in v.split(",")]), kernel=k)
    iters = int(sys.argv[2]) if len(sys.argv) > 2 else 100
    n = 512
    fn = L.lib.stencil_dbg_timestamps
    fn.restype = ctypes.c_int
    buf = (ctypes.c_ulonglong * (4 * 32768))()
    cnt = ctypes.c_uint()
    with S.Plan(n, n, n, 4, si.coeffs_as("heat", 4, "f32"), "f32") as p:
        p.set_config(**cfg)
        x, y = p.alloc(), p.alloc()
        p.fill_counter(x, 2)
        for _ in range(3):
            p.run(x, y, iters)
        torch.cuda.synchronize()
        assert fn(buf, ctypes.byref(cnt)) == 0
        p.run(x, y, iters)
        torch.cuda.synchronize()
        assert fn(buf, ctypes.byref(cnt)) == 0
    m = cnt.value
    full = [(buf[4 * i], buf[4 * i + 1], buf[4 * i + 2], buf[4 * i + 3]) for i in range(m)]
    recs = [(a, b) for a, b, _, _ in full]
    ctas = m // iters
    launches = [recs[i * ctas:(i + 1) * ctas] for i in range(iters)]
    spans, gaps, start_spread, end_spread, work = [], [], [], [], []
    prev_end = None
    for ls in launches:
        s0 = min(a for a, _ in ls)
        s1 = max(a for a, _ in ls)
        e0 = min(b for _, b in ls)
        e1 = max(b for _, b in ls)
        spans.append((e1 - s0) / 1e3)
        start_spread.append((s1 - s0) / 1e3)
        end_spread.append((e1 - e0) / 1e3)
        work.append(statistics.mean((b - a) for a, b in ls) / 1e3)
        if prev_end is not None:
            gaps.append((s0 - prev_end) / 1e3)
        prev_end = e1
    total = (launches[-1] and max(b for _, b in launches[-1]) - min(a for a, _ in launches[0])) / 1e3
    out = {"cfg": sys.argv[1], "iters": iters, "ctas_per_launch": ctas,
           "total_us": round(total, 1), "per_sweep_us": round(total / iters, 2),
           "span_us_median": round(statistics.median(spans), 2),
           "gap_us_median": round(statistics.median(gaps), 2), "gap_us_max": round(max(gaps), 2),
           "cta_start_spread_us_median": round(statistics.median(start_spread), 2),
           "cta_end_spread_us_median": round(statistics.median(end_spread), 2),
           "cta_mean_work_us_median": round(statistics.median(work), 2)}
    out["idle_frac"] = round(1 - out["cta_mean_work_us_median"] / out["per_sweep_us"], 4)
    # per CTA (block index, SM): mean work and mean end offset from its launch's first start, over the run
    per = {}
    for li in range(iters):
        blk = full[li * ctas:(li + 1) * ctas]
        s0 = min(a for a, _, _, _ in blk)
        for a, b, bid, sm in blk:
            e = per.setdefault(bid, {"work": [], "end": [], "sm": set()})
            e["work"].append((b - a) / 1e3)
            e["end"].append((b - s0) / 1e3)
            e["sm"].add(sm)
    out["per_cta"] = {str(bid): {"work": round(statistics.mean(e["work"]), 2), "end": round(statistics.mean(e["end"]), 2),
                                 "sm": sorted(e["sm"])[:3]} for bid, e in sorted(per.items())}
    print(json.dumps(out))


if __name__ == "__main__":
    main()
