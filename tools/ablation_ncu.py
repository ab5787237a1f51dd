"""ncu metrics of each kernel's best configuration from tools/ablation.py's JSON (run on the GPU box):
instructions per point, global-load sectors per request, DRAM bytes per launch, duration.

    python tools/ablation_ncu.py gpurun_out/ablation.json --r 4 > gpurun_out/ablation_ncu.json
"""
import argparse
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
METRICS = ["gpu__time_duration.sum", "smsp__inst_executed.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
           "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum",
           "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "lts__t_sectors_srcunit_tex_op_read.sum",
           "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active"]
KEYS = ["tx", "ty", "rx", "ry", "stages", "zsegs", "zbox", "ytiles"]

ap = argparse.ArgumentParser()
ap.add_argument("json")
ap.add_argument("--r", type=int, default=4)
a = ap.parse_args()
d = json.load(open(a.json))
row = next(x for x in d["rows"] if x["r"] == a.r)
n, _, nz = d["grid"]
out = {"grid": d["grid"], "r": a.r, "dtype": d["dtype"], "kernels": {}}
for k, v in row["kernels"].items():
    for which in ("tb", "rb"):
        if f"{which}_cfg" not in v:
            continue
        cfg = f"{k}:" + ",".join(str(v[f"{which}_cfg"][kk]) for kk in KEYS)
        cmd = ["ncu", "--metrics", ",".join(METRICS), "--clock-control", "none", "-k", "regex:sweep|ldg|inplane_ws|fp_tma",
               "-s", "1", "-c", "1", "--csv", sys.executable, os.path.join(ROOT, "tools", "run_config.py"),
               "--n", str(n), "--nz", str(nz), "--r", str(a.r), "--dtype", d["dtype"], "--iters", "3", cfg]
        p = subprocess.run(cmd, capture_output=True, text=True, timeout=600)
        rows = [r for r in csv.reader(io.StringIO(p.stdout)) if len(r) > 14 and r[0] != "ID"]
        m = {r[12]: r[14].replace(",", "") for r in rows}
        unit = {r[12]: r[13] for r in rows}
        def num(key):
            try:
                x = float(m[key])
            except (KeyError, ValueError):
                return None
            return x * {"Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "usecond": 1e-3, "msecond": 1.0,
                        "nsecond": 1e-6}.get(unit.get(key, ""), 1.0)
        pts = n * n * nz
        ent = {"cfg": cfg, "duration_ms": num("gpu__time_duration.sum"),
               "instr_per_point": (num("smsp__inst_executed.sum") or 0) * 32 / pts,
               "dram_bytes_per_launch": (num("dram__bytes_read.sum") or 0) + (num("dram__bytes_write.sum") or 0),
               "global_ld_sectors_per_request": ((num("l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum") or 0) /
                                                 max(1.0, num("l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum") or 0)),
               "l2_read_sectors_per_point": (num("lts__t_sectors_srcunit_tex_op_read.sum") or 0) / pts,
               "smem_bank_conflicts": num("l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum"),
               "fma_pipe_pct": num("sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active")}
        out["kernels"][f"{k}:{which}"] = ent
        print(k, which, ent, file=sys.stderr, flush=True)
print(json.dumps(out))
