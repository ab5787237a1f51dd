#!/usr/bin/env python3
"""Summarise the ncu outputs of tools/profile.sh into profiles/ (tracked).

    python tools/ncu_summary.py --tag r1 --cfg inplane:16,16,4,4,4,2,2,9

Writes
  profiles/<tag>_launches.csv / .txt   every launch of a short bench run and each kernel's share of the step
  profiles/<tag>_inplane_ncu.txt       --set full summary of the in-plane sweep (SOL, memory, stalls, mix)
  profiles/<tag>_forward_ncu.txt       the same for the forward-plane baseline
  profiles/ncu_traffic.json            dram bytes per launch per config (bench.py roofline.traffic)
"""
from __future__ import annotations

import argparse
import collections
import csv
import io
import json
import os
import re
import shutil
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "gpurun_out")
PROF = os.path.join(ROOT, "profiles")

KEYS = [
    ("gpu__time_duration.sum", "duration"),
    ("sm__cycles_elapsed.avg.per_second", "SM clock"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("dram__throughput.avg.pct_of_peak_sustained_elapsed", "DRAM throughput % of peak"),
    ("lts__t_sectors_srcunit_tex_op_read.sum", "L2 read sectors (from SMs)"),
    ("lts__t_sector_op_read_hit_rate.pct", "L2 read hit rate"),
    ("lts__t_sectors_srcunit_ltcfabric.sum", "L2 cross-die fabric sectors"),
    ("smsp__inst_executed.sum", "warp instructions"),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue active %"),
    ("sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active", "FMA pipe active %"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps active % (occupancy)"),
    ("launch__registers_per_thread", "registers/thread"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
    ("launch__shared_mem_per_block_dynamic", "dynamic smem/block"),
    ("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "smem wavefronts"),
    ("l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "smem bank conflicts"),
]


def ncu_csv(args):
    out = subprocess.run(["ncu", *args, "--csv"], capture_output=True, text=True).stdout
    return list(csv.reader(io.StringIO(out)))


def raw_metrics(rep):
    rows = ncu_csv(["-i", rep, "--page", "raw"])
    return {h: (u, v) for h, u, v in zip(rows[0], rows[1], rows[2])}


def source_mix(rep, points):
    rows = ncu_csv(["-i", rep, "--page", "source", "--print-source", "sass"])
    h = rows[1]
    iS, iE = h.index("Source"), h.index("Instructions Executed")
    iA = h.index("Warp Stall Sampling (All Samples)")
    op, st = collections.Counter(), collections.Counter()
    for r in rows[2:]:
        if len(r) <= iA:
            continue
        m = re.match(r"(@!?U?P\w+\s+)?([A-Z0-9]+)", r[iS].strip())
        if m:
            op[m.group(2)] += int(r[iE] or 0)
            st[m.group(2)] += int(r[iA] or 0)
    tot_s = max(1, sum(st.values()))
    lines = [f"instructions per interior point (thread-level): {sum(op.values()) * 32 / points:.2f}"]
    for k, v in op.most_common(16):
        lines.append(f"  {k:8s} {v * 32 / points:6.2f}/pt   stall samples {100 * st[k] / tot_s:5.1f}%")
    return lines


def summarise(rep, title, points):
    d = raw_metrics(rep)
    lines = [f"# {title}", f"# source: {os.path.basename(rep)} (ncu --set full --clock-control none)", ""]
    for k, name in KEYS:
        if k in d:
            lines.append(f"{name:32s} {d[k][1]:>18s} {d[k][0]}  [{k}]")
    stalls = {k: v for k, v in d.items()
              if k.startswith("smsp__average_warps_issue_stalled_") and k.endswith("_per_issue_active.ratio")}
    top = sorted(((float(v[1]) if v[1] not in ("", "n/a") else 0.0, k) for k, v in stalls.items()), reverse=True)[:8]
    lines += ["", "warp stall reasons (cycles per issued instruction):"]
    for val, k in top:
        lines.append(f"  {k[len('smsp__average_warps_issue_stalled_'):-len('_per_issue_active.ratio')]:24s} {val:.3f}")
    lines += [""] + source_mix(rep, points)
    return lines, d


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--tag", default="r1")
    ap.add_argument("--cfg", default="inplane:16,16,4,4,4,2,2,9")
    ap.add_argument("--points", type=int, default=512 ** 3)
    a = ap.parse_args()
    os.makedirs(PROF, exist_ok=True)
    # 1. launch list
    lc = os.path.join(OUT, f"launches_{a.tag}.csv")
    if os.path.exists(lc):
        shutil.copy(lc, os.path.join(PROF, f"{a.tag}_launches.csv"))
        rows = [r for r in csv.reader(open(lc)) if len(r) > 12 and r[0] != "ID"]
        per = collections.defaultdict(list)
        for r in rows:
            if r[12] == "gpu__time_duration.sum":
                name = re.sub(r"\(.*", "", r[4]).replace("void ", "")
                per[name].append(float(r[14]))
        tot = sum(sum(v) for v in per.values())
        with open(os.path.join(PROF, f"{a.tag}_launches.txt"), "w") as f:
            f.write("# every kernel launch of `bench.py --profile --iters 10 --steps 2 --warmup 1` under\n"
                    "# ncu --metrics gpu__time_duration.sum --clock-control none (cold-cache, serialised: compare shares)\n")
            for name, v in sorted(per.items(), key=lambda kv: -sum(kv[1])):
                f.write(f"{name:70s} launches {len(v):4d}  total {sum(v)/1e3:9.1f} us  "
                        f"mean {sum(v)/len(v)/1e3:8.2f} us  share {100*sum(v)/tot:5.1f}%\n")
    # 2. full reports
    traffic = {}
    tp = os.path.join(PROF, "ncu_traffic.json")
    if os.path.exists(tp):
        traffic = json.load(open(tp))
    for kind, rep in (("inplane", f"inplane_{a.tag}.ncu-rep"), ("forward", f"forward_{a.tag}.ncu-rep")):
        path = os.path.join(OUT, rep)
        if not os.path.exists(path):
            continue
        lines, d = summarise(path, f"{kind} sweep kernel, 512^3 r=4 fp32", a.points)
        with open(os.path.join(PROF, f"{a.tag}_{kind}_ncu.txt"), "w") as f:
            f.write("\n".join(lines) + "\n")
        if kind == "inplane" and "dram__bytes_read.sum" in d:
            def to_bytes(k):
                u, v = d[k]
                scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1)
                return float(v) * scale
            traffic.setdefault("per_config", {})[a.cfg] = {
                "dram_bytes_per_launch": to_bytes("dram__bytes_read.sum") + to_bytes("dram__bytes_write.sum"),
                "source": f"profiles/{a.tag}_inplane_ncu.txt (ncu --set full, cache flushed before the launch)",
            }
    # 3. DRAM without cache flush (cross-sweep L2 reuse)
    dc = os.path.join(OUT, f"dram_nocacheflush_{a.tag}.csv")
    if os.path.exists(dc):
        shutil.copy(dc, os.path.join(PROF, f"{a.tag}_dram_nocacheflush.csv"))
        rows = [r for r in csv.reader(open(dc)) if len(r) > 12 and r[0] != "ID"]
        byid = collections.defaultdict(dict)
        for r in rows:
            byid[r[0]][r[12]] = float(r[14])
        rd = [v.get("dram__bytes_read.sum", 0) + v.get("dram__bytes_write.sum", 0) for v in byid.values()]
        if rd and a.cfg in traffic.get("per_config", {}):
            traffic["per_config"][a.cfg]["dram_bytes_per_launch_no_flush"] = sum(rd) / len(rd)
    with open(tp, "w") as f:
        json.dump(traffic, f, indent=1)


if __name__ == "__main__":
    main()
