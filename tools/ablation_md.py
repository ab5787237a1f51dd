#!/usr/bin/env python3
"""Markdown tables of the loading ablation from tools/ablation.py and tools/ablation_ncu.py output.

    python tools/ablation_md.py profiles/r2_ablation.json profiles/r2_ablation_ncu_r4.json \
        profiles/r2_ablation_ncu_r1.json > tables.md
"""
import json
import sys

LABEL = {
    "forward": "forward-plane (SDK FDTD3d shape; RB = register rows, Fig. 10 (i))",
    "ip_classic": "in-plane, classic loads (Fig. 6a)",
    "ip_vertical": "in-plane, vertical (Fig. 6b)",
    "ip_horizontal": "in-plane, horizontal (Fig. 6c)",
    "ip_fullslice": "in-plane, full slice, scalar (Fig. 6d)",
    "ip_fullslice_v": "in-plane, full slice, 16-B vectors (P:L189-191)",
    "fp_tma": "forward-plane with K-IP's loads (TMA box, 16-B columns, register rows)",
    "inplane": "K-IP: full slice as one TMA box",
    "inplane_ws": "K-IP warp-specialized",
}


def main():
    d = json.load(open(sys.argv[1]))
    rows = d["rows"]
    kernels = list(rows[0]["kernels"].keys())
    print("| kernel | " + " | ".join(f"r={x['r']} TB / RB Gpts/s (x FP)" for x in rows) + " |")
    print("|---" * (len(rows) + 1) + "|")
    for k in kernels:
        cells = []
        for x in rows:
            v = x["kernels"].get(k, {})
            tb = v.get("tb_gpts")
            rb = v.get("rb_gpts")
            tbs = v.get("tb_speedup_vs_fp_tb")
            rbs = v.get("rb_speedup_vs_fp_tb")
            cells.append(f"{tb if tb is not None else '-'} / {rb if rb is not None else '-'} "
                         f"({tbs if tbs is not None else '-'} / {rbs if rbs is not None else '-'})")
        print(f"| {LABEL.get(k, k)} | " + " | ".join(cells) + " |")
    for path in sys.argv[2:]:
        n = json.load(open(path))
        print()
        print(f"## ncu, r = {n['r']}, each kernel at its TB / RB configuration (one sweep, cache flushed; "
              "`--clock-control none`)")
        print()
        print("| kernel:config | duration us | instr / point | DRAM MB / launch | global-load sectors / request | "
              "L2 read sectors / point | FMA pipe % |")
        print("|---|---|---|---|---|---|---|")
        for k, v in n["kernels"].items():
            cfg = v["cfg"].split(":", 1)[1]
            dur = v["duration_ms"]
            dur_us = dur / 1000.0 if dur and dur > 1000 else (dur or 0) * 1000.0   # ncu reported ns
            print(f"| {k} `{cfg}` | {dur_us:.1f} | {v['instr_per_point']:.1f} | {v['dram_bytes_per_launch'] / 1e6:.0f} | "
                  f"{v['global_ld_sectors_per_request']:.2f} | {v['l2_read_sectors_per_point']:.2f} | "
                  f"{v['fma_pipe_pct']:.1f} |")


if __name__ == "__main__":
    main()
