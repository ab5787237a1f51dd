"""Per-configuration ceilings of the C3 sweeps (profiles/<tag>_configs.json): HBM (measured copy bandwidth),
shared-memory crossbar, FMA / FP64 pipe and issue, each as Gpts/s at the maximum SM clock on the SMs the
grid occupies (one CTA per SM), and the measured rate as a fraction of the lowest.

    python tools/rooflines.py profiles/r2c_configs.json [--peak 6458.7] > profiles/r2c_rooflines.md

Counts per interior point, from the kernel structure (inplane_ws.cuh / inplane.cuh):
  shared loads  ((RY + 2r) * RXV + RY * 2 * NVH) 16-byte LDS per step per thread, RX * RY points per step
  TMA writes    (W + 2 HX)(H + 2r) s bytes per plane-tile, W * H points
  FP slots      f32: (6r + 1 + n_odd) / 2 (packed FFMA2/FADD2/FMUL2, the n_odd odd-m x pairs as scalar FADD);
                f64: 6r + 1 (DFMA / DADD)
  issue         ncu instructions per point where captured (profiles/r2_high_order_ncu.md, r2c_inplane_ncu.txt)
Machine: 128 B/clk/SM shared-memory crossbar (B300_MICROARCH.md), 64 FMA-pipe thread-instructions per clk per
SM (FFMA2 and DFMA: one warp instruction per 2 cycles per sub-partition), 128 issue slots per clk per SM.
"""
import argparse
import json
import math

CLK = 1.965e9
ISSUE = {("f32", 4): 18.0, ("f32", 5): 24.6, ("f32", 6): 29.4, ("f64", 4): 34.9, ("f64", 6): 54.9}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("configs")
    ap.add_argument("--peak", type=float, default=6458.7)
    ap.add_argument("--sms", type=int, default=148)
    a = ap.parse_args()
    d = json.load(open(a.configs))
    print("# Ceilings of the C3 heat sweeps (512^3) per tuned configuration\n")
    print(__doc__.split("\n\n", 1)[1].replace("    python", "    python"))
    print("| dtype | r | config | CTAs | measured Gpts/s | HBM | smem | FP pipe | issue | lowest | measured / lowest |")
    print("|---|---|---|---|---|---|---|---|---|---|---|")
    for e in d["c3"]:
        if e["app"] != "jacobi":
            continue
        dt, r, c = e["dtype"], e["r"], e["inplane_cfg"]
        s = 4 if dt == "f32" else 8
        vec = 16 // s
        hx = math.ceil(r / vec) * vec
        nvh = hx // vec
        rxv = c["rx"] // vec
        W, H = c["tx"] * c["rx"], c["ty"] * c["ry"]
        n = 512
        ytiles = c.get("ytiles") or math.ceil(n / H)
        ctas = math.ceil(n / W) * ytiles * c["zsegs"]
        sms = min(ctas, a.sms)
        lds = ((c["ry"] + 2 * r) * rxv + c["ry"] * 2 * nvh) * 16 / (c["rx"] * c["ry"])
        tma = (W + 2 * hx) * (H + 2 * r) * s / (W * H)
        smem = 128 * CLK * sms / (lds + tma) / 1e9
        hbm = a.peak * 1e9 / (2 * s) / 1e9
        n_odd = (r + 1) // 2
        fp = (6 * r + 1 + n_odd) / 2 if dt == "f32" else 6 * r + 1
        fpc = 64 * CLK * sms / fp / 1e9
        ins = ISSUE.get((dt, r))
        iss = 128 * CLK * sms / ins / 1e9 if ins else None
        cands = {"HBM": hbm, "smem": smem, "FP pipe": fpc}
        if iss:
            cands["issue"] = iss
        low = min(cands, key=cands.get)
        m = e["inplane_gpts"]
        cfg = f"{c['kernel']}:{c['tx']},{c['ty']},{c['rx']},{c['ry']},{c['stages']},{c['zsegs']},{c['zbox']}"
        print(f"| {dt} | {r} | `{cfg}` | {ctas} | {m:.0f} | {hbm:.0f} | {smem:.0f} ({lds + tma:.0f} B/pt) | "
              f"{fpc:.0f} ({fp:g}/pt) | {'%.0f' % iss if iss else '-'} | {low} | {m / cands[low]:.2f} |")


if __name__ == "__main__":
    main()
