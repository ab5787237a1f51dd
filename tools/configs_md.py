"""Render tools/configs_bench.py + tools/divgrad_bench.py JSON as the markdown tables of profiles/<tag>_configs.md.

    python tools/configs_md.py profiles/r2c_configs.json profiles/r2c_divgrad.json [--peak 6458.7] > profiles/r2c_configs.md
"""
import argparse
import json


def cfg_str(c):
    return f"{c['kernel']}:" + ",".join(str(c[k]) for k in ("tx", "ty", "rx", "ry", "stages", "zsegs", "zbox"))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("configs")
    ap.add_argument("divgrad")
    ap.add_argument("--peak", type=float, default=None, help="copy GB/s for the fractions (default: the JSON's)")
    a = ap.parse_args()
    d = json.load(open(a.configs))
    g = json.load(open(a.divgrad))
    peak = a.peak or g.get("peak_GBs")
    print(f"# BASELINE configs[0] and [2] on {d.get('device', 'B200')} (tools/configs_bench.py, tools/divgrad_bench.py)\n")
    print(f"Fractions are of the measured copy bandwidth ({peak} GB/s, MEASURED_PEAKS.json). In-plane = the faster of "
          "the classic and the warp-specialized kernel after `stencil_tune` (beta = 5 %, model-B, sustained "
          "refinement 150 ms); forward-plane = the SDK-shape baseline tuned over its space; 20 (wave: 21) sweeps "
          "per timed run, median of 3; grids 512^3.\n")
    c1 = d.get("c1")
    if c1:
        print(f"C1 (64^3 r=1 f32, 10 sweeps, launch-bound, CUDA-graph replay): {c1['gpts']:.1f} Gpts/s, "
              f"{c1['ms_per_run_10_iters'] * 1e3:.0f} us per 10-sweep run, max rel err vs oracle {c1['max_rel_err']:.1e}.\n")
    print("## C3: heat stencils (Table IV orders 2..12) and the leapfrog wave\n")
    print("| stencil | dtype | r | in-plane Gpts/s | alg. GB/s | frac of copy | config | forward-plane Gpts/s | speedup |")
    print("|---|---|---|---|---|---|---|---|---|")
    for e in d["c3"]:
        gbs = e["inplane_GBs"]
        print(f"| {e['app']} | {e['dtype']} | {e['r']} | {e['inplane_gpts']:.1f} | {gbs:.0f} | {gbs / peak:.2f} | "
              f"`{cfg_str(e['inplane_cfg'])}` | {e['forward_gpts']:.1f} | {e['speedup']:.2f} |")
    print("\n## Div (3 -> 1) and Grad (1 -> 3), Table V (4 s algorithmic bytes per point)\n")
    print("| stencil | dtype | r | Gpts/s | frac of copy | config |")
    print("|---|---|---|---|---|---|")
    for e in g["rows"]:
        print(f"| {e['app']} | {e['dtype']} | {e['r']} | {e['gpts']:.1f} | {e['alg_GBs'] / peak:.3f} | `{cfg_str(e['cfg'])}` |")


if __name__ == "__main__":
    main()
