"""Render tools/configs_bench.py --c4-only JSON as the C4 table (profiles/<tag>_c4.md).

    python tools/c4_md.py profiles/r2e_c4.json > profiles/r2e_c4.md
"""
import json
import statistics
import sys

KN = {0: "inplane", 2: "inplane_ws"}


def main():
    d = json.load(open(sys.argv[1]))
    print("# BASELINE configs[3] (C4): exhaustive tuning vs beta = 5 % model-pruned picks\n")
    print("`tools/configs_bench.py --c4-only`.  f32, r = 1, 2, 4 on n^3 grids; each in-plane kernel tuned exhaustively "
          "over its own space under the same short-run conditions (`STENCIL_TUNE_SUSTAIN_MS=0`).  'beta 5 % pick' = the "
          "best measured rate among the top 5 % of the space as ranked by the model, as a fraction of the exhaustive "
          "best (P:L372-376).  Spearman = rank correlation of the model with measurement.\n")
    print("| n | r | kernel | M | exhaustive best Gpts/s | exhaustive s | model-P pick / best | model-P Spearman | "
          "model-B pick / best | model-B Spearman | best config |")
    print("|---|---|---|---|---|---|---|---|---|---|---|")
    for e in d["c4"]:
        c = e["best_cfg"]
        cfg = ",".join(str(c[k]) for k in ("tx", "ty", "rx", "ry", "stages", "zsegs", "zbox", "ytiles"))
        print(f"| {e['n']} | {e['r']} | {e['kernel']} | {e['M']} | {e['exhaustive_best_gpts']:.1f} | "
              f"{e['exhaustive_seconds']:.0f} | {e['model_paper_beta5_frac']:.3f} | {e['model_paper_spearman']:.2f} | "
              f"{e['model_b200_beta5_frac']:.3f} | {e['model_b200_spearman']:.2f} | `{cfg}` |")
    for key, name in (("model_b200_beta5_frac", "Model-B"), ("model_paper_beta5_frac", "model-P")):
        v = [e[key] for e in d["c4"]]
        print(f"\n{name}: mean {statistics.mean(v):.3f}, worst {min(v):.3f} of the exhaustive best.")


if __name__ == "__main__":
    main()
