"""SASS census of the instantiation bench.py times (and of its classic / forward-plane peers):
opcode counts that prove the Blackwell path (UTMALDG = TMA tensor loads, SYNCS = mbarrier operations,
FFMA2 / FADD2 / FMUL2 = packed FP32x2, USETMAXREG = register hand-off) and the per-step mix.

    python tools/sass_census.py > profiles/r2_sass_census.md
"""
import collections
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402

LIB = os.path.join(ROOT, "paper_conf_ipps_tangtkwkgtw13_b200", "libstencil.so")
BUILD = os.path.join(ROOT, "paper_conf_ipps_tangtkwkgtw13_b200", "_build")


def mangled(kind, dtype, r, bx, rxv, ry, zb):
    T = "f" if dtype == "f32" else "d"
    if kind == "inplane_ws":
        return f"_ZN7stencil17inplane_ws_kernelI{T}Li{r}ELi{bx}ELi{rxv}ELi{ry}ELi{zb}ELb0ELb0ELb0EE"
    if kind == "inplane":
        return f"_ZN7stencil20inplane_sweep_kernelI{T}Li{r}ELi{bx}ELi{rxv}ELi{ry}ELb0ELb0ELb0EE"
    return f"_ZN7stencil20forward_sweep_kernelI{T}Li{r}ELb0ELb0ELi1EE"


def census(obj, prefix):
    names = [l.split("Function : ")[1].strip() for l in
             subprocess.run(["cuobjdump", "-sass", obj], capture_output=True, text=True).stdout.splitlines()
             if "Function : " in l]
    fn = next((n for n in names if n.startswith(prefix)), None)
    if fn is None:
        return None, None
    sass = subprocess.run(["cuobjdump", "-sass", "-fun", fn, obj], capture_output=True, text=True).stdout
    ops = collections.Counter()
    for l in sass.splitlines():
        m = re.match(r"\s+/\*[0-9a-f]+\*/\s+(@!?U?P\w+\s+)?([A-Z0-9_]+)", l)
        if m:
            ops[m.group(2)] += 1
    return fn, ops


cfg = bench.pinned_config("c2")
vec = 4
rows = [("timed by bench.py (tune_cache.txt)", cfg["kernel"], "kern_f32_r4_ws.o" if cfg["kernel"] == "inplane_ws" else "kern_f32_r4.o",
         mangled(cfg["kernel"], "f32", 4, cfg["tx"], cfg["rx"] // vec, cfg["ry"], cfg["zbox"]))]
rows.append(("classic in-plane, same tile", "inplane", "kern_f32_r4.o", mangled("inplane", "f32", 4, cfg["tx"], cfg["rx"] // vec, cfg["ry"], 0)))
rows.append(("forward-plane baseline", "forward", "kern_f32_r4.o", mangled("forward", "f32", 4, 0, 0, 1, 0)))
print("# SASS census, 512^3 r=4 f32 (cuobjdump -sass of the in-tree build objects)\n")
print(f"bench.py configuration: `{cfg}`\n")
keys = ["UTMALDG", "UTMASTG", "SYNCS", "USETMAXREG", "FFMA2", "FADD2", "FMUL2", "FFMA", "FADD", "LDS", "STS",
        "LDG", "STG", "MOV", "IADD3", "IMAD", "BRA", "BAR"]
print("| kernel | function | total | " + " | ".join(keys) + " |")
print("|---|---|---|" + "---|" * len(keys))
for title, kind, obj, pre in rows:
    fn, ops = census(os.path.join(BUILD, obj), pre)
    if fn is None:
        print(f"| {title} | (not found: {pre}) |")
        continue
    print(f"| {title} | `{fn[:60]}...` | {sum(ops.values())} | " + " | ".join(str(ops.get(k, 0)) for k in keys) + " |")
print("\nThe unrolled sweep body is 2r (or lcm(2r, zbox)) plane steps; per step and thread (RX x RY points) the"
      " FFMA2/FADD2/FMUL2 count is the 6r+1 lane operations per point of the fixed order halved, plus the odd-m"
      " x pairs as scalar FADD (the x-neighbour pairs at odd offsets straddle the packed lanes).")
