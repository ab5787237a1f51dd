"""Build a slim A/B variant of libstencil.so: the non-kernel sources plus only the named kernel
translation units (the other kern_*.cu registrations become empty stubs), compiled with extra defines.

    python tools/variant_lib.py OUT.so -D STENCIL_STG_U64 kern_f32_r4_ws.cu kern_f32_r4.cu

The full library is ~330 MB; a variant with two kernel units is a few MB, so several ship to the GPU
box in one snapshot (load one with STENCIL_LIB=OUT.so).  Non-kernel objects are reused from the main
build (paper_conf_ipps_tangtkwkgtw13_b200/_build).
"""
import argparse
import os
import re
import shutil
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "paper_conf_ipps_tangtkwkgtw13_b200"))
import build as B  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("out")
    ap.add_argument("-D", dest="defines", action="append", default=[])
    ap.add_argument("sources", nargs="+")
    a = ap.parse_args()
    bdir = B.BUILD + "_variant_" + os.path.basename(a.out).replace(".so", "")
    os.makedirs(bdir, exist_ok=True)
    objs, stubs = [], []
    for src in B._sources():
        obj = os.path.join(bdir, src.replace(".cu", ".o"))
        if src in a.sources:
            cmd = [B.NVCC, *B.ARCH, *B.FLAGS, *[f"-D{d}" for d in a.defines], "-c", os.path.join(B.CSRC, src),
                   "-o", obj]
            subprocess.run(cmd, check=True)
        elif src.startswith("kern_"):
            name = re.search(r"STENCIL_REGISTER\w*\((\w+)", open(os.path.join(B.CSRC, src)).read()).group(1)
            stubs.append(name)
            continue
        else:
            shutil.copy2(os.path.join(B.BUILD, src.replace(".cu", ".o")), obj)
        objs.append(obj)
    stub = os.path.join(bdir, "stubs.cu")
    with open(stub, "w") as f:
        f.write("#include <vector>\nnamespace stencil { struct KernelEntry;\n")
        for n in stubs:
            f.write(f"void {n}(std::vector<KernelEntry>&) {{}}\n")
        f.write("}\n")
    subprocess.run([B.NVCC, *B.ARCH, *B.FLAGS, "-c", stub, "-o", stub + ".o"], check=True)
    objs.append(stub + ".o")
    subprocess.run([B.NVCC, *B.ARCH, "-shared", "-o", a.out, *objs, "-ldl", "-lpthread"], check=True)
    print(a.out, os.path.getsize(a.out))


if __name__ == "__main__":
    main()
