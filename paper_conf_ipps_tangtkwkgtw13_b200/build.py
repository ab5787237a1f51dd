"""Build libstencil.so in-tree with nvcc for sm_100a.

    python paper_conf_ipps_tangtkwkgtw13_b200/build.py [--force] [--ptxas-v]

Each .cu under csrc/ is compiled in parallel to an object file, then linked
into ``paper_conf_ipps_tangtkwkgtw13_b200/libstencil.so`` (static cudart, no
link-time dependency on libcuda or NCCL).
"""
from __future__ import annotations

import argparse
import concurrent.futures as cf
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
ROOT = os.path.dirname(HERE)
BUILD = os.path.join(HERE, "_build")
LIB = os.path.join(HERE, "libstencil.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")

ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-Xcompiler", "-Wall",
         "-I", os.path.join(ROOT, "include")]


def _sources():
    return sorted(f for f in os.listdir(CSRC) if f.endswith(".cu"))


def _deps():
    return [os.path.join(CSRC, f) for f in os.listdir(CSRC)] + [os.path.join(ROOT, "include", "stencil.h")]


def _stale(target: str, deps) -> bool:
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, ptxas_v: bool = False, verbose: bool = False, defines=(), out: str | None = None) -> str:
    """Build libstencil.so (or, with ``out``/``defines``, an experiment variant of it)."""
    lib = out or LIB
    bdir = BUILD if not out else BUILD + "_" + os.path.basename(out).replace(".so", "")
    os.makedirs(bdir, exist_ok=True)
    deps = _deps()
    if not force and not _stale(lib, deps):
        return lib
    extra = (["-Xptxas", "-v"] if ptxas_v else []) + [f"-D{d}" for d in defines]

    def compile_one(src):
        obj = os.path.join(bdir, src.replace(".cu", ".o"))
        cmd = [NVCC, *ARCH, *FLAGS, *extra, "-c", os.path.join(CSRC, src), "-o", obj]
        p = subprocess.run(cmd, capture_output=True, text=True)
        if p.returncode != 0:
            raise RuntimeError(f"nvcc failed for {src}:\n{p.stderr}")
        return obj, p.stderr

    with cf.ThreadPoolExecutor(max_workers=os.cpu_count() or 4) as ex:
        results = list(ex.map(compile_one, _sources()))
    if verbose or ptxas_v:
        for _, err in results:
            sys.stderr.write(err)
    objs = [o for o, _ in results]
    cmd = [NVCC, *ARCH, "-shared", "-o", lib + ".tmp", *objs, "-ldl", "-lpthread"]
    p = subprocess.run(cmd, capture_output=True, text=True)
    if p.returncode != 0:
        raise RuntimeError(f"link failed:\n{p.stderr}")
    os.replace(lib + ".tmp", lib)
    return lib


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--force", action="store_true")
    ap.add_argument("--ptxas-v", action="store_true")
    ap.add_argument("-D", dest="defines", action="append", default=[], help="extra -D for an experiment variant")
    ap.add_argument("--out", default=None, help="output .so path for an experiment variant")
    a = ap.parse_args()
    print(build(force=a.force, ptxas_v=a.ptxas_v, verbose=True, defines=a.defines, out=a.out))
