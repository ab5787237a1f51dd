"""C-ABI library tests that need no GPU: the library loads, exports every symbol
include/stencil.h declares, and its host-only logic (layout, status codes,
slab partition, exchange plan, performance models) is right."""
import ctypes
import math
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def L():
    from conftest import build_library
    build_library()
    import paper_conf_ipps_tangtkwkgtw13_b200 as pkg
    return pkg


def header_functions():
    src = open(os.path.join(ROOT, "include", "stencil.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(stencil_[a-z0-9_]+)\s*\(", src)))


def test_exports_every_declared_symbol(L):
    names = header_functions()
    assert len(names) >= 20
    raw = ctypes.CDLL(L._lib.LIB_PATH)
    missing = [n for n in names if not hasattr(raw, n)]
    assert not missing, missing
    # and the Python binding declares a signature for each of them
    assert set(names) <= set(L._lib._SIGS), set(names) - set(L._lib._SIGS)


def test_abi_version_and_strings(L):
    lib = L.lib
    assert lib.stencil_abi_version() == 7
    for code, name in L._lib.STATUS.items():
        assert lib.stencil_status_string(code).decode() == name


@pytest.mark.parametrize("dtype,s,A", [("f32", 4, 32), ("f64", 8, 16)])
@pytest.mark.parametrize("n,r", [((512, 512, 512), 4), ((64, 64, 64), 1), ((37, 23, 19), 3), ((1, 1, 1), 2)])
def test_layout_arithmetic(L, dtype, s, A, n, r):
    nx, ny, nz = n
    lay = L.layout_compute(nx, ny, nz, r, dtype)
    assert lay.elem_size == s and lay.interior_x0 == A and lay.x_origin == A - r
    assert lay.pitch_x % A == 0 and lay.pitch_x >= A + nx + r and lay.pitch_x - (A + nx + r) < A
    assert lay.pitch_x * s % 128 == 0
    assert lay.rows_y == ny + 2 * r and lay.planes_z == nz + 2 * r
    assert lay.bytes == lay.planes_z * lay.rows_y * lay.pitch_x * s


@pytest.mark.parametrize("r,dtype,pitch", [(5, "f32", 576), (6, "f32", 576), (5, "f64", 544), (6, "f64", 544)])
def test_layout_orders_10_12(L, r, dtype, pitch):
    # Table IV orders 10 and 12: r = 5, 6 are supported
    lay = L.layout_compute(512, 512, 512, r, dtype)
    assert lay.radius == r and lay.pitch_x == pitch and lay.rows_y == 512 + 2 * r


def test_layout_c2_value(L):
    lay = L.layout_compute(512, 512, 512, 4, "f32")
    assert lay.pitch_x == 576 and lay.bytes == 520 * 520 * 576 * 4   # 623 MB


@pytest.mark.parametrize("args,code", [
    ((0, 5, 5, 1, "f32"), 1), ((5, 5, 5, 0, "f32"), 1), ((5, 5, 5, 7, "f64"), 1),
    ((5, 5, 5, 7, "f32"), 1)])
def test_layout_errors(L, args, code):
    with pytest.raises(L.StencilError) as e:
        L.layout_compute(*args)
    assert e.value.status == code
    assert L.lib.stencil_last_error_detail().decode() != ""


def test_null_safe_destroy(L):
    L.lib.stencil_destroy(None)


@pytest.mark.parametrize("nz,P", [(1024, 8), (512, 2), (100, 3), (17, 4), (8, 1)])
def test_slab_partition_covers_grid(L, nz, P):
    z = 0
    sizes = []
    for rank in range(P):
        z0, n = L.slab_partition(nz, P, rank, 1)
        assert z0 == z
        z += n
        sizes.append(n)
    assert z == nz and max(sizes) - min(sizes) <= 1


def test_slab_partition_rejects_thin_slabs(L):
    with pytest.raises(L.StencilError):
        L.slab_partition(12, 4, 0, 4)   # 3 planes per rank < r


def test_exchange_plan_offsets(L):
    r = 4
    lay = L.layout_compute(64, 48, 32, r, "f32")
    plane = lay.rows_y * lay.pitch_x * 4
    x = L.exchange_plan(lay, 4, 1)
    assert (x["peer_lo"], x["peer_hi"]) == (0, 2)
    assert x["msg_bytes"] == r * plane
    assert x["recv_lo_off"] == 0 and x["send_lo_off"] == r * plane
    assert x["send_hi_off"] == 32 * plane and x["recv_hi_off"] == (32 + r) * plane
    assert x["recv_hi_off"] + x["msg_bytes"] == lay.bytes
    e0, e3 = L.exchange_plan(lay, 4, 0), L.exchange_plan(lay, 4, 3)
    assert e0["peer_lo"] == -1 and e3["peer_hi"] == -1


# ---- models: C++ model-P must equal oracle/model_p.py (Eqs. 6-14) ----------------
def _gpu(L, **kw):
    from oracle import model_p as mp
    g = dict(SM=148, BW=6.5e12, Smem=228 * 1024, Reg=65536, Blk_SM=32, Warp_SM=64, Lat=600.0, Clock=1.965e9)
    g.update(kw)
    G = L._lib.GpuParams(g["SM"], g["BW"], g["Smem"], g["Reg"], g["Blk_SM"], g["Warp_SM"], g["Lat"], g["Clock"])
    return G, mp.GPU(**g)


@pytest.mark.parametrize("tx,ty,rx,ry,r,regs", [(32, 4, 4, 4, 4, 237), (256, 1, 1, 8, 1, 20), (64, 2, 8, 2, 2, 143),
                                                (16, 8, 2, 1, 3, 60), (32, 16, 4, 1, 1, 45)])
@pytest.mark.parametrize("literal", [0, 1])
def test_model_paper_matches_oracle(L, tx, ty, rx, ry, r, regs, literal):
    from oracle import model_p as mp
    G, g = _gpu(L)
    s = 4
    W, H = tx * rx, ty * ry
    smem = (W + 2 * r) * (H + 2 * r) * s * 3
    K = L._lib.ModelKernel(512, 512, 512, tx, ty, rx, ry, r, s, regs, smem, 8 * r + 1, 3, 1, 4, 0, 0)
    k = mp.Kernel(LX=512, LY=512, TX=tx, TY=ty, RX=rx, RY=ry, r=r, s=s, K_R=regs * tx * ty, K_S=smem, Ops=8 * r + 1)
    blks, act, st, rem = ctypes.c_double(), ctypes.c_int(), ctypes.c_int(), ctypes.c_int()
    v = L.lib.stencil_model_paper(ctypes.byref(G), ctypes.byref(K), literal, ctypes.byref(blks), ctypes.byref(act),
                                  ctypes.byref(st), ctypes.byref(rem))
    assert blks.value == mp.blks(k)
    assert act.value == mp.act_blks(g, k)
    assert st.value == mp.stages(g, k)
    assert rem.value == mp.rem_blks(g, k)
    assert math.isclose(v, mp.perf(g, k, literal_tc=bool(literal)), rel_tol=1e-12)


def test_model_b200_properties(L):
    G, _ = _gpu(L)
    def pred(**kw):
        d = dict(lx=512, ly=512, lz=512, tx=32, ty=4, rx=4, ry=4, radius=4, elem_size=4, regs_per_thread=237,
                 smem_per_block=53000, ops_per_point=33, stages=4, zbox=1, zsegs=4, ytiles=0, active_blocks=2,
                 inputs=1)
        d.update(kw)
        K = L._lib.ModelKernel(*[d[f] for f, _ in L._lib.ModelKernel._fields_])
        return L.lib.stencil_model_b200(ctypes.byref(G), ctypes.byref(K))
    base = pred()
    assert 0 < base <= 6.5e12 / 8 * 1.0001        # never above the DRAM roofline (8 B/pt)
    G2, _ = _gpu(L, BW=13e12)
    K = L._lib.ModelKernel(512, 512, 512, 32, 4, 4, 4, 4, 4, 237, 53000, 33, 4, 1, 4, 0, 2, 1)
    assert L.lib.stencil_model_b200(ctypes.byref(G2), ctypes.byref(K)) >= base
    assert pred(stages=2, active_blocks=1) <= base   # less in flight never helps
    assert pred(zsegs=32) < pred(zsegs=4)            # more segments -> more re-reads
    assert pred(zbox=2) >= pred(zbox=1)              # deeper boxes -> more bytes in flight
    assert pred(inputs=2) < base                     # a second input grid adds traffic
    assert pred(ry=1) < pred(ry=4)                   # column-block reuse: fewer LDS per point
    assert pred(ty=1, active_blocks=1) < base        # 1 warp per SM cannot hide latency


def test_forward_kernels_do_not_spill(L):
    """Every forward-plane instantiation must be spill-free: the tuner drops
    kernels with local memory (P:L254 register constraint), so one spilling
    instantiation empties that (dtype, r) search space.  (ptxas once chose 32
    registers + a stack frame for float r = 4 under __launch_bounds__(512).)"""
    import shutil
    import subprocess
    tool = shutil.which("cuobjdump") or "/usr/local/cuda/bin/cuobjdump"
    if not os.path.exists(tool):
        pytest.skip("cuobjdump not available")
    out = subprocess.run([tool, "-res-usage", L._lib.LIB_PATH], capture_output=True, text=True).stdout
    lines = out.splitlines()
    seen = 0
    for i, ln in enumerate(lines):
        # the SDK shape (one register row, template argument RY = 1): register-row variants that spill
        # are excluded by the tuner and do not empty the space
        if "Function" in ln and "forward_sweep_kernel" in ln and "Li1EEEv" in ln:
            seen += 1
            usage = lines[i + 1]
            assert "STACK:0" in usage and "LOCAL:0" in usage, (ln, usage)
    assert seen == 2 * 6 * 3   # dtype x r = 1..6 x (plain, second grid, per-axis)


@pytest.mark.parametrize("idx", [0, 1])
@pytest.mark.parametrize("literal", [0, 1])
def test_model_paper_hand_values(L, idx, literal):
    """The library's model-P (stencil_model_paper) against the hand-derived Eqs. (6)-(14) values of
    tests/golden/model_p_hand.json (readings R12-R14)."""
    import json
    import os
    with open(os.path.join(os.path.dirname(__file__), "golden", "model_p_hand.json")) as f:
        d = json.load(f)
    g, c = d["gpu"], d["cases"][idx]
    k = c["kernel"]
    G = L._lib.GpuParams(g["SM"], g["BW"], g["Smem"], g["Reg"], g["Blk_SM"], g["Warp_SM"], float(g["Lat"]), g["Clock"])
    W, H = k["TX"] * k["RX"], k["TY"] * k["RY"]
    K = L._lib.ModelKernel(k["LX"], k["LY"], 512, k["TX"], k["TY"], k["RX"], k["RY"], k["r"], k["s"],
                           k["regs_per_thread"], (W + 2 * k["r"]) * (H + 2 * k["r"]) * k["s"], k["Ops"], 3, 1, 1, 0, 0, 0)
    blks, act, st, rem = ctypes.c_double(), ctypes.c_int(), ctypes.c_int(), ctypes.c_int()
    v = L.lib.stencil_model_paper(ctypes.byref(G), ctypes.byref(K), literal, ctypes.byref(blks), ctypes.byref(act),
                                  ctypes.byref(st), ctypes.byref(rem))
    it = c["integer"]
    assert (blks.value, act.value, st.value, rem.value) == (it["Blks"], it["ActBlks"], it["Stages"], it["RemBlks"])
    expect = c["literal"]["Perf"] if literal else c["Perf"]
    assert math.isclose(v, expect, rel_tol=2e-9)


def test_bench_has_a_pinned_c2_configuration():
    """bench.py times the configuration tune_cache.txt holds for BASELINE configs[1] (the full-grid
    parity test runs exactly that one)."""
    import bench
    cfg = bench.pinned_config("c2")
    assert cfg is not None and cfg["kernel"] in ("inplane", "inplane_ws")
    e = bench.cache_entry(512, 512, 512, 4, "f32", kernel="forward")
    assert e is not None and e[0] == "forward"
