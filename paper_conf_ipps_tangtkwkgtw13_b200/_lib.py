"""ctypes binding of libstencil.so (include/stencil.h).  Argument marshalling only.

The library is built in-tree by ``paper_conf_ipps_tangtkwkgtw13_b200.build``;
there is NO fallback: if ``libstencil.so`` is missing, importing the package
raises.
"""
from __future__ import annotations

import ctypes
import os

HERE = os.path.dirname(os.path.abspath(__file__))
# STENCIL_LIB selects another build of the same library (A/B experiments, tools/ab.sh)
LIB_PATH = os.environ.get("STENCIL_LIB") or os.path.join(HERE, "libstencil.so")

F32, F64 = 0, 1
DTYPE_CODES = {"f32": F32, "f64": F64}
KERNEL_INPLANE, KERNEL_FORWARD, KERNEL_INPLANE_WS = 0, 1, 2
KERNEL_CODES = {"inplane": KERNEL_INPLANE, "forward": KERNEL_FORWARD, "inplane_ws": KERNEL_INPLANE_WS,
                # the paper's in-plane loading variants with per-thread loads (Fig. 6; ablation)
                "ip_classic": 3, "ip_vertical": 4, "ip_horizontal": 5, "ip_fullslice": 6, "ip_fullslice_v": 7,
                # forward-plane with the in-plane kernel's TMA loads (ablation)
                "fp_tma": 8}
TMA_KERNELS = ("inplane", "inplane_ws", "fp_tma")
MODEL_PAPER, MODEL_B200 = 0, 1

STATUS = {
    0: "STENCIL_SUCCESS",
    1: "STENCIL_ERROR_INVALID_VALUE",
    2: "STENCIL_ERROR_NOT_SUPPORTED",
    3: "STENCIL_ERROR_MISALIGNED",
    4: "STENCIL_ERROR_OUT_OF_MEMORY",
    5: "STENCIL_ERROR_CUDA",
    6: "STENCIL_ERROR_NCCL",
}

i32, i64, dbl, vp = ctypes.c_int32, ctypes.c_int64, ctypes.c_double, ctypes.c_void_p


class Layout(ctypes.Structure):
    _fields_ = [("nx", i64), ("ny", i64), ("nz", i64), ("radius", i32), ("dtype", i32),
                ("elem_size", i64), ("pitch_x", i64), ("rows_y", i64), ("planes_z", i64),
                ("interior_x0", i64), ("x_origin", i64), ("bytes", i64)]


class Config(ctypes.Structure):
    _fields_ = [("kernel", i32), ("tx", i32), ("ty", i32), ("rx", i32), ("ry", i32),
                ("stages", i32), ("zsegs", i32), ("zbox", i32), ("ytiles", i32)]

    def as_dict(self):
        return {f: getattr(self, f) for f, _ in self._fields_}


class Stats(ctypes.Structure):
    _fields_ = [("launches", i64), ("aux_launches", i64), ("timing_enabled", i32),
                ("last_run_sweeps", i32), ("last_run_sweep_ms", dbl), ("timed_sweeps", i64),
                ("timed_sweep_ms", dbl), ("sweep_ms_min", dbl), ("sweep_ms_max", dbl)]


class TuneReport(ctypes.Structure):
    _fields_ = [("model", i32), ("beta_percent", dbl), ("space_size", i32), ("timed", i32),
                ("best", Config), ("best_ms_per_iter", dbl), ("best_predicted_gpts", dbl),
                ("best_measured_gpts", dbl), ("best_rank_by_model", i32), ("best_burst_gpts", dbl)]


class TuneEntry(ctypes.Structure):
    _fields_ = [("cfg", Config), ("pred_paper_gpts", dbl), ("pred_b200_gpts", dbl),
                ("measured_gpts", dbl), ("regs_per_thread", i32), ("smem_bytes", i32),
                ("active_blocks", i32)]


class GpuParams(ctypes.Structure):
    _fields_ = [("sm", i32), ("bw", dbl), ("smem", i32), ("reg", i32), ("blk_sm", i32),
                ("warp_sm", i32), ("lat_cycles", dbl), ("clock_hz", dbl)]


class ModelKernel(ctypes.Structure):
    _fields_ = [("lx", i64), ("ly", i64), ("lz", i64), ("tx", i32), ("ty", i32), ("rx", i32),
                ("ry", i32), ("radius", i32), ("elem_size", i32), ("regs_per_thread", i32),
                ("smem_per_block", i32), ("ops_per_point", i32), ("stages", i32), ("zbox", i32), ("zsegs", i32),
                ("ytiles", i32), ("active_blocks", i32), ("inputs", i32)]


class ExchangePlan(ctypes.Structure):
    _fields_ = [("peer_lo", i32), ("peer_hi", i32), ("send_lo_off", i64), ("recv_lo_off", i64),
                ("send_hi_off", i64), ("recv_hi_off", i64), ("msg_bytes", i64)]


P = ctypes.POINTER
class P2PEndpoint(ctypes.Structure):
    _fields_ = [("grid", ctypes.c_void_p * 2), ("flags", ctypes.c_void_p), ("rank", i32), ("nz_local", i64)]


class P2PTargets(ctypes.Structure):
    _fields_ = [("lo_rank", i32), ("hi_rank", i32), ("planes", i32), ("lo_delta", i64), ("hi_delta", i64)]


_SIGS = {
    "stencil_status_string": (ctypes.c_char_p, [i32]),
    "stencil_last_error_detail": (ctypes.c_char_p, []),
    "stencil_abi_version": (ctypes.c_int, []),
    "stencil_layout_compute": (i32, [i64, i64, i64, ctypes.c_int, i32, P(Layout)]),
    "stencil_plan_create": (i32, [P(vp), i64, i64, i64, ctypes.c_int, P(dbl), i32]),
    "stencil_destroy": (None, [vp]),
    "stencil_plan_layout": (i32, [vp, P(Layout)]),
    "stencil_plan_set_config": (i32, [vp, P(Config)]),
    "stencil_plan_get_config": (i32, [vp, P(Config)]),
    "stencil_run": (i32, [vp, vp, vp, ctypes.c_int, vp]),
    "stencil_plan_create_app": (i32, [P(vp), i64, i64, i64, ctypes.c_int, P(dbl), i32, i32, dbl]),
    "stencil_plan_create_axes": (i32, [P(vp), i64, i64, i64, ctypes.c_int, P(dbl), i32]),
    "stencil_run_host": (i32, [vp, vp, vp, ctypes.c_int, vp]),
    "stencil_residual": (i32, [vp, vp, vp, vp, P(dbl)]),
    "stencil_run_host_wait": (i32, [vp, vp]),
    "stencil_run_until": (i32, [vp, vp, vp, ctypes.c_int, dbl, ctypes.c_int, vp, P(ctypes.c_int), P(dbl)]),
    "stencil_plan_create_p2p": (i32, [P(vp), i64, i64, i64, ctypes.c_int, P(dbl), i32, ctypes.c_int, ctypes.c_int]),
    "stencil_p2p_endpoint": (i32, [vp, P(P2PEndpoint)]),
    "stencil_p2p_connect": (i32, [vp, P(P2PEndpoint), P(P2PEndpoint)]),
    "stencil_p2p_export": (i32, [vp, vp]),
    "stencil_p2p_import": (i32, [vp, vp, vp]),
    "stencil_p2p_run": (i32, [vp, ctypes.c_int, vp, P(ctypes.c_int)]),
    "stencil_p2p_quiesce": (i32, [vp, vp]),
    "stencil_p2p_targets": (i32, [P(Layout), i64, ctypes.c_int, ctypes.c_int, P(P2PTargets)]),
    "stencil_p2p_residual": (i32, [vp, vp, P(dbl)]),
    "stencil_run_source": (i32, [vp, vp, vp, vp, ctypes.c_int, vp]),
    "stencil_run_wave": (i32, [vp, vp, vp, ctypes.c_int, vp]),
    "stencil_plan_create_divgrad": (i32, [P(vp), i64, i64, i64, ctypes.c_int, P(dbl), i32, i32]),
    "stencil_run_div": (i32, [vp, vp, vp, vp, vp, vp]),
    "stencil_run_grad": (i32, [vp, vp, vp, vp, vp, vp]),
    "stencil_plan_reserve": (i32, [vp]),
    "stencil_plan_set_timing": (i32, [vp, ctypes.c_int]),
    "stencil_plan_stats": (i32, [vp, P(Stats)]),
    "stencil_tune": (i32, [vp, i32, i32, dbl, ctypes.c_int, ctypes.c_int, vp, vp, vp, P(TuneReport)]),
    "stencil_tune_results": (i32, [vp, P(TuneEntry), ctypes.c_int, P(ctypes.c_int)]),
    "stencil_model_paper": (dbl, [P(GpuParams), P(ModelKernel), ctypes.c_int, P(dbl), P(ctypes.c_int),
                                  P(ctypes.c_int), P(ctypes.c_int)]),
    "stencil_model_b200": (dbl, [P(GpuParams), P(ModelKernel)]),
    "stencil_slab_partition": (i32, [i64, ctypes.c_int, ctypes.c_int, ctypes.c_int, P(i64), P(i64)]),
    "stencil_exchange_plan": (i32, [P(Layout), ctypes.c_int, ctypes.c_int, P(ExchangePlan)]),
    "stencil_nccl_unique_id": (i32, [vp]),
    "stencil_plan_create_dist_local": (i32, [P(vp), i64, i64, i64, ctypes.c_int, P(dbl), i32, ctypes.c_int]),
    "stencil_run_dist_local": (i32, [P(vp), ctypes.c_int, P(vp), P(vp), ctypes.c_int, P(vp)]),
    "stencil_p2p_run_until": (i32, [vp, ctypes.c_int, dbl, ctypes.c_int, vp, P(ctypes.c_int), P(dbl)]),
    "stencil_plan_create_dist": (i32, [P(vp), i64, i64, i64, ctypes.c_int, P(dbl), i32, vp, ctypes.c_int,
                                       ctypes.c_int]),
    "stencil_fill_counter": (i32, [vp, vp, ctypes.c_uint64, vp]),
}


APP_CODES = {"jacobi": 0, "source": 1, "wave": 2, "div": 3, "grad": 4}   # stencil_app_t


class StencilError(RuntimeError):
    def __init__(self, status: int, where: str, detail: str):
        self.status = status
        super().__init__(f"{where}: {STATUS.get(status, status)}: {detail}")


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(
            f"{LIB_PATH} is missing: build it with `python paper_conf_ipps_tangtkwkgtw13_b200/build.py` "
            "(there is no CPU fallback)")
    lib = ctypes.CDLL(LIB_PATH)
    for name, (res, args) in _SIGS.items():
        fn = getattr(lib, name)
        fn.restype = res
        fn.argtypes = args
    return lib


lib = _load()


def check(status: int, where: str):
    if status != 0:
        raise StencilError(status, where, lib.stencil_last_error_detail().decode())
