"""Python face of the C ABI: ``Plan`` objects over torch device memory.

Argument marshalling only -- every step of the sweep runs in libstencil.so.
torch supplies device memory, streams and (for ``DistPlan``) the process group
used to broadcast the NCCL id.
"""
from __future__ import annotations

import ctypes

import numpy as np

from . import _lib
from ._lib import Config, Layout, Stats, TuneEntry, TuneReport, check, lib

_NP = {"f32": np.float32, "f64": np.float64}


def layout_compute(nx: int, ny: int, nz: int, r: int, dtype: str = "f32") -> Layout:
    """Pitched layout of include/stencil.h (host only)."""
    L = Layout()
    check(lib.stencil_layout_compute(nx, ny, nz, r, _lib.DTYPE_CODES[dtype], ctypes.byref(L)), "layout_compute")
    return L


def _stream_handle(stream):
    import torch
    if stream is None:
        stream = torch.cuda.current_stream()
    return ctypes.c_void_p(stream.cuda_stream)


def _ptr(t):
    return ctypes.c_void_p(t.data_ptr())


class Plan:
    """A single-GPU plan bound to the current CUDA device.

    ``app``: "jacobi" (stencil_plan_create: Fig. 1 sweeps of Eq. 1), or an
    application stencil with a second grid (stencil_plan_create_app, Table V):
    "source" (u <- S(u) + d f, run_source) or "wave" (u+ = S(u) + d u-, run_wave).
    ``coeffs``: r+1 values c0..cr (Eq. 1, isotropic), or -- jacobi only -- 1+3r
    values c0, cx_1..cx_r, cy_1..cy_r, cz_1..cz_r (per-axis symmetric
    coefficients, stencil_plan_create_axes).
    """

    def __init__(self, nx: int, ny: int, nz: int, r: int, coeffs, dtype: str = "f32", app: str = "jacobi",
                 d: float = 0.0, _handle=None):
        self.dtype = dtype
        self.r = int(r)
        self.app = app
        coeffs = [float(x) for x in coeffs]
        self.axes = len(coeffs) == 1 + 3 * r
        if len(coeffs) != r + 1 and not (self.axes and app == "jacobi"):
            raise ValueError(f"need r+1 coefficients (or 1+3r per-axis ones for jacobi), got {len(coeffs)}")
        c = (ctypes.c_double * len(coeffs))(*coeffs)
        if _handle is None:
            h = ctypes.c_void_p()
            if self.axes:
                check(lib.stencil_plan_create_axes(ctypes.byref(h), nx, ny, nz, r, c, _lib.DTYPE_CODES[dtype]),
                      "plan_create_axes")
            elif app == "jacobi":
                check(lib.stencil_plan_create(ctypes.byref(h), nx, ny, nz, r, c, _lib.DTYPE_CODES[dtype]),
                      "plan_create")
            else:
                check(lib.stencil_plan_create_app(ctypes.byref(h), nx, ny, nz, r, c, _lib.DTYPE_CODES[dtype],
                                                  _lib.APP_CODES[app], float(d)), "plan_create_app")
            _handle = h
        self._h = _handle
        self.layout = Layout()
        check(lib.stencil_plan_layout(self._h, ctypes.byref(self.layout)), "plan_layout")

    # ---- lifetime ----------------------------------------------------------------
    def close(self):
        if getattr(self, "_h", None):
            lib.stencil_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    # ---- memory --------------------------------------------------------------------
    @property
    def np_dtype(self):
        return _NP[self.dtype]

    def alloc(self, device=None):
        """A zeroed device grid of layout.bytes (torch tensor, dtype of the plan)."""
        import torch
        L = self.layout
        tdt = torch.float32 if self.dtype == "f32" else torch.float64
        return torch.zeros(L.planes_z * L.rows_y * L.pitch_x, dtype=tdt, device=device or "cuda")

    def outer_view(self, t):
        """(nz+2r, ny+2r, nx+2r) view of a grid tensor (x fastest)."""
        L = self.layout
        v = t.view(L.planes_z, L.rows_y, L.pitch_x)
        return v[:, :, L.x_origin: L.x_origin + L.nx + 2 * L.radius]

    def interior_view(self, t):
        r = self.layout.radius
        return self.outer_view(t)[r:-r, r:-r, r:-r]

    def upload(self, outer: np.ndarray, t=None):
        """Copy a numpy outer grid into a (new) device grid; padding is zero."""
        import torch
        L = self.layout
        if outer.shape != (L.planes_z, L.rows_y, L.nx + 2 * L.radius):
            raise ValueError(f"outer grid shape {outer.shape} does not match the plan")
        if t is None:
            t = self.alloc()
        self.outer_view(t).copy_(torch.from_numpy(np.ascontiguousarray(outer, dtype=self.np_dtype)))
        return t

    def download(self, t) -> np.ndarray:
        return self.outer_view(t).cpu().numpy().copy()

    # ---- configuration -------------------------------------------------------------
    @property
    def config(self) -> dict:
        c = Config()
        check(lib.stencil_plan_get_config(self._h, ctypes.byref(c)), "get_config")
        d = c.as_dict()
        d["kernel"] = {v: k for k, v in _lib.KERNEL_CODES.items()}[d["kernel"]]
        return d

    def set_config(self, kernel="inplane", tx=32, ty=4, rx=None, ry=1, stages=4, zsegs=1, zbox=1, ytiles=0):
        vec = 4 if self.dtype == "f32" else 2
        if rx is None:
            rx = vec if kernel in _lib.TMA_KERNELS else 1
        c = Config(_lib.KERNEL_CODES[kernel], tx, ty, rx, ry, stages, zsegs, zbox, ytiles)
        check(lib.stencil_plan_set_config(self._h, ctypes.byref(c)), "set_config")

    # ---- execution ---------------------------------------------------------------
    def run(self, src, dst, iters: int, stream=None):
        """dst <- S^iters(src) (stencil_run); asynchronous on ``stream``."""
        check(lib.stencil_run(self._h, _ptr(src), _ptr(dst), int(iters), _stream_handle(stream)), "run")

    def residual_between(self, a, b, stream=None) -> float:
        """max over interior points |a - b| (stencil_residual, host-synchronous)"""
        res = ctypes.c_double(0.0)
        check(lib.stencil_residual(self._h, _ptr(a), _ptr(b), _stream_handle(stream), ctypes.byref(res)),
              "residual")
        return res.value

    def run_host(self, host_in, host_out, iters: int, stream=None):
        """host_out <- S^iters(host_in) for pinned HOST tensors of layout.bytes (stencil_run_host);
        successive calls pipeline upload / sweeps / download; follow with :meth:`host_wait`."""
        check(lib.stencil_run_host(self._h, _ptr(host_in), _ptr(host_out), int(iters), _stream_handle(stream)),
              "run_host")

    def host_wait(self, stream=None):
        """make ``stream`` wait for every download issued by run_host so far"""
        check(lib.stencil_run_host_wait(self._h, _stream_handle(stream)), "run_host_wait")

    def run_until(self, src, dst, max_iters: int, tol: float, check_every: int = 1, stream=None):
        """Fig. 1 with its stop criterion (stencil_run_until, host-synchronous):
        sweep until max|u_t - u_{t-1}| <= tol at a check; returns (sweeps, residual)."""
        n, res = ctypes.c_int(0), ctypes.c_double(0.0)
        check(lib.stencil_run_until(self._h, _ptr(src), _ptr(dst), int(max_iters), float(tol), int(check_every),
                                    _stream_handle(stream), ctypes.byref(n), ctypes.byref(res)), "run_until")
        return n.value, res.value

    def run_source(self, src, f, dst, iters: int, stream=None):
        """dst <- (u <- S(u) + d f)^iters (src) (stencil_run_source, SOURCE plans)."""
        check(lib.stencil_run_source(self._h, _ptr(src), _ptr(f), _ptr(dst), int(iters), _stream_handle(stream)),
              "run_source")

    def run_wave(self, u_prev, u, iters: int, stream=None):
        """``iters`` leapfrog steps in place (stencil_run_wave, WAVE plans)."""
        check(lib.stencil_run_wave(self._h, _ptr(u_prev), _ptr(u), int(iters), _stream_handle(stream)), "run_wave")

    def run_raw(self, src_ptr: int, dst_ptr: int, iters: int, stream_handle: int = 0):
        check(lib.stencil_run(self._h, ctypes.c_void_p(src_ptr), ctypes.c_void_p(dst_ptr), int(iters),
                              ctypes.c_void_p(stream_handle)), "run")

    def reserve(self):
        check(lib.stencil_plan_reserve(self._h), "reserve")

    def set_timing(self, mode=True):
        """0/False off, 1/True events around each run's sweeps, 2 an event after every sweep."""
        check(lib.stencil_plan_set_timing(self._h, int(mode)), "set_timing")

    def stats(self) -> dict:
        s = Stats()
        check(lib.stencil_plan_stats(self._h, ctypes.byref(s)), "stats")
        return {f: getattr(s, f) for f, _ in Stats._fields_}

    def fill_counter(self, t, seed: int, stream=None):
        check(lib.stencil_fill_counter(self._h, _ptr(t), ctypes.c_uint64(seed), _stream_handle(stream)),
              "fill_counter")

    # ---- tuning ----------------------------------------------------------------------
    def tune(self, kernel="inplane", model="b200", beta=5.0, iters_per_rep=4, reps=3, scratch=None,
             stream=None) -> dict:
        """stencil_tune (synchronous).  ``scratch``: two grids holding a valid input (clobbered)."""
        if scratch is None:
            raise ValueError("tune needs two scratch grids holding an input field")
        rep = TuneReport()
        m = _lib.MODEL_PAPER if model == "paper" else _lib.MODEL_B200
        check(lib.stencil_tune(self._h, _lib.KERNEL_CODES[kernel], m, float(beta), int(iters_per_rep), int(reps),
                               _ptr(scratch[0]), _ptr(scratch[1]), _stream_handle(stream), ctypes.byref(rep)),
              "tune")
        out = {f: getattr(rep, f) for f, _ in TuneReport._fields_}
        out["best"] = rep.best.as_dict()
        return out

    def tune_results(self) -> list:
        n = ctypes.c_int()
        check(lib.stencil_tune_results(self._h, None, 0, ctypes.byref(n)), "tune_results")
        arr = (TuneEntry * max(1, n.value))()
        check(lib.stencil_tune_results(self._h, arr, n.value, ctypes.byref(n)), "tune_results")
        res = []
        for e in arr[: n.value]:
            d = {f: getattr(e, f) for f, _ in TuneEntry._fields_ if f != "cfg"}
            d["cfg"] = e.cfg.as_dict()
            res.append(d)
        return res


def nccl_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    check(lib.stencil_nccl_unique_id(buf), "nccl_unique_id")
    return buf.raw


def slab_partition(nz_global: int, nranks: int, rank: int, r: int):
    z0, n = ctypes.c_int64(), ctypes.c_int64()
    check(lib.stencil_slab_partition(nz_global, nranks, rank, r, ctypes.byref(z0), ctypes.byref(n)),
          "slab_partition")
    return z0.value, n.value


def exchange_plan(layout: Layout, nranks: int, rank: int) -> dict:
    x = _lib.ExchangePlan()
    check(lib.stencil_exchange_plan(ctypes.byref(layout), nranks, rank, ctypes.byref(x)), "exchange_plan")
    return {f: getattr(x, f) for f, _ in _lib.ExchangePlan._fields_}


def p2p_targets(layout: Layout, nz_global: int, nranks: int, rank: int) -> dict:
    """host-only: where a p2p slab's fused boundary stores land (stencil_p2p_targets)"""
    t = _lib.P2PTargets()
    check(lib.stencil_p2p_targets(ctypes.byref(layout), int(nz_global), nranks, rank, ctypes.byref(t)),
          "p2p_targets")
    return {f: getattr(t, f) for f, _ in _lib.P2PTargets._fields_}


class DistPlan(Plan):
    """z-slab plan of one rank (stencil_plan_create_dist).  ``uid``: 128-byte NCCL id from rank 0."""

    def __init__(self, nx, ny, nz_global, r, coeffs, dtype, uid: bytes, rank: int, nranks: int):
        c = (ctypes.c_double * (r + 1))(*[float(x) for x in coeffs])
        h = ctypes.c_void_p()
        ub = ctypes.create_string_buffer(uid, 128)
        check(lib.stencil_plan_create_dist(ctypes.byref(h), nx, ny, nz_global, r, c, _lib.DTYPE_CODES[dtype], ub,
                                           rank, nranks), "plan_create_dist")
        self.rank, self.nranks, self.nz_global = rank, nranks, nz_global
        self.z0, self.nz_local = slab_partition(nz_global, nranks, rank, r)
        super().__init__(nx, ny, self.nz_local, r, coeffs, dtype, _handle=h)


class DivGrad(Plan):
    """Table V "Div" (3 grids -> 1) or "Grad" (1 -> 3) stencil (stencil_plan_create_divgrad).
    ``a``: the r first-derivative weights a_1..a_r (a_m multiplies f[+m] - f[-m])."""

    def __init__(self, nx, ny, nz, r, a, dtype="f32", app="div"):
        if len(a) != r:
            raise ValueError(f"need r = {r} weights a_1..a_r")
        c = (ctypes.c_double * r)(*[float(x) for x in a])
        h = ctypes.c_void_p()
        check(lib.stencil_plan_create_divgrad(ctypes.byref(h), nx, ny, nz, r, c, _lib.DTYPE_CODES[dtype],
                                              _lib.APP_CODES[app]), "plan_create_divgrad")
        super().__init__(nx, ny, nz, r, [0.0] * (r + 1), dtype, _handle=h)
        self.app = app

    def div(self, u, v, w, out, stream=None):
        """out <- Div(u, v, w) (stencil_run_div), asynchronous"""
        check(lib.stencil_run_div(self._h, _ptr(u), _ptr(v), _ptr(w), _ptr(out), _stream_handle(stream)), "run_div")

    def grad(self, f, gx, gy, gz, stream=None):
        """(gx, gy, gz) <- Grad(f) (stencil_run_grad), asynchronous"""
        check(lib.stencil_run_grad(self._h, _ptr(f), _ptr(gx), _ptr(gy), _ptr(gz), _stream_handle(stream)),
              "run_grad")


class LocalRankGroup:
    """All ranks of a distributed plan in ONE process (stencil_plan_create_dist_local): the DistPlan's
    partition, boundary/interior split, events and exchange offsets, with cudaMemcpyAsync as the
    transport (the multi-rank logic testable on one GPU)."""

    def __init__(self, nx, ny, nz_global, r, coeffs, dtype, nranks: int):
        c = (ctypes.c_double * (r + 1))(*[float(x) for x in coeffs])
        hs = (ctypes.c_void_p * nranks)()
        check(lib.stencil_plan_create_dist_local(hs, nx, ny, nz_global, r, c, _lib.DTYPE_CODES[dtype], nranks),
              "plan_create_dist_local")
        self.plans = []
        for k in range(nranks):
            z0, nzl = slab_partition(nz_global, nranks, k, r)
            q = Plan(nx, ny, nzl, r, coeffs, dtype, _handle=ctypes.c_void_p(hs[k]))
            q.z0, q.nz_local, q.rank, q.nranks = z0, nzl, k, nranks
            self.plans.append(q)

    def run(self, ins, outs, iters: int, streams):
        n = len(self.plans)
        hs = (ctypes.c_void_p * n)(*[q._h for q in self.plans])
        ip = (ctypes.c_void_p * n)(*[t.data_ptr() for t in ins])
        op = (ctypes.c_void_p * n)(*[t.data_ptr() for t in outs])
        sp = (ctypes.c_void_p * n)(*[_stream_handle(s) for s in streams])
        check(lib.stencil_run_dist_local(hs, n, ip, op, int(iters), sp), "run_dist_local")

    def close(self):
        for q in self.plans:
            q.close()

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()


class P2PSlab(Plan):
    """z-slab plan of one rank with the halo exchange fused into the sweep
    (stencil_plan_create_p2p).  The plan owns its two grids;
    neighbours are wired with :meth:`connect` (plans in this process) or
    :meth:`export_handles` / :meth:`import_handles` (CUDA IPC across processes).
    """

    def __init__(self, nx, ny, nz_global, r, coeffs, dtype, rank: int, nranks: int):
        c = (ctypes.c_double * (r + 1))(*[float(x) for x in coeffs])
        h = ctypes.c_void_p()
        check(lib.stencil_plan_create_p2p(ctypes.byref(h), nx, ny, nz_global, r, c, _lib.DTYPE_CODES[dtype],
                                          rank, nranks), "plan_create_p2p")
        self.rank, self.nranks, self.nz_global = rank, nranks, nz_global
        self.z0, self.nz_local = slab_partition(nz_global, nranks, rank, r)
        super().__init__(nx, ny, self.nz_local, r, coeffs, dtype, _handle=h)
        self.current = 0

    def endpoint(self):
        ep = _lib.P2PEndpoint()
        check(lib.stencil_p2p_endpoint(self._h, ctypes.byref(ep)), "p2p_endpoint")
        return ep

    def connect(self, lo=None, hi=None):
        """lo / hi: the neighbouring P2PSlab objects (same process) or None."""
        elo = lo.endpoint() if lo is not None else None
        ehi = hi.endpoint() if hi is not None else None
        check(lib.stencil_p2p_connect(self._h, ctypes.byref(elo) if elo else None,
                                      ctypes.byref(ehi) if ehi else None), "p2p_connect")

    def export_handles(self) -> bytes:
        buf = ctypes.create_string_buffer(192)
        check(lib.stencil_p2p_export(self._h, buf), "p2p_export")
        return buf.raw

    def import_handles(self, lo: bytes | None, hi: bytes | None):
        lb = ctypes.create_string_buffer(lo, 192) if lo else None
        hb = ctypes.create_string_buffer(hi, 192) if hi else None
        check(lib.stencil_p2p_import(self._h, lb, hb), "p2p_import")

    def grid_view(self, i: int):
        """torch view (outer shape) of plan-owned grid i (no copy)."""
        import torch
        ep = self.endpoint()
        L = self.layout
        n = L.planes_z * L.rows_y * L.pitch_x
        t = _device_tensor(ep.grid[i], n, torch.float32 if self.dtype == "f32" else torch.float64)
        v = t.view(L.planes_z, L.rows_y, L.pitch_x)
        return v[:, :, L.x_origin: L.x_origin + L.nx + 2 * L.radius]

    def fill_local(self, global_outer: np.ndarray):
        """Copy this rank's slab (its nz_local + 2r outer planes) of the GLOBAL outer field into both grids."""
        import torch
        r = self.layout.radius
        local = np.ascontiguousarray(global_outer[self.z0: self.z0 + self.nz_local + 2 * r], dtype=self.np_dtype)
        for i in (0, 1):
            self.grid_view(i).copy_(torch.from_numpy(local))
        self.current = 0

    def run(self, iters: int, stream=None):
        cur = ctypes.c_int(0)
        check(lib.stencil_p2p_run(self._h, int(iters), _stream_handle(stream), ctypes.byref(cur)), "p2p_run")
        self.current = cur.value
        return self.current

    def quiesce(self, stream=None):
        """stream-side wait until no neighbour peer store into this plan's grids is in flight"""
        check(lib.stencil_p2p_quiesce(self._h, _stream_handle(stream)), "p2p_quiesce")

    def grid_tensor(self, i: int):
        """flat torch tensor aliasing plan-owned grid i (layout.bytes)"""
        import torch
        ep = self.endpoint()
        L = self.layout
        return _device_tensor(ep.grid[i], L.planes_z * L.rows_y * L.pitch_x,
                              torch.float32 if self.dtype == "f32" else torch.float64)

    def residual(self, stream=None) -> float:
        """max over this slab's interior |u_e - u_{e-1}| after its latest sweep (host-synchronous)"""
        res = ctypes.c_double(0.0)
        check(lib.stencil_p2p_residual(self._h, _stream_handle(stream), ctypes.byref(res)), "p2p_residual")
        return res.value

    def run_until(self, max_iters: int, tol: float, check_every: int = 1, group=None, stream=None):
        """Fig. 1 with its stop criterion across the slabs (reading R5b), entirely in the library
        (stencil_p2p_run_until): sweeps in blocks of ``check_every``, the global residual reduced over
        the slabs on the devices through the mapped flag buffers.  Every rank calls it with the same
        arguments (``group`` is accepted for API compatibility and unused).  Returns (sweeps, residual)."""
        t, res = ctypes.c_int(0), ctypes.c_double(0.0)
        check(lib.stencil_p2p_run_until(self._h, int(max_iters), float(tol), int(check_every),
                                        _stream_handle(stream), ctypes.byref(t), ctypes.byref(res)), "p2p_run_until")
        self.current = self.endpoint_current()
        return t.value, res.value

    def endpoint_current(self) -> int:
        """index of the grid holding the latest state (epoch parity)"""
        cur = ctypes.c_int(0)
        check(lib.stencil_p2p_run(self._h, 0, None, ctypes.byref(cur)), "p2p_run")
        return cur.value

    def local_result(self) -> np.ndarray:
        """outer view of the grid holding the latest state, as numpy"""
        return self.grid_view(self.current).cpu().numpy().copy()


def _device_tensor(ptr: int, numel: int, dtype):
    """A torch tensor aliasing ``numel`` elements of device memory at ``ptr`` (owned by the library)."""
    import torch

    class _CAI:
        def __init__(self):
            typestr = "<f4" if dtype == torch.float32 else "<f8"
            self.__cuda_array_interface__ = {"shape": (numel,), "typestr": typestr, "data": (int(ptr), False),
                                             "version": 3, "strides": None}

    return torch.as_tensor(_CAI(), device="cuda")
