"""Thin ctypes binding of libtriosim.so (include/triosim.h): argument marshalling only.

Every step of the hot path runs in the library's sm_100a kernels.  There is no
CPU fallback: importing works anywhere (so the CPU test-suite can check the
exported symbols), but creating a context fails loudly without the built
library or without a B200.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

from . import workloads as W

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("TRIOSIM_LIB", os.path.join(HERE, "libtriosim.so"))

EXPORTS = ["triosim_create", "triosim_destroy", "triosim_last_error", "triosim_load_trace", "triosim_build_sweep",
           "triosim_simulate_batch", "triosim_results", "triosim_release", "triosim_launch_counts",
           "triosim_results_device_ptr", "triosim_work_counters", "triosim_timing", "triosim_timings",
           "triosim_set_breakdown", "triosim_breakdown", "triosim_timeline", "triosim_stage_partition"]

STATUS = {0: "OK", -1: "EINVAL", -2: "ENOMEM", -3: "ECUDA", -4: "ENOTFOUND", -5: "ERANGE", -6: "EUNSUPPORTED"}


class TrioSimError(RuntimeError):
    def __init__(self, fn, status, msg=""):
        super().__init__(f"{fn}: {STATUS.get(status, status)} {msg}")
        self.status = status


class _TraceDesc(C.Structure):
    _fields_ = [("n_ops", C.c_uint32), ("n_tensors", C.c_uint32), ("n_io", C.c_uint32), ("trace_batch", C.c_uint32),
                ("ops", C.c_void_p), ("tensors", C.c_void_p), ("io", C.c_void_p)]


class _Topology(C.Structure):
    _fields_ = [("n_nodes", C.c_uint32), ("n_gpus", C.c_uint32), ("n_links", C.c_uint32), ("net_model", C.c_uint32),
                ("links", C.c_void_p), ("ring_order", C.c_void_p), ("photonic", C.c_void_p)]


NET_FLOW, NET_PHOTONIC = 0, 1


class _Plans(C.Structure):
    _fields_ = [("n_plans", C.c_uint32), ("off", C.c_void_p), ("first_layer", C.c_void_p)]


_lib = None


def load_library(path=LIB_PATH):
    """Load libtriosim.so (raises if it was not built -- no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(path):
            raise FileNotFoundError(f"{path} missing: run __graft_entry__.build() (nvcc, sm_100a)")
        L = C.CDLL(path)
        P, i32, u32, u64 = C.c_void_p, C.c_int32, C.c_uint32, C.c_uint64
        L.triosim_create.argtypes = [C.c_int, C.POINTER(P)]
        L.triosim_destroy.argtypes = [P]
        L.triosim_destroy.restype = None
        L.triosim_last_error.argtypes = [P]
        L.triosim_last_error.restype = C.c_char_p
        L.triosim_load_trace.argtypes = [P, C.POINTER(_TraceDesc), C.POINTER(i32)]
        L.triosim_build_sweep.argtypes = [P, i32, P, u32, P, P, u64, C.POINTER(i32)]
        L.triosim_simulate_batch.argtypes = [P, i32, u64, u64, P]
        L.triosim_results.argtypes = [P, i32, u64, u64, P, C.c_int, P]
        L.triosim_release.argtypes = [P, i32]
        L.triosim_launch_counts.argtypes = [P, C.POINTER(u64), C.POINTER(u64), C.POINTER(u64)]
        L.triosim_work_counters.argtypes = [P, i32, C.POINTER(u64)]
        L.triosim_timing.argtypes = [P, C.c_int]
        L.triosim_timings.argtypes = [P, P, P, i32]
        L.triosim_set_breakdown.argtypes = [P, i32, C.c_int]
        L.triosim_timeline.argtypes = [P, i32, u64, P, u64, P, u64, C.POINTER(u64), C.POINTER(u64)]
        L.triosim_breakdown.argtypes = [P, i32, u64, u64, P, P, C.c_int, P]
        L.triosim_results_device_ptr.argtypes = [P, i32]
        L.triosim_results_device_ptr.restype = P
        for f in EXPORTS:
            if f not in ("triosim_destroy", "triosim_last_error", "triosim_results_device_ptr"):
                getattr(L, f).restype = C.c_int32
        _lib = L
    return _lib


def _ptr(a):
    return None if a is None else a.ctypes.data_as(C.c_void_p)


def triosim_stage_partition(trace: W.Trace, n_stages: int) -> list:
    """Automatic GPipe stage plan (R8) as build_sweep computes it: host-only, no device."""
    L = load_library()
    ops = np.ascontiguousarray(trace.ops, W.OP_DTYPE)
    ts = np.ascontiguousarray(trace.tensors, W.TENSOR_DTYPE)
    io = np.ascontiguousarray(trace.io, np.uint32)
    d = _TraceDesc(len(ops), len(ts), len(io), int(trace.trace_batch), _ptr(ops), _ptr(ts), _ptr(io))
    out = np.zeros(max(int(n_stages), 1), np.uint32)
    st = L.triosim_stage_partition(C.byref(d), int(n_stages), _ptr(out))
    if st != 0:
        raise TrioSimError("triosim_stage_partition", st)
    return [int(x) for x in out[:n_stages]]


class Context:
    """One libtriosim context on one CUDA device (triosim_create)."""

    def __init__(self, device=0):
        self.L = load_library()
        self.h = C.c_void_p()
        st = self.L.triosim_create(int(device), C.byref(self.h))
        if st != 0:
            raise TrioSimError("triosim_create", st, "(needs a B200 / sm_100 device)")
        self._keep = {}

    def _check(self, fn, st):
        if st != 0:
            raise TrioSimError(fn, st, self.L.triosim_last_error(self.h).decode())

    def close(self):
        if self.h:
            self.L.triosim_destroy(self.h)
            self.h = C.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # -- the four calls of the boundary --
    def triosim_load_trace(self, trace: W.Trace) -> int:
        ops = np.ascontiguousarray(trace.ops, W.OP_DTYPE)
        ts = np.ascontiguousarray(trace.tensors, W.TENSOR_DTYPE)
        io = np.ascontiguousarray(trace.io, np.uint32)
        d = _TraceDesc(len(ops), len(ts), len(io), int(trace.trace_batch), _ptr(ops), _ptr(ts), _ptr(io))
        h = C.c_int32()
        self._check("triosim_load_trace", self.L.triosim_load_trace(self.h, C.byref(d), C.byref(h)))
        return h.value

    def triosim_build_sweep(self, trace_id: int, topos, points, plans=None) -> int:
        tarr = (_Topology * max(len(topos), 1))()
        keep = []
        for i, tp in enumerate(topos):
            links = np.ascontiguousarray(tp.links, W.LINK_DTYPE)
            ro = None if tp.ring_order is None else np.ascontiguousarray(tp.ring_order, np.uint32)
            ph = getattr(tp, "photonic", None)
            ph = None if ph is None else np.ascontiguousarray(np.asarray(ph, W.PHOTONIC_DTYPE).reshape(1))
            keep += [links, ro, ph]
            tarr[i] = _Topology(tp.n_nodes, tp.n_gpus, len(links), NET_FLOW if ph is None else NET_PHOTONIC,
                                _ptr(links), _ptr(ro), _ptr(ph))
        pl = None
        if plans:
            off = np.zeros(len(plans) + 1, np.uint32)
            flat = []
            for k, p in enumerate(plans):
                flat += list(p)
                off[k + 1] = len(flat)
            fl = np.asarray(flat if flat else [0], np.uint32)
            keep += [off, fl]
            pl = _Plans(len(plans), _ptr(off), _ptr(fl))
        pts = np.ascontiguousarray(points, W.POINT_DTYPE)
        h = C.c_int32()
        st = self.L.triosim_build_sweep(self.h, int(trace_id), C.cast(tarr, C.c_void_p), len(topos),
                                        C.cast(C.pointer(pl), C.c_void_p) if pl is not None else None, _ptr(pts),
                                        len(pts), C.byref(h))
        self._check("triosim_build_sweep", st)
        return h.value

    def triosim_simulate_batch(self, sweep_id: int, first: int, count: int, stream=0):
        """stream: a cudaStream_t handle as int (e.g. torch.cuda.current_stream().cuda_stream); 0 = default."""
        st = self.L.triosim_simulate_batch(self.h, int(sweep_id), int(first), int(count),
                                           C.c_void_p(int(stream)) if stream else None)
        self._check("triosim_simulate_batch", st)

    def triosim_results(self, sweep_id: int, first: int, count: int, out=None, device_ptr=None, stream=0):
        """Host results (numpy RESULT_DTYPE) or, with device_ptr, a stream-ordered copy into device memory."""
        if device_ptr is not None:
            st = self.L.triosim_results(self.h, int(sweep_id), int(first), int(count), C.c_void_p(int(device_ptr)), 1,
                                        C.c_void_p(int(stream)) if stream else None)
            self._check("triosim_results", st)
            return None
        if out is None:
            out = np.zeros(count, W.RESULT_DTYPE)
        st = self.L.triosim_results(self.h, int(sweep_id), int(first), int(count), _ptr(out), 0,
                                    C.c_void_p(int(stream)) if stream else None)
        self._check("triosim_results", st)
        return out

    def triosim_set_breakdown(self, sweep_id: int, enable=True):
        """Record the per-layer breakdown (R22) in later simulate_batch calls."""
        self._check("triosim_set_breakdown", self.L.triosim_set_breakdown(self.h, int(sweep_id), 1 if enable else 0))

    def triosim_breakdown(self, sweep_id: int, first: int, count: int, n_layers: int, device_ptrs=None, stream=0):
        """Per-layer (compute, comm) times [count, n_layers] as numpy arrays, or, with device_ptrs =
        (compute_ptr, comm_ptr), a stream-ordered write into device memory."""
        sp = C.c_void_p(int(stream)) if stream else None
        if device_ptrs is not None:
            cp, mp = (None if v is None else C.c_void_p(int(v)) for v in device_ptrs)
            self._check("triosim_breakdown", self.L.triosim_breakdown(self.h, int(sweep_id), int(first), int(count),
                                                                      cp, mp, 1, sp))
            return None
        comp = np.zeros((count, n_layers))
        comm = np.zeros((count, n_layers))
        self._check("triosim_breakdown", self.L.triosim_breakdown(self.h, int(sweep_id), int(first), int(count),
                                                                  _ptr(comp), _ptr(comm), 0, sp))
        return comp, comm

    def triosim_timeline(self, sweep_id: int, point: int, task_cap=None, flow_cap=None):
        """R23 timeline of one point: (tasks TASK_REC_DTYPE sorted by (gpu, prog), flows FLOW_REC_DTYPE sorted
        by (release, code)).  Without caps, a first call sizes the arrays."""
        nt, nf = C.c_uint64(), C.c_uint64()
        for _ in range(2):
            tc = 0 if task_cap is None else int(task_cap)
            fc = 0 if flow_cap is None else int(flow_cap)
            tasks = np.zeros(tc, W.TASK_REC_DTYPE)
            flows = np.zeros(fc, W.FLOW_REC_DTYPE)
            self._check("triosim_timeline", self.L.triosim_timeline(self.h, int(sweep_id), int(point), _ptr(tasks), tc,
                                                                    _ptr(flows), fc, C.byref(nt), C.byref(nf)))
            if nt.value <= tc and nf.value <= fc:
                return tasks[:nt.value], flows[:nf.value]
            task_cap, flow_cap = nt.value, nf.value
        raise TrioSimError("triosim_timeline", -1, "record counts changed between calls")

    def triosim_release(self, handle: int):
        self._check("triosim_release", self.L.triosim_release(self.h, int(handle)))

    def launch_counts(self):
        a, b, c = C.c_uint64(), C.c_uint64(), C.c_uint64()
        self._check("triosim_launch_counts", self.L.triosim_launch_counts(self.h, C.byref(a), C.byref(b), C.byref(c)))
        return a.value, b.value, c.value

    def timing(self, enable=True):
        self._check("triosim_timing", self.L.triosim_timing(self.h, 1 if enable else 0))

    def timings(self, max_n=512):
        tot = np.zeros(max_n, np.float32)
        k3 = np.zeros(max_n, np.float32)
        n = self.L.triosim_timings(self.h, _ptr(tot), _ptr(k3), max_n)
        if n < 0:
            self._check("triosim_timings", n)
        return tot[:n], k3[:n]

    def work_counters(self, sweep_id: int) -> int:
        v = C.c_uint64()
        self._check("triosim_work_counters", self.L.triosim_work_counters(self.h, int(sweep_id), C.byref(v)))
        return v.value

    def results_device_ptr(self, sweep_id: int) -> int:
        return self.L.triosim_results_device_ptr(self.h, int(sweep_id)) or 0

    # -- convenience --
    def run_sweep(self, sw: W.Sweep, stream=0, breakdown=False):
        """Results of every point; with breakdown=True also the per-layer (compute, comm) arrays (R22)."""
        tid = self.triosim_load_trace(sw.trace)
        sid = self.triosim_build_sweep(tid, sw.topos, sw.points, sw.plans or None)
        if breakdown:
            self.triosim_set_breakdown(sid, True)
        self.triosim_simulate_batch(sid, 0, len(sw.points), stream)
        res = self.triosim_results(sid, 0, len(sw.points), stream=stream)
        if breakdown:
            bd = self.triosim_breakdown(sid, 0, len(sw.points), sw.trace.n_layers, stream=stream)
        self.triosim_release(sid)
        self.triosim_release(tid)
        return (res, *bd) if breakdown else res
