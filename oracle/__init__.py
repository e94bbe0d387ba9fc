"""ctypes wrapper around the CPU oracle (oracle/triosim_oracle.c).

TEST INFRASTRUCTURE ONLY: imported by tests/, __graft_entry__.smoke() and the
cpu_baseline / --impl reference leg of bench.py -- never by the product package
(paper_conf_isca_libwmvgjbj025_b200/), which must fail loudly without its CUDA
library instead of falling back here.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
import threading

import numpy as np

from paper_conf_isca_libwmvgjbj025_b200 import workloads as W

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "triosim_oracle.c")
LIB = os.path.join(HERE, "liboracle.so")
CFLAGS = ["-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math", "-Wall", "-Wno-unused-function", "-fPIC",
          "-shared"]

_lock = threading.Lock()
_lib = None


def build(force=False) -> str:
    """Compile liboracle.so (gcc, -O2 -ffp-contract=off: no FMA contraction, no fast-math)."""
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(SRC):
        tmp = LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, SRC, "-o", tmp, "-lm"])
        os.replace(tmp, LIB)
    return LIB


def lib():
    global _lib
    with _lock:
        if _lib is None:
            build()
            L = C.CDLL(LIB)
            P = C.c_void_p
            u32, i32, i64, f64 = C.c_uint32, C.c_int32, C.c_int64, C.c_double
            L.oracle_run_point.argtypes = [P, u32, P, u32, P, u32, u32, u32, u32, P, u32, P, P, u32, C.c_int, P, P, P,
                                           P, P, P, i64, P, i64, P, P]
            L.oracle_run_point.restype = C.c_int
            L.oracle_export_graph.argtypes = [P, u32, P, u32, P, u32, u32, u32, u32, P, u32, P, P, u32, C.c_int, P,
                                              P, P, P, P, P, P, P, P, P, P, P, P, P]
            L.oracle_export_graph.restype = C.c_int
            L.oracle_sim_graph.argtypes = [i64, P, P, P, P, P, P, P, P, P, P, i32, f64, u32, u32, P, u32, f64, f64, P, P, P]
            L.oracle_sim_graph.restype = C.c_int
            L.oracle_route.argtypes = [u32, u32, P, u32, u32, u32, P, i32]
            L.oracle_route.restype = C.c_int
            L.oracle_waterfill.argtypes = [i32, P, i32, P, P, P, P]
            L.oracle_waterfill.restype = C.c_int64
            L.oracle_partition.argtypes = [P, u32, P, u32, P, u32, u32, u32, P]
            L.oracle_partition.restype = C.c_int
            L.oracle_check_trace.argtypes = [P, u32, P, u32, P, u32, u32, P]
            L.oracle_check_trace.restype = C.c_int
            _lib = L
    return _lib


def _p(a):
    return None if a is None else a.ctypes.data_as(C.c_void_p)


def _trace_args(tr: W.Trace):
    ops = np.ascontiguousarray(tr.ops, W.OP_DTYPE)
    ts = np.ascontiguousarray(tr.tensors, W.TENSOR_DTYPE)
    io = np.ascontiguousarray(tr.io, np.uint32)
    keep = (ops, ts, io)
    return keep, [_p(ops), len(ops), _p(ts), len(ts), _p(io), len(io), int(tr.trace_batch)]


def _topo_args(topo: W.Topology):
    links = np.ascontiguousarray(topo.links, W.LINK_DTYPE)
    ro = None if topo.ring_order is None else np.ascontiguousarray(topo.ring_order, np.uint32)
    return (links, ro), [topo.n_nodes, topo.n_gpus, _p(links), len(links), _p(ro)]


def _phot(topo: W.Topology):
    ph = getattr(topo, "photonic", None)
    return None if ph is None else np.ascontiguousarray(np.asarray(ph, W.PHOTONIC_DTYPE).reshape(1))


class OracleError(RuntimeError):
    pass


def run_point(tr: W.Trace, topo: W.Topology, pt, plan=None, breakdown=False, timeline=False):
    """Simulate one design point; returns a RESULT_DTYPE record (and, with breakdown=True, the
    per-layer compute and communication times of DESIGN.md R22; with timeline=True, the R23 task
    and flow records, TASK_REC_DTYPE ordered by (gpu, prog) and FLOW_REC_DTYPE by (release, code))."""
    if timeline:
        return _run_point_timeline(tr, topo, pt, plan)
    k1, ta = _trace_args(tr)
    k2, tpa = _topo_args(topo)
    pl = None if plan is None else np.ascontiguousarray(plan, np.uint32)
    ptv = np.array(pt, W.POINT_DTYPE).reshape(1)
    out = np.zeros(1, W.RESULT_DTYPE)
    ph = _phot(topo)
    lc = lm = None
    if breakdown:
        lc, lm = np.zeros(max(tr.n_layers, 1)), np.zeros(max(tr.n_layers, 1))
    rc = lib().oracle_run_point(*ta, *tpa, _p(pl), 0 if pl is None else len(pl), 0 if pl is None else 1, _p(ptv),
                                _p(out), _p(ph), _p(lc), _p(lm), None, 0, None, 0, None, None)
    if rc != 0:
        raise OracleError(f"oracle_run_point rc={rc}")
    if breakdown:
        return out[0], lc[:tr.n_layers], lm[:tr.n_layers]
    return out[0]


def _run_point_timeline(tr, topo, pt, plan):
    k1, ta = _trace_args(tr)
    k2, tpa = _topo_args(topo)
    pl = None if plan is None else np.ascontiguousarray(plan, np.uint32)
    ptv = np.array(pt, W.POINT_DTYPE).reshape(1)
    ph = _phot(topo)
    nt, nf = C.c_int64(), C.c_int64()
    tasks = np.zeros(0, W.TASK_REC_DTYPE)
    flows = np.zeros(0, W.FLOW_REC_DTYPE)
    for _ in range(2):   # first call sizes the record arrays, the second fills them
        out = np.zeros(1, W.RESULT_DTYPE)
        rc = lib().oracle_run_point(*ta, *tpa, _p(pl), 0 if pl is None else len(pl), 0 if pl is None else 1, _p(ptv),
                                    _p(out), _p(ph), None, None, _p(tasks), len(tasks), _p(flows), len(flows),
                                    C.byref(nt), C.byref(nf))
        if rc != 0:
            raise OracleError(f"oracle_run_point rc={rc}")
        if nt.value <= len(tasks) and nf.value <= len(flows):
            return out[0], tasks[:nt.value], flows[:nf.value]
        tasks = np.zeros(nt.value, W.TASK_REC_DTYPE)
        flows = np.zeros(nf.value, W.FLOW_REC_DTYPE)
    raise OracleError("timeline sizes changed between calls")


def run_sweep(sw: W.Sweep, idx=None, breakdown=False):
    """Oracle results for points idx of a sweep; topology index and plan index are resolved
    here in DESIGN.md R3 order (topology first, the plan inside the point checks).  With
    breakdown=True also returns per-layer compute / comm arrays [len(idx), n_layers] (R22)."""
    idx = range(len(sw.points)) if idx is None else idx
    res = np.zeros(len(idx), W.RESULT_DTYPE)
    if breakdown:
        L = sw.trace.n_layers
        bc, bm = np.zeros((len(idx), L)), np.zeros((len(idx), L))
    for q, i in enumerate(idx):
        pt = sw.points[i]
        if pt["topo"] >= len(sw.topos):
            res[q]["status"] = W.PT_BAD_CONFIG
            continue
        plan = None
        if pt["stage_plan"] >= 0:
            plan = sw.plans[pt["stage_plan"]] if pt["stage_plan"] < len(sw.plans) else []
        if breakdown:
            res[q], bc[q], bm[q] = run_point(sw.trace, sw.topos[pt["topo"]], pt, plan, breakdown=True)
        else:
            res[q] = run_point(sw.trace, sw.topos[pt["topo"]], pt, plan)
    if breakdown:
        return res, bc, bm
    return res


def export_graph(tr, topo, pt, plan=None):
    """The explicit task graph the oracle builds for one point (dict of numpy arrays)."""
    k1, ta = _trace_args(tr)
    k2, tpa = _topo_args(topo)
    pl = None if plan is None else np.ascontiguousarray(plan, np.uint32)
    ptv = np.array(pt, W.POINT_DTYPE).reshape(1)
    nn, nd, st = np.zeros(1, np.int64), np.zeros(1, np.int64), np.zeros(1, np.int32)
    L = lib()
    args = [*ta, *tpa, _p(pl), 0 if pl is None else len(pl), 0 if pl is None else 1, _p(ptv)]
    rc = L.oracle_export_graph(*args, _p(nn), _p(nd), *([None] * 10), _p(st))
    if rc != 0:
        raise OracleError(f"export rc={rc}")
    n, m = int(nn[0]), int(nd[0])
    g = dict(type=np.zeros(n, np.int32), gpu=np.zeros(n, np.int32), dur=np.zeros(n), src=np.zeros(n, np.int32),
             dst=np.zeros(n, np.int32), bytes=np.zeros(n), code=np.zeros(n, np.uint64), flags=np.zeros(n, np.int32),
             dep_off=np.zeros(n + 1, np.int64), dep_ids=np.zeros(max(m, 1), np.int32))
    rc = L.oracle_export_graph(*args, _p(nn), _p(nd), _p(g["type"]), _p(g["gpu"]), _p(g["dur"]), _p(g["src"]),
                               _p(g["dst"]), _p(g["bytes"]), _p(g["code"]), _p(g["flags"]), _p(g["dep_off"]),
                               _p(g["dep_ids"]), _p(st))
    if rc != 0:
        raise OracleError(f"export rc={rc}")
    g["status"] = int(st[0])
    return g


def sim_graph(g, topo: W.Topology, bw_scale=1.0, lat_scale=1.0, n_coll=0, coll_payload=0.0, times=False):
    """Simulate an explicit task graph; with times=True also return per-node completion times."""
    k2, tpa = _topo_args(topo)
    n = len(g["type"])
    out = np.zeros(1, W.RESULT_DTYPE)
    td = np.full(max(n, 1), np.nan)
    arrs = [np.ascontiguousarray(g[k], dt) for k, dt in
            (("type", np.int32), ("gpu", np.int32), ("dur", np.float64), ("src", np.int32), ("dst", np.int32),
             ("bytes", np.float64), ("code", np.uint64), ("flags", np.int32), ("dep_off", np.int64),
             ("dep_ids", np.int32))]
    ph = _phot(topo)
    rc = lib().oracle_sim_graph(n, *[_p(a) for a in arrs], int(n_coll), float(coll_payload), *tpa[:4],
                                float(bw_scale), float(lat_scale), _p(out), _p(td), _p(ph))
    if rc != 0:
        raise OracleError(f"sim_graph rc={rc}")
    return (out[0], td[:n]) if times else out[0]


def route(topo: W.Topology, src, dst):
    links = np.ascontiguousarray(topo.links, W.LINK_DTYPE)
    out = np.zeros(topo.n_nodes + 1, np.int32)
    h = lib().oracle_route(topo.n_nodes, topo.n_gpus, _p(links), len(links), src, dst, _p(out), len(out))
    if h < -50:
        raise OracleError(f"route rc={h}")
    return None if h < 0 else [int(x) for x in out[:h]]


def waterfill(bw, routes):
    """Max-min progressive filling on given link bandwidths and flow routes (lists of link ids).
    Returns (rates, rounds)."""
    bw = np.ascontiguousarray(bw, np.float64)
    off = np.zeros(len(routes), np.int64)
    ln = np.zeros(len(routes), np.int32)
    flat = []
    for i, r in enumerate(routes):
        off[i] = len(flat)
        ln[i] = len(r)
        flat += list(r)
    fl = np.asarray(flat if flat else [0], np.int32)
    rate = np.zeros(len(routes))
    rounds = lib().oracle_waterfill(len(bw), _p(bw), len(routes), _p(off), _p(ln), _p(fl), _p(rate))
    return rate, int(rounds)


def partition(tr: W.Trace, S):
    k1, ta = _trace_args(tr)
    out = np.zeros(S, np.uint32)
    rc = lib().oracle_partition(*ta, S, _p(out))
    if rc != 0:
        raise OracleError(f"partition rc={rc}")
    return [int(x) for x in out]


def check_trace(tr: W.Trace):
    k1, ta = _trace_args(tr)
    nl = np.zeros(1, np.uint32)
    rc = lib().oracle_check_trace(*ta, _p(nl))
    return rc, int(nl[0])
