"""Hand-built traces and graphs for the closed-form pins (no method arithmetic)."""
from __future__ import annotations

import numpy as np

from paper_conf_isca_libwmvgjbj025_b200 import workloads as W


class HandTrace:
    def __init__(self, b0=1):
        self.b0 = b0
        self.ops, self.ts, self.io = [], [], []

    def tensor(self, nbytes, cat=W.CAT_ACT, scaled=True):
        self.ts.append((nbytes, cat, 1 if scaled else 0))
        return len(self.ts) - 1

    def op(self, layer, phase, ins, outs, time, role=0, scaled=True):
        self.ops.append((layer, phase, role, W.OPF_BATCH_SCALED if scaled else 0, len(self.io), len(ins), len(outs),
                         time))
        self.io += list(ins) + list(outs)
        return len(self.ops) - 1

    def build(self):
        ops = np.zeros(len(self.ops), W.OP_DTYPE)
        for i, (l, ph, r, fl, off, ni, no, t) in enumerate(self.ops):
            ops[i] = (1, l, ph, r, fl, off, ni, no, 0, t, 0.0)
        ts = np.zeros(len(self.ts), W.TENSOR_DTYPE)
        for i, (nb, c, s) in enumerate(self.ts):
            ts[i] = (nb, c, s, 0, 0)
        nl = int(max(o[0] for o in self.ops if o[1] == W.PH_FWD)) + 1
        return W.Trace("hand", ops, ts, np.asarray(self.io, np.uint32), self.b0, nl)


class HandGraph:
    """Explicit task graph in the oracle's export layout."""

    def __init__(self):
        self.nodes = []  # (type, gpu, dur, src, dst, bytes, code, flags)
        self.deps = []

    def task(self, gpu, dur, deps=()):
        self.nodes.append((0, gpu, dur, 0, 0, 0.0, len(self.nodes), 0))
        self.deps.append(list(deps))
        return len(self.nodes) - 1

    def flow(self, src, dst, nbytes, deps=()):
        self.nodes.append((1, 0, 0.0, src, dst, float(nbytes), len(self.nodes), 0))
        self.deps.append(list(deps))
        return len(self.nodes) - 1

    def barrier(self, deps=(), coll_start=False):
        self.nodes.append((2, 0, 0.0, 0, 0, 0.0, len(self.nodes), 1 if coll_start else 0))
        self.deps.append(list(deps))
        return len(self.nodes) - 1

    def arrays(self):
        n = len(self.nodes)
        g = {k: np.zeros(n, dt) for k, dt in (("type", np.int32), ("gpu", np.int32), ("dur", np.float64),
                                              ("src", np.int32), ("dst", np.int32), ("bytes", np.float64),
                                              ("code", np.uint64), ("flags", np.int32))}
        for i, nd in enumerate(self.nodes):
            for k, v in zip(("type", "gpu", "dur", "src", "dst", "bytes", "code", "flags"), nd):
                g[k][i] = v
        off = np.zeros(n + 1, np.int64)
        flat = []
        for i, d in enumerate(self.deps):
            flat += d
            off[i + 1] = len(flat)
        g["dep_off"] = off
        g["dep_ids"] = np.asarray(flat if flat else [0], np.int32)
        return g


def links_of(topo):
    return [(int(l["src"]), int(l["dst"]), float(l["bw_Bps"]), float(l["lat_s"])) for l in topo.links]


def one_wgrad_trace(S_bytes, t_f=2.0 ** -10, t_b=2.0 ** -9, t_o=0.0, role=0, n_opt=0):
    """FWD op -> loss; one BWD op producing a single weight gradient of S_bytes."""
    h = HandTrace(b0=1)
    x = h.tensor(64, W.CAT_INPUT)
    w = h.tensor(S_bytes, W.CAT_WEIGHT, scaled=False)
    y = h.tensor(64)
    h.op(0, W.PH_FWD, [x, w], [y], t_f, role=role)
    g = h.tensor(S_bytes, W.CAT_WGRAD, scaled=False)
    h.op(0, W.PH_BWD, [y, x], [g], t_b, role=role)
    for _ in range(n_opt):
        w2 = h.tensor(S_bytes, W.CAT_WEIGHT, scaled=False)
        h.op(0, W.PH_OPT, [w, g], [w2], t_o, scaled=False)
    return h.build()


def rel(a, b):
    return abs(a - b) / max(abs(b), 1e-300)
