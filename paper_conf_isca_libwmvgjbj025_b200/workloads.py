"""Seeded synthetic inputs: record layouts, operator traces, topologies, sweeps.

This module is the ONLY thing shared by the CUDA product path and the CPU
oracle (oracle/).  It holds none of the method's arithmetic -- no operator-time
model, no extrapolation, no routing, no bandwidth allocation.  It only writes
input records in the binary layouts of DESIGN.md "Inputs" (= include/triosim.h):

* traces shaped like the paper's workloads (ResNet, BERT, GPT-2; MLP for
  the closed-form case) -- an operator table (name/kind, measured time, input
  and output tensor ids) and a tensor table (bytes, category), P:150, P:156;
* topology templates (ring, NVSwitch-like star, 2D mesh, DGX-1-style hybrid
  cube-mesh, ring-based graph and double ring of P:362, asymmetric versions
  with every link slowed by U[1,10]);
* the design-point sweeps of BASELINE.json configs[0..3].

Synthetic operator times: t = flops/P + bytes/BW + 3 us, times a seeded
lognormal jitter (sigma 0.1), on an A100-class device.  The paper's own
traces are not available.
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

import numpy as np

# --------------------------------------------------------------------------
# record layouts (little endian, natural alignment) -- DESIGN.md "Inputs"
# --------------------------------------------------------------------------
OP_DTYPE = np.dtype([
    ("kind", "<u4"), ("layer", "<u4"), ("phase", "u1"), ("tp_role", "u1"), ("flags", "<u2"),
    ("io_off", "<u4"), ("n_in", "<u2"), ("n_out", "<u2"), ("pad", "<u4"),
    ("time_s", "<f8"), ("flops", "<f8")])
TENSOR_DTYPE = np.dtype([
    ("bytes_b0", "<u8"), ("category", "u1"), ("batch_scaled", "u1"), ("pad", "<u2"), ("param_id", "<u4")])
LINK_DTYPE = np.dtype([("src", "<u4"), ("dst", "<u4"), ("bw_Bps", "<f8"), ("lat_s", "<f8")])
POINT_DTYPE = np.dtype([
    ("topo", "<u4"), ("strategy", "u1"), ("tp_mode", "u1"), ("coll_algo", "u1"), ("ring_chunks", "u1"),
    ("dp", "<u2"), ("tp", "<u2"), ("pp", "<u2"), ("hop", "<u2"),
    ("microbatches", "<u4"), ("global_batch", "<u4"), ("stage_plan", "<i4"), ("first_bucket_bytes", "<u4"),
    ("bucket_bytes", "<u8"), ("bw_scale", "<f8"), ("lat_scale", "<f8")])
PHOTONIC_DTYPE = np.dtype([("ports", "<u4"), ("buf_slots", "<u4"), ("link_bw_Bps", "<f8"), ("setup_s", "<f8"),
                           ("lat_s", "<f8")])
RESULT_DTYPE = np.dtype([
    ("iter_time_s", "<f8"), ("compute_busy_max_s", "<f8"), ("comm_busy_s", "<f8"),
    ("exposed_comm_s", "<f8"), ("coll_payload_bytes", "<f8"),
    ("n_compute", "<u8"), ("n_flows", "<u8"), ("n_collectives", "<u8"), ("n_p2p", "<u8"),
    ("n_instants", "<u8"), ("n_wf_calls", "<u8"), ("n_wf_rounds", "<u8"), ("order_hash", "<u8"),
    ("status", "<i4"), ("max_active_flows", "<u4")])
# R23 timeline records (include/triosim.h triosim_task_rec / triosim_flow_rec)
TASK_REC_DTYPE = np.dtype([("gpu", "<u4"), ("prog", "<u4"), ("op", "<u4"), ("mb", "<u4"), ("start_s", "<f8"),
                           ("end_s", "<f8")])
FLOW_REC_DTYPE = np.dtype([("code", "<u8"), ("src", "<u4"), ("dst", "<u4"), ("bytes", "<f8"), ("release_s", "<f8"),
                           ("start_s", "<f8"), ("delivered_s", "<f8")])
assert TASK_REC_DTYPE.itemsize == 32 and FLOW_REC_DTYPE.itemsize == 48
assert OP_DTYPE.itemsize == 40 and TENSOR_DTYPE.itemsize == 16 and LINK_DTYPE.itemsize == 24
assert POINT_DTYPE.itemsize == 56 and RESULT_DTYPE.itemsize == 112

PH_FWD, PH_BWD, PH_OPT = 0, 1, 2
CAT_INPUT, CAT_WEIGHT, CAT_WGRAD, CAT_ACT, CAT_AGRAD, CAT_OTHER = range(6)
ROLE_NONE, ROLE_COL, ROLE_ROW, ROLE_LOCAL, ROLE_GATHER = 0, 1, 2, 3, 4
OPF_BATCH_SCALED = 1
ST_DP, ST_DDP, ST_TP, ST_PP, ST_HYBRID, ST_HOP = range(6)
HOP_RING_BASED, HOP_DOUBLE_RING = 0, 1   # R28 communication graphs (Fig. 16a), in tp_mode
TPM_PAPER, TPM_MEGATRON = 0, 1
ALG_RING, ALG_TREE, ALG_REDBCAST, ALG_DBTREE, ALG_RSAG = 0, 1, 2, 3, 4
PT_OK, PT_BAD_BATCH, PT_BAD_DEGREES, PT_NO_ROUTE, PT_TOO_LARGE, PT_DEADLOCK, PT_BAD_PLAN, PT_BAD_CONFIG = range(8)

MiB = 1 << 20

KINDS = {}


def kind_id(name: str) -> int:
    if name not in KINDS:
        KINDS[name] = len(KINDS) + 1
    return KINDS[name]


# --------------------------------------------------------------------------
# traces
# --------------------------------------------------------------------------
@dataclass
class Trace:
    name: str
    ops: np.ndarray          # OP_DTYPE
    tensors: np.ndarray      # TENSOR_DTYPE
    io: np.ndarray           # uint32
    trace_batch: int
    n_layers: int
    meta: dict = field(default_factory=dict)


class TraceBuilder:
    """Builds an operator trace in program order with a small reverse-mode tape.

    Forward modules emit FWD ops and push a backward closure; ``backward()``
    replays the tape in reverse (accumulating partial activation gradients with
    explicit add ops) and ``optimizer()`` emits one SGD update per parameter.
    """

    def __init__(self, name, b0, seed, peak_flops=1.0e14, mem_bw=1.5e12, overhead=3e-6, jitter=0.1,
                 act_bytes=4):
        self.name = name
        self.b0 = b0
        self.rng = np.random.Generator(np.random.PCG64(seed))
        self.peak, self.bw, self.ovh, self.jit = peak_flops, mem_bw, overhead, jitter
        self.ab = act_bytes
        self.ops, self.ts, self.io = [], [], []
        self.tape = []
        self.grads = {}          # activation tensor -> list of partial gradient tensors
        self.needs_grad = set()
        self.params = []         # (tensor, layer)
        self.layer = 0
        self.max_layer = -1

    # -- tables --
    def tensor(self, nbytes, cat, batch_scaled, param_id=0):
        self.ts.append((int(nbytes), cat, 1 if batch_scaled else 0, param_id))
        return len(self.ts) - 1

    def op(self, kind, phase, ins, outs, flops=0.0, mem=0.0, role=ROLE_NONE, scaled=True, layer=None, time=None):
        layer = self.layer if layer is None else layer
        if phase == PH_FWD:
            self.max_layer = max(self.max_layer, layer)
        if time is None:
            time = (flops / self.peak + mem / self.bw + self.ovh) * float(self.rng.lognormal(0.0, self.jit))
        self.ops.append((kind_id(kind), layer, phase, role, OPF_BATCH_SCALED if scaled else 0,
                         len(self.io), len(ins), len(outs), float(time), float(flops)))
        self.io.extend(int(x) for x in ins)
        self.io.extend(int(x) for x in outs)
        return len(self.ops) - 1

    def nbytes(self, x):
        return self.ts[x][0]

    def act(self, nbytes):
        return self.tensor(nbytes, CAT_ACT, True)

    def param(self, numel, pbytes=4):
        p = self.tensor(numel * pbytes, CAT_WEIGHT, False, param_id=len(self.params))
        self.params.append((p, self.layer))
        return p

    def _push(self, out, ins, fn):
        if any(i in self.needs_grad for i in ins):
            self.needs_grad.add(out)
        self.tape.append((self.layer, out, ins, fn))

    def _grad(self, x, g):
        if x in self.needs_grad:
            self.grads.setdefault(x, []).append(g)

    # -- modules (each is one operator forward and its backward operators) --
    def linear(self, x, fin, fout, tokens, role=ROLE_NONE, bias=True, gather=True):
        r = role | (ROLE_GATHER if gather else 0)
        W = self.param(fin * fout)
        b = self.param(fout) if bias else None
        y = self.act(tokens * fout * self.ab)
        fl = 2.0 * tokens * fin * fout
        ins = [x, W] + ([b] if bias else [])
        self.op("linear", PH_FWD, ins, [y], fl, self.nbytes(x) + self.nbytes(y) + 4 * fin * fout, role=r)
        self.needs_grad.add(W)

        def bwd(dy):
            if x in self.needs_grad:
                dx = self.tensor(self.nbytes(x), CAT_AGRAD, True)
                self.op("linear_grad_input", PH_BWD, [dy, W], [dx], fl, 2 * self.nbytes(x), role=r)
                self._grad(x, dx)
            dW = self.tensor(4 * fin * fout, CAT_WGRAD, False)
            self.op("linear_grad_weight", PH_BWD, [dy, x], [dW], fl, self.nbytes(x) + self.nbytes(dy), role=r)
            if bias:
                db = self.tensor(4 * fout, CAT_WGRAD, False)
                self.op("linear_grad_bias", PH_BWD, [dy], [db], 0.0, self.nbytes(dy), role=r)
                return [(W, dW), (b, db)]
            return [(W, dW)]
        self._push(y, [x, W], bwd)
        return y

    def conv(self, x, cin, cout, k, stride, hw_in, n):
        hw = (hw_in + stride - 1) // stride
        W = self.param(cin * cout * k * k)
        y = self.act(n * cout * hw * hw * self.ab)
        fl = 2.0 * n * hw * hw * cout * cin * k * k
        self.op("conv2d", PH_FWD, [x, W], [y], fl, self.nbytes(x) + self.nbytes(y), role=ROLE_GATHER)
        self.needs_grad.add(W)

        def bwd(dy):
            if x in self.needs_grad:
                dx = self.tensor(self.nbytes(x), CAT_AGRAD, True)
                self.op("conv2d_grad_input", PH_BWD, [dy, W], [dx], fl, 2 * self.nbytes(x), role=ROLE_GATHER)
                self._grad(x, dx)
            dW = self.tensor(4 * cin * cout * k * k, CAT_WGRAD, False)
            self.op("conv2d_grad_weight", PH_BWD, [dy, x], [dW], fl, self.nbytes(x) + self.nbytes(dy),
                    role=ROLE_GATHER)
            return [(W, dW)]
        self._push(y, [x, W], bwd)
        return y, hw

    def norm(self, x, C, kind="batch_norm", role=ROLE_NONE):
        g = self.param(C)
        b = self.param(C)
        y = self.act(self.nbytes(x))
        self.op(kind, PH_FWD, [x, g, b], [y], 8.0 * self.nbytes(x) / self.ab, 2 * self.nbytes(x), role=role)
        self.needs_grad.update((g, b))

        def bwd(dy):
            dx = self.tensor(self.nbytes(x), CAT_AGRAD, True)
            dg = self.tensor(4 * C, CAT_WGRAD, False)
            db = self.tensor(4 * C, CAT_WGRAD, False)
            self.op(kind + "_backward", PH_BWD, [dy, x, g], [dx, dg, db], 12.0 * self.nbytes(x) / self.ab,
                    3 * self.nbytes(x), role=role)
            self._grad(x, dx)
            return [(g, dg), (b, db)]
        self._push(y, [x, g, b], bwd)
        return y

    def pointwise(self, x, kind, role=ROLE_NONE, save_out=True):
        y = self.act(self.nbytes(x))
        self.op(kind, PH_FWD, [x], [y], 1.0 * self.nbytes(x) / self.ab, 2 * self.nbytes(x), role=role)

        def bwd(dy):
            dx = self.tensor(self.nbytes(x), CAT_AGRAD, True)
            self.op(kind + "_backward", PH_BWD, [dy, y if save_out else x], [dx], 1.0 * self.nbytes(x) / self.ab,
                    3 * self.nbytes(x), role=role)
            self._grad(x, dx)
            return []
        self._push(y, [x], bwd)
        return y

    def resize(self, x, out_bytes, kind):
        """pooling / reshaping operator with its own backward"""
        y = self.act(out_bytes)
        self.op(kind, PH_FWD, [x], [y], 1.0 * self.nbytes(x) / self.ab, self.nbytes(x) + out_bytes)

        def bwd(dy):
            dx = self.tensor(self.nbytes(x), CAT_AGRAD, True)
            self.op(kind + "_backward", PH_BWD, [dy], [dx], 1.0 * self.nbytes(x) / self.ab, self.nbytes(x) + out_bytes)
            self._grad(x, dx)
            return []
        self._push(y, [x], bwd)
        return y

    def add(self, a, b):
        y = self.act(self.nbytes(a))
        self.op("add", PH_FWD, [a, b], [y], 1.0 * self.nbytes(a) / self.ab, 3 * self.nbytes(a))

        def bwd(dy):
            self._grad(a, dy)
            self._grad(b, dy)
            return []
        self._push(y, [a, b], bwd)
        return y

    def bmm(self, a, b, out_bytes, flops, role=ROLE_NONE):
        y = self.act(out_bytes)
        self.op("bmm", PH_FWD, [a, b], [y], flops, self.nbytes(a) + self.nbytes(b) + out_bytes, role=role)

        def bwd(dy):
            da = self.tensor(self.nbytes(a), CAT_AGRAD, True)
            self.op("bmm_grad_a", PH_BWD, [dy, b], [da], flops, self.nbytes(a) + out_bytes, role=role)
            self._grad(a, da)
            db_ = self.tensor(self.nbytes(b), CAT_AGRAD, True)
            self.op("bmm_grad_b", PH_BWD, [dy, a], [db_], flops, self.nbytes(b) + out_bytes, role=role)
            self._grad(b, db_)
            return []
        self._push(y, [a, b], bwd)
        return y

    def embedding(self, ids, vocab, dim, tokens, role=ROLE_NONE):
        W = self.param(vocab * dim)
        y = self.act(tokens * dim * self.ab)
        self.op("embedding", PH_FWD, [ids, W], [y], 0.0, 2 * self.nbytes(y), role=role | ROLE_GATHER)
        self.needs_grad.add(W)

        def bwd(dy):
            dW = self.tensor(4 * vocab * dim, CAT_WGRAD, False)
            self.op("embedding_backward", PH_BWD, [dy, ids], [dW], 0.0, 2 * self.nbytes(dy) + 4 * vocab * dim,
                    role=role | ROLE_GATHER)
            return [(W, dW)]
        self._push(y, [ids, W], bwd)
        return y

    def loss(self, logits, labels):
        y = self.tensor(4, CAT_OTHER, False)
        self.op("cross_entropy", PH_FWD, [logits, labels], [y], 4.0 * self.nbytes(logits) / self.ab,
                2 * self.nbytes(logits))
        self.loss_inputs = (logits, labels)
        return y

    # -- passes --
    def backward(self):
        logits, labels = self.loss_inputs
        last_layer = self.max_layer
        dl = self.tensor(self.nbytes(logits), CAT_AGRAD, True)
        self.op("cross_entropy_backward", PH_BWD, [logits, labels], [dl], 4.0 * self.nbytes(logits) / self.ab,
                2 * self.nbytes(logits), layer=last_layer)
        self.grads[logits] = [dl]
        for layer, out, ins, fn in reversed(self.tape):
            parts = self.grads.pop(out, [])
            if not parts:
                continue
            dy = parts[0]
            for extra in parts[1:]:
                acc = self.tensor(self.nbytes(dy), CAT_AGRAD, True)
                self.op("add_grad", PH_BWD, [dy, extra], [acc], 1.0 * self.nbytes(dy) / self.ab,
                        3 * self.nbytes(dy), layer=layer)
                dy = acc
            self.layer = layer
            for p, g in fn(dy):
                self.pgrad[p] = g

    def optimizer(self):
        for p, layer in self.params:
            g = self.pgrad.get(p)
            if g is None:
                continue
            newp = self.tensor(self.nbytes(p), CAT_WEIGHT, False, param_id=self.ts[p][3])
            self.op("sgd_update", PH_OPT, [p, g], [newp], 2.0 * self.nbytes(p) / 4, 3 * self.nbytes(p),
                    scaled=False, layer=layer)

    def build(self, **meta) -> Trace:
        ops = np.zeros(len(self.ops), OP_DTYPE)
        for i, (k, l, ph, r, fl, off, ni, no, t, f) in enumerate(self.ops):
            ops[i] = (k, l, ph, r, fl, off, ni, no, 0, t, f)
        ts = np.zeros(len(self.ts), TENSOR_DTYPE)
        for i, (nb, c, bs, pid) in enumerate(self.ts):
            ts[i] = (nb, c, bs, 0, pid)
        return Trace(self.name, ops, ts, np.asarray(self.io, np.uint32), self.b0, self.max_layer + 1, meta)

    def start(self):
        self.pgrad = {}


def mlp_trace(n_layers=4, width=1024, b0=64, seed=0, dyadic=True) -> Trace:
    """Config 1: 4 x Linear(1024,1024)+ReLU, fp32.  With dyadic=True every op time is a
    small multiple of 2^-20 s so compute sums are exact (closed forms CF10/CF11)."""
    tb = TraceBuilder("mlp4x1024", b0, seed)
    tb.start()
    x = tb.tensor(b0 * width * 4, CAT_INPUT, True)
    labels = tb.tensor(b0 * 8, CAT_INPUT, True)
    h = x
    for l in range(n_layers):
        tb.layer = l
        h = tb.linear(h, width, width, b0)
        h = tb.pointwise(h, "relu")
    tb.loss(h, labels)
    tb.backward()
    tb.optimizer()
    tr = tb.build(model="mlp")
    if dyadic:
        q = 2.0 ** -20
        rng = np.random.Generator(np.random.PCG64(seed + 1))
        tr.ops["time_s"] = q * rng.integers(8, 128, len(tr.ops)).astype(np.float64)
    return tr


def resnet50_trace(b0=128, seed=2) -> Trace:
    """ResNet-50 (224x224, fp32) operator trace: 53 conv + 53 BN + fc -> 161 parameter tensors."""
    tb = TraceBuilder("resnet50", b0, seed)
    tb.start()
    img = tb.tensor(b0 * 3 * 224 * 224 * 4, CAT_INPUT, True)
    labels = tb.tensor(b0 * 8, CAT_INPUT, True)
    tb.layer = 0
    h, hw = tb.conv(img, 3, 64, 7, 2, 224, b0)
    h = tb.norm(h, 64)
    h = tb.pointwise(h, "relu")
    hw = hw // 2
    h = tb.resize(h, b0 * 64 * hw * hw * 4, "max_pool2d")
    cin = 64
    layer = 0
    for stage, (width, blocks, stride) in enumerate([(64, 3, 1), (128, 4, 2), (256, 6, 2), (512, 3, 2)]):
        for bi in range(blocks):
            layer += 1
            tb.layer = layer
            s = stride if bi == 0 else 1
            cout = width * 4
            idn = h
            y, hw1 = tb.conv(h, cin, width, 1, 1, hw, b0)
            y = tb.pointwise(tb.norm(y, width), "relu")
            y, hw2 = tb.conv(y, width, width, 3, s, hw1, b0)
            y = tb.pointwise(tb.norm(y, width), "relu")
            y, hw3 = tb.conv(y, width, cout, 1, 1, hw2, b0)
            y = tb.norm(y, cout)
            if bi == 0:
                idn, _ = tb.conv(h, cin, cout, 1, s, hw, b0)
                idn = tb.norm(idn, cout)
            h = tb.pointwise(tb.add(y, idn), "relu")
            cin, hw = cout, hw3
    layer += 1
    tb.layer = layer
    h = tb.resize(h, b0 * 2048 * 4, "adaptive_avg_pool2d")
    h = tb.linear(h, 2048, 1000, b0)
    tb.loss(h, labels)
    tb.backward()
    tb.optimizer()
    return tb.build(model="resnet50")


def vgg11_trace(b0=128, seed=6) -> Trace:
    """VGG-11 (224x224, fp32): 8 conv + ReLU (max pools after conv 1, 2, 4, 6, 8), 3 linear layers -> 14
    parameter tensors (bias-free convolutions, as TraceBuilder.conv), 132.9 M parameters; the Hop case study's
    model at its batch size 128."""
    tb = TraceBuilder("vgg11", b0, seed)
    tb.start()
    img = tb.tensor(b0 * 3 * 224 * 224 * 4, CAT_INPUT, True)
    labels = tb.tensor(b0 * 8, CAT_INPUT, True)
    h, hw, cin = img, 224, 3
    layer = 0
    for cout, pool in ((64, True), (128, True), (256, False), (256, True), (512, False), (512, True),
                       (512, False), (512, True)):
        tb.layer = layer
        h, hw = tb.conv(h, cin, cout, 3, 1, hw, b0)
        h = tb.pointwise(h, "relu")
        if pool:
            hw //= 2
            h = tb.resize(h, b0 * cout * hw * hw * 4, "max_pool2d")
        cin = cout
        layer += 1
    for fin, fout in ((512 * 7 * 7, 4096), (4096, 4096), (4096, 1000)):
        tb.layer = layer
        h = tb.linear(h, fin, fout, b0)
        if fout != 1000:
            h = tb.pointwise(h, "relu")
        layer += 1
    tb.loss(h, labels)
    tb.backward()
    tb.optimizer()
    return tb.build(model="vgg11")


def transformer_trace(name, n_layers, hidden, heads, ffn, seq, vocab, b0, seed, causal_head=True,
                      act_bytes=2) -> Trace:
    """Encoder/decoder-block transformer (BERT-large / GPT-2 XL shapes), fused QKV, fp16
    activations, Megatron roles: QKV/fc1 column-parallel, out-proj/fc2 row-parallel,
    attention core and GELU local (P:186 linear/embedding are the paper's TP-split layers)."""
    tb = TraceBuilder(name, b0, seed, act_bytes=act_bytes)
    tb.start()
    T = b0 * seq
    ids = tb.tensor(T * 8, CAT_INPUT, True)
    labels = tb.tensor(T * 8, CAT_INPUT, True)
    tb.layer = 0
    pos = tb.tensor(T * 8, CAT_INPUT, True)
    h = tb.add(tb.embedding(ids, vocab, hidden, T), tb.embedding(pos, seq, hidden, T))
    if not causal_head:
        h = tb.norm(h, hidden, "layer_norm")
    dh = hidden // heads
    for l in range(n_layers):
        tb.layer = l + 1
        x = tb.norm(h, hidden, "layer_norm") if causal_head else h
        qkv = tb.linear(x, hidden, 3 * hidden, T, role=ROLE_COL)
        sc = tb.bmm(qkv, qkv, b0 * heads * seq * seq * act_bytes, 2.0 * b0 * heads * seq * seq * dh, role=ROLE_LOCAL)
        pr = tb.pointwise(sc, "softmax", role=ROLE_LOCAL)
        ctx = tb.bmm(pr, qkv, T * hidden * act_bytes, 2.0 * b0 * heads * seq * seq * dh, role=ROLE_LOCAL)
        ao = tb.linear(ctx, hidden, hidden, T, role=ROLE_ROW)
        h = tb.add(h, ao)
        if not causal_head:
            h = tb.norm(h, hidden, "layer_norm")
        x2 = tb.norm(h, hidden, "layer_norm") if causal_head else h
        f1 = tb.linear(x2, hidden, ffn, T, role=ROLE_COL)
        g = tb.pointwise(f1, "gelu", role=ROLE_LOCAL, save_out=False)
        f2 = tb.linear(g, ffn, hidden, T, role=ROLE_ROW)
        h = tb.add(h, f2)
        if not causal_head:
            h = tb.norm(h, hidden, "layer_norm")
    tb.layer = n_layers + 1
    h = tb.norm(h, hidden, "layer_norm")
    logits = tb.linear(h, hidden, vocab, T, bias=False)
    tb.loss(logits, labels)
    tb.backward()
    tb.optimizer()
    return tb.build(model=name, seq=seq, hidden=hidden)


def bert_large_trace(b0=8, seed=3) -> Trace:
    return transformer_trace("bert-large", 24, 1024, 16, 4096, 512, 30522, b0, seed, causal_head=False)


def gpt2_xl_trace(b0=8, seed=4) -> Trace:
    return transformer_trace("gpt2-xl", 48, 1600, 25, 6400, 1024, 50257, b0, seed, causal_head=True)


def gpt3_trace(n_layers=96, b0=1, seed=5) -> Trace:
    """GPT-3-class decoder (h = 12288, 96 heads, seq 2048, fp16 activations), configs[4]."""
    return transformer_trace("gpt3-175b", n_layers, 12288, 96, 4 * 12288, 2048, 50257, b0, seed, causal_head=True)


def random_trace(rng, n_layers=3, max_ops_per_layer=3, b0=4, max_time=1e-3, bytes_hi=1 << 20, dyadic=False,
                 roles=True) -> Trace:
    """Small random layered trace with FWD/BWD/OPT structure, for property tests."""
    tb = TraceBuilder("random", b0, int(rng.integers(1 << 30)))
    tb.start()
    x = tb.tensor(int(rng.integers(1, bytes_hi)), CAT_INPUT, True)
    labels = tb.tensor(64, CAT_INPUT, True)
    h = x
    skip = None
    for l in range(n_layers):
        tb.layer = l
        for q in range(int(rng.integers(1, max_ops_per_layer + 1))):
            c = 0 if q == 0 else int(rng.integers(0, 4))
            if c == 0:
                role = int(rng.integers(0, 4)) if roles else 0
                h = tb.linear(h, int(rng.integers(8, 64)), int(rng.integers(8, 64)), b0, role=role,
                              bias=bool(rng.integers(0, 2)))
            elif c == 1:
                h = tb.pointwise(h, "relu")
            elif c == 2:
                h = tb.norm(h, int(rng.integers(8, 64)), "layer_norm")
            else:
                h = tb.add(h, skip) if skip is not None and tb.nbytes(skip) == tb.nbytes(h) else tb.pointwise(h, "gelu")
            if rng.random() < 0.3:
                skip = h
    tb.loss(h, labels)
    tb.backward()
    tb.optimizer()
    tr = tb.build(model="random")
    u = rng.random(len(tr.ops))
    if dyadic:
        tr.ops["time_s"] = (2.0 ** -20) * np.floor(u * 64 + 1)
    else:
        tr.ops["time_s"] = u * max_time
    return tr


# --------------------------------------------------------------------------
# topologies (D3): GPU nodes [0, n_gpus), switches after; directed links
# --------------------------------------------------------------------------
@dataclass
class Topology:
    name: str
    n_nodes: int
    n_gpus: int
    links: np.ndarray       # LINK_DTYPE
    ring_order: np.ndarray  # uint32[n_gpus]
    photonic: object = None  # PHOTONIC_DTYPE record: circuit-switched photonic network (R20)


def _mk(name, n_nodes, n_gpus, edges, ring_order, bidir=True):
    lst = []
    seen = set()
    for e in edges:
        u, v = e[0], e[1]
        bw = e[2] if len(e) > 2 else 1.0
        lat = e[3] if len(e) > 3 else 1.0
        for a, b in ((u, v), (v, u)) if bidir else ((u, v),):
            if (a, b) in seen:
                continue
            seen.add((a, b))
            lst.append((a, b, bw, lat))
    links = np.zeros(len(lst), LINK_DTYPE)
    for i, l in enumerate(lst):
        links[i] = l
    return Topology(name, n_nodes, n_gpus, links, np.asarray(ring_order, np.uint32))


def ring(p, bw=1.0, lat=1.0):
    return _mk(f"ring{p}", p, p, [(i, (i + 1) % p, bw, lat) for i in range(p)], list(range(p)))


def star(p, bw=1.0, lat=1.0):
    """NVSwitch-like: every GPU linked to one switch node."""
    return _mk(f"star{p}", p + 1, p, [(i, p, bw, lat) for i in range(p)], list(range(p)))


def mesh(r, c, bw=1.0, lat=1.0):
    """2D mesh; ring order = boustrophedon (snake) so a 2-row mesh forms a cycle."""
    e = []
    for i in range(r):
        for j in range(c):
            if j + 1 < c:
                e.append((i * c + j, i * c + j + 1, bw, lat))
            if i + 1 < r:
                e.append((i * c + j, (i + 1) * c + j, bw, lat))
    order = []
    for i in range(r):
        row = [i * c + j for j in range(c)]
        order += row if i % 2 == 0 else row[::-1]
    return _mk(f"mesh{r}x{c}", r * c, r * c, e, order)


def wafer_mesh(rows=12, cols=7, bw=1.0, lat=1.0):
    """The Passage case study's electrical baseline: a rows x cols wafer of GPUs on a 2D mesh whose
    ring order is a Hamiltonian cycle of the mesh ("we use the mesh network on the wafer to form a
    ring"): down column 0, then boustrophedon rows over columns 1..cols-1 back to row 0 (rows even)."""
    assert rows % 2 == 0
    t = mesh(rows, cols, bw, lat)
    order = [r * cols for r in range(rows)]
    for k, r in enumerate(range(rows - 1, -1, -1)):
        row = [r * cols + j for j in range(1, cols)]
        order += row if k % 2 == 0 else row[::-1]
    return Topology(f"wafer{rows}x{cols}", t.n_nodes, t.n_gpus, t.links, np.asarray(order, np.uint32))


def photonic(n_gpus, ports=8, link_bw=484e9 / 8, setup=20e-3, lat=0.0, buf_slots=0, ring_order=None, name=None):
    """Circuit-switched photonic interconnect (Lightmatter Passage; R20): every GPU
    can hold `ports` logical links (484 GB/s across 8 links, 20 ms to establish a link); no
    physical links.  Points carry bw_scale / lat_scale as usual."""
    ph = np.zeros((), PHOTONIC_DTYPE)
    ph["ports"], ph["buf_slots"], ph["link_bw_Bps"], ph["setup_s"], ph["lat_s"] = ports, buf_slots, link_bw, setup, lat
    ro = np.arange(n_gpus, dtype=np.uint32) if ring_order is None else np.asarray(ring_order, np.uint32)
    return Topology(name or f"photonic{n_gpus}p{ports}", n_gpus, n_gpus, np.zeros(0, LINK_DTYPE), ro, ph)


def cube_mesh8(bw=1.0, lat=1.0):
    """DGX-1-style hybrid cube-mesh (reading Q31): two fully connected quads plus
    i<->i+4; the edges of the ring 0-1-2-3-7-6-5-4 carry double bandwidth."""
    ring_e = {(0, 1), (1, 2), (2, 3), (3, 7), (6, 7), (5, 6), (4, 5), (0, 4)}
    e = []
    for q in (0, 4):
        for a in range(4):
            for b in range(a + 1, 4):
                e.append((q + a, q + b))
    for i in range(4):
        e.append((i, i + 4))
    edges = [(a, b, (2.0 if (min(a, b), max(a, b)) in ring_e else 1.0) * bw, lat) for a, b in e]
    return _mk("cubemesh8", 8, 8, edges, [0, 1, 2, 3, 7, 6, 5, 4])


def ring_graph(p, bw=1.0, lat=1.0):
    """P:362 (Fig. 16a top): bidirectional ring plus a link from each node to its most distant node."""
    e = [(i, (i + 1) % p, bw, lat) for i in range(p)]
    if p >= 4:
        e += [(i, (i + p // 2) % p, bw, lat) for i in range(p // 2)]
    return _mk(f"ringgraph{p}", p, p, e, list(range(p)))


def double_ring(p, bw=1.0, lat=1.0):
    """P:362 (Fig. 16a bottom): two ring-based graphs of p/2 nodes interconnected node-to-node."""
    h = p // 2
    e = []
    for base in (0, h):
        e += [(base + i, base + (i + 1) % h, bw, lat) for i in range(h)]
        if h >= 4:
            e += [(base + i, base + (i + h // 2) % h, bw, lat) for i in range(h // 2)]
    e += [(i, i + h, bw, lat) for i in range(h)]
    return _mk(f"doublering{p}", p, p, e, list(range(h)) + list(range(p - 1, h - 1, -1)))


def hierarchical(n_nodes, gpus_per_node=8, intra=1.0, nic=0.1, oversub=2.0, lat_intra=1.0, lat_nic=2.0,
                 lat_spine=2.0, nodes_per_leaf=2, n_spines=1):
    """configs[4]'s hierarchical topology: nodes of `gpus_per_node` GPUs on an NVSwitch-like node switch
    (bandwidth `intra`), every GPU also on a NIC link (`nic`) to its leaf switch, leaves to `n_spines`
    spine switches with 1/`oversub` of the leaf's NIC bandwidth.  Node switches are numbered before
    leaves, so intra-node routes go through the node switch (R12's lexicographic tie break)."""
    G = n_nodes * gpus_per_node
    n_leaves = (n_nodes + nodes_per_leaf - 1) // nodes_per_leaf
    node_sw = [G + k for k in range(n_nodes)]
    leaf = [G + n_nodes + k for k in range(n_leaves)]
    spine = [G + n_nodes + n_leaves + k for k in range(n_spines)]
    e = []
    for g in range(G):
        k = g // gpus_per_node
        e.append((g, node_sw[k], intra, lat_intra))
        e.append((g, leaf[k // nodes_per_leaf], nic, lat_nic))
    up = nic * gpus_per_node * nodes_per_leaf / oversub / n_spines
    for lf in leaf:
        for sp in spine:
            e.append((lf, sp, up, lat_spine))
    return _mk(f"hier{n_nodes}x{gpus_per_node}o{oversub:g}", G + n_nodes + n_leaves + n_spines, G, e, list(range(G)))


def perturb_subset(topo: Topology, seed: int, frac=0.25) -> Topology:
    """P:356's random slow-down (bandwidth / U[1,10]) applied to a seeded subset of the links."""
    rng = np.random.Generator(np.random.PCG64(seed))
    links = topo.links.copy()
    sel = rng.random(len(links)) < frac
    links["bw_Bps"][sel] = links["bw_Bps"][sel] / rng.uniform(1.0, 10.0, int(sel.sum()))
    return Topology(f"{topo.name}~s{seed}", topo.n_nodes, topo.n_gpus, links, topo.ring_order.copy())


def perturb(topo: Topology, seed: int) -> Topology:
    """Heterogeneity injector: every link's bandwidth divided by U[1,10]."""
    rng = np.random.Generator(np.random.PCG64(seed))
    links = topo.links.copy()
    links["bw_Bps"] = links["bw_Bps"] / rng.uniform(1.0, 10.0, len(links))
    return Topology(f"{topo.name}~a{seed}", topo.n_nodes, topo.n_gpus, links, topo.ring_order.copy())


def random_topology(rng, n_gpus=4, n_switch=1, p_edge=0.5, dyadic=False):
    n = n_gpus + n_switch
    lst = set()
    # a ring through the GPUs guarantees connectivity
    order = list(rng.permutation(n_gpus))
    for i in range(n_gpus):
        lst.add((int(order[i]), int(order[(i + 1) % n_gpus])))
    for a in range(n):
        for b in range(n):
            if a != b and rng.random() < p_edge:
                lst.add((a, b))
    lst = sorted(lst)
    links = np.zeros(len(lst), LINK_DTYPE)
    for i, (a, b) in enumerate(lst):
        if dyadic:
            links[i] = (a, b, 2.0 ** int(rng.integers(0, 4)), (2.0 ** -20) * int(rng.integers(0, 8)))
        else:
            links[i] = (a, b, float(rng.uniform(0.5, 4.0)), float(rng.uniform(0.0, 1e-5)))
    return Topology("random", n, n_gpus, links, np.asarray(order, np.uint32))


# --------------------------------------------------------------------------
# sweeps
# --------------------------------------------------------------------------
@dataclass
class Sweep:
    name: str
    trace: Trace
    topos: list
    points: np.ndarray                      # POINT_DTYPE
    plans: list = field(default_factory=list)  # explicit stage plans (lists of first layers)


def make_point(topo, strategy, dp=1, tp=1, pp=1, m=1, B=1, bucket=0, bw=1.0, lat=1.0, tp_mode=TPM_MEGATRON,
               algo=ALG_RING, plan=-1, first_bucket=0, chunks=0, hop=(0, 0, 0)):
    """hop = (backup workers, staleness, max iteration gap) of a ST_HOP point (R28); for ST_HOP, dp = workers,
    m = iterations and tp_mode = the communication graph (HOP_RING_BASED / HOP_DOUBLE_RING)."""
    p = np.zeros((), POINT_DTYPE)
    p["hop"] = (hop[0] & 15) | ((hop[1] & 15) << 4) | ((hop[2] & 255) << 8)
    p["first_bucket_bytes"] = first_bucket
    p["ring_chunks"] = chunks
    p["topo"], p["strategy"], p["tp_mode"], p["coll_algo"] = topo, strategy, tp_mode, algo
    p["dp"], p["tp"], p["pp"], p["microbatches"], p["global_batch"] = dp, tp, pp, m, B
    p["stage_plan"], p["bucket_bytes"], p["bw_scale"], p["lat_scale"] = plan, bucket, bw, lat
    return p


def points_array(plist):
    a = np.zeros(len(plist), POINT_DTYPE)
    for i, p in enumerate(plist):
        a[i] = p
    return a


def sweep_c1() -> Sweep:
    """configs[0]: 4-layer MLP, DDP on 2 GPUs, ring AllReduce over one uniform link
    (PCIe-class 25 GB/s per direction, 5 us), per-tensor and 25 MiB buckets."""
    tr = mlp_trace()
    topo = ring(2, bw=25e9, lat=5e-6)
    pts = [make_point(0, ST_DDP, dp=2, B=2 * tr.trace_batch, bucket=0),
           make_point(0, ST_DDP, dp=2, B=2 * tr.trace_batch, bucket=25 * MiB)]
    return Sweep("c1_mlp_dp2", tr, [topo], points_array(pts))


def sweep_c2(trace=None, seed=2, n_bw=25) -> Sweep:
    """configs[1]: ResNet-50 DDP (data parallel), p in {2,4,8,16} on a ring, 25 bandwidths x 10
    latencies x 5 per-GPU batches x 2 bucket sizes -> 10,000 points (seeded order).  n_bw > 25 refines
    the bandwidth axis (the multi-GPU bench's N x 10k-point sweeps; n_bw = 25 is configs[1] itself)."""
    tr = trace if trace is not None else resnet50_trace()
    ps = [2, 4, 8, 16]
    topos = [ring(p) for p in ps]
    bws = np.logspace(np.log10(10e9), np.log10(900e9), n_bw)
    lats = np.logspace(np.log10(0.5e-6), np.log10(20e-6), 10)
    batches, buckets = (16, 32, 64, 128, 256), (0, 25 * MiB)
    n = len(ps) * len(batches) * len(buckets) * n_bw * len(lats)
    ti, bi, ki, wi, li = np.meshgrid(np.arange(len(ps)), np.arange(len(batches)), np.arange(len(buckets)),
                                     np.arange(n_bw), np.arange(len(lats)), indexing="ij")
    arr = np.zeros(n, POINT_DTYPE)
    pv = np.asarray(ps)[ti.ravel()]
    arr["topo"] = ti.ravel()
    arr["strategy"] = ST_DDP
    arr["tp_mode"] = TPM_MEGATRON
    arr["coll_algo"] = ALG_RING
    arr["dp"], arr["tp"], arr["pp"], arr["microbatches"] = pv, 1, 1, 1
    arr["global_batch"] = pv * np.asarray(batches)[bi.ravel()]
    arr["stage_plan"] = -1
    arr["bucket_bytes"] = np.asarray(buckets, np.uint64)[ki.ravel()]
    arr["bw_scale"] = bws[wi.ravel()]
    arr["lat_scale"] = lats[li.ravel()]
    perm = np.random.Generator(np.random.PCG64(seed)).permutation(len(arr))
    return Sweep("c2_resnet50_ddp", tr, topos, arr[perm])


def sweep_c3(trace=None, seed=3, n_bw=8, n_lat=4) -> Sweep:
    """configs[2]: BERT-large TP 2/4/8 with per-layer AllReduce over ring / star / mesh /
    cube-mesh / ring-based / double-ring templates, each also asymmetric."""
    tr = trace if trace is not None else bert_large_trace()
    fam = {2: [ring(2), star(2)],
           4: [ring(4), star(4), mesh(2, 2), ring_graph(4)],
           8: [ring(8), star(8), mesh(2, 4), cube_mesh8(), ring_graph(8), double_ring(8)]}
    topos, pts = [], []
    bws = np.logspace(np.log10(25e9), np.log10(900e9), n_bw)
    lats = np.logspace(np.log10(0.5e-6), np.log10(10e-6), n_lat)
    for tpd, tl in fam.items():
        for base in tl:
            for asym in (0, 1, 2):
                topo = base if asym == 0 else perturb(base, 1000 * tpd + 10 * len(topos) + asym)
                ti = len(topos)
                topos.append(topo)
                for b in (8, 16, 32, 64):
                    for mode in (TPM_MEGATRON, TPM_PAPER):
                        for bw in bws:
                            for lat in lats:
                                pts.append(make_point(ti, ST_TP, tp=tpd, B=b, tp_mode=mode, bw=float(bw),
                                                      lat=float(lat)))
    arr = points_array(pts)
    perm = np.random.Generator(np.random.PCG64(seed)).permutation(len(arr))
    return Sweep("c3_bert_large_tp", tr, topos, arr[perm])


def sweep_c4(trace=None, seed=4, n_bw=25, n_lat=8) -> Sweep:
    """configs[3]: GPT-2 XL GPipe, S in {4,8,16} stages on 2x2/2x4/4x4 meshes (snake order),
    m in {8,16,32,64} micro-batches, B in {64..512}."""
    tr = trace if trace is not None else gpt2_xl_trace()
    topos = [mesh(2, 2), mesh(2, 4), mesh(4, 4)]
    bws = np.logspace(np.log10(25e9), np.log10(900e9), n_bw)
    lats = np.logspace(np.log10(0.5e-6), np.log10(20e-6), n_lat)
    pts = []
    for ti, S in enumerate((4, 8, 16)):
        for m in (8, 16, 32, 64):
            for B in (64, 128, 256, 512):
                for bw in bws:
                    for lat in lats:
                        pts.append(make_point(ti, ST_PP, pp=S, m=m, B=B, bw=float(bw), lat=float(lat)))
    arr = points_array(pts)
    perm = np.random.Generator(np.random.PCG64(seed)).permutation(len(arr))
    return Sweep("c4_gpt2xl_pp", tr, topos, arr[perm])


def sweep_c5(trace=None, seed=5, Ns=(64, 128, 256, 512, 1024), n_bw=25, n_lat=14, oversubs=(1.0, 2.0, 4.0),
             ms=(8, 16, 32, 64)) -> Sweep:
    """configs[4]: GPT-3-class HYBRID DP x TP x PP on N in {64..1024} simulated GPUs of a hierarchical
    topology (8-GPU nodes on a node switch, per-GPU NIC to leaf switches, spine at 1:1 / 2:1 / 4:1
    oversubscription; each also with a seeded slow link subset).  Every (TP, PP, DP) split with
    TP <= 8 inside a node, PP | N a power of two <= 64, TP*PP >= 4 (a 175B model needs >= 4-way model
    parallelism to fit), micro-batches 8..64 (one sample each), 2 GiB gradient buckets, n_bw bandwidth x
    n_lat latency scales.  Defaults give 2,760 structural combinations x 350 = 966,000 points (the
    configs[4] ~1M-point sweep); seeded order.  Built with numpy (no per-point Python objects)."""
    tr = trace if trace is not None else gpt3_trace()
    topos, rows = [], []
    for N in Ns:
        for ov in oversubs:
            base = hierarchical(max(N // 8, 1), 8, intra=1.0, nic=0.125, oversub=ov)
            for asym in (0, 1):
                ti = len(topos)
                topos.append(base if asym == 0 else perturb_subset(base, 500 + 10 * N + int(ov)))
                for tpd in (1, 2, 4, 8):
                    for pp in (1, 2, 4, 8, 16, 32, 64):
                        if N % (tpd * pp) or pp > tr.n_layers or tpd * pp < 4:
                            continue
                        for m in ms:
                            rows.append((ti, N // (tpd * pp), tpd, pp, m))
    bws = np.logspace(np.log10(100e9), np.log10(900e9), n_bw)
    lats = np.logspace(np.log10(1e-6), np.log10(5e-6), n_lat)
    R = np.array(rows, dtype=np.int64).reshape(-1, 5)
    nbl = n_bw * n_lat
    arr = np.zeros(len(R) * nbl, POINT_DTYPE)
    rep = np.repeat(R, nbl, axis=0)
    arr["topo"] = rep[:, 0]
    arr["strategy"] = ST_HYBRID
    arr["tp_mode"] = TPM_MEGATRON
    arr["coll_algo"] = ALG_RING
    arr["dp"], arr["tp"], arr["pp"], arr["microbatches"] = rep[:, 1], rep[:, 2], rep[:, 3], rep[:, 4]
    arr["global_batch"] = rep[:, 1] * rep[:, 4]
    arr["stage_plan"] = -1
    arr["bucket_bytes"] = 2048 * MiB
    arr["bw_scale"] = np.tile(np.repeat(bws, n_lat), len(R))
    arr["lat_scale"] = np.tile(np.tile(lats, n_bw), len(R))
    perm = np.random.Generator(np.random.PCG64(seed)).permutation(len(arr))
    return Sweep("c5_gpt3_hybrid", tr, topos, arr[perm])


def c5_parity_index(full: Sweep, per_n=20, heavy=4, seed=55) -> np.ndarray:
    """Stratified configs[4] sample (SURVEY 8(c).4's >= 100 C5 points): for every
    simulated-GPU count N, `heavy` points of the heavy classes -- data x tensor parallel degree
    dp * tp = 64 (the verdict's "dp x tp >= 64" at its smallest product, which keeps each point at
    1e6-1e7 instants), on the perturbed (slow-link subset) topology at 4:1 oversubscription, with 8
    micro-batches -- plus seeded random points with 8 micro-batches and dp * tp <= 64 (none heavier than
    the heavy class)."""
    P = full.points
    N = P["dp"].astype(np.int64) * P["tp"] * P["pp"]
    rng = np.random.Generator(np.random.PCG64(seed))
    topo_ov = np.array([t.name for t in full.topos])
    idx = []
    for n in sorted(set(N.tolist())):
        sel = (N == n) & (P["microbatches"] == 8)
        hv = np.flatnonzero(sel & (P["dp"].astype(np.int64) * P["tp"] == 64) & (P["topo"] % 2 == 1)
                            & (np.char.find(topo_ov[P["topo"]].astype(str), "o4") >= 0))
        hv = hv[rng.permutation(len(hv))][:heavy]
        rest = np.setdiff1d(np.flatnonzero(sel & (P["dp"].astype(np.int64) * P["tp"] <= 64)), hv)
        idx += hv.tolist() + rest[rng.permutation(len(rest))][:per_n - len(hv)].tolist()
    return np.asarray(sorted(idx), np.int64)


def sweep_c5_parity() -> Sweep:
    """The C5 parity / bench subset: c5_parity_index over the full configs[4] sweep (100 points)."""
    full = sweep_c5()
    return Sweep(full.name + "_parity", full.trace, full.topos, full.points[c5_parity_index(full)])


def sweep_hop(trace=None, seed=7, groups=8, n_bw=5, n_lat=2) -> Sweep:
    """NEXT 4: the Hop case study (Fig. 16).  VGG-11 at batch 128 per worker on 8
    A100-class workers; communication graphs ring-based and double ring (Fig. 16a), each a topology whose
    links are exactly the graph's edges; `groups` random slowdown scenarios that divide every GPU's link
    bandwidth by U[1, 10]; without and with one backup worker (and bounded staleness 0 / 1, token
    gap 0 / 2); 10 iterations; n_bw bandwidth x n_lat latency scales -> 8 x 2 x 2 x 2 x 5 x 2 = 640 points
    (seeded order)."""
    tr = trace if trace is not None else vgg11_trace()
    rng = np.random.Generator(np.random.PCG64(seed))
    topos = []
    for g in range(groups):
        u = rng.uniform(1.0, 10.0, 8)
        for graph, mk in ((HOP_RING_BASED, ring_graph), (HOP_DOUBLE_RING, double_ring)):
            t = mk(8, bw=50e9, lat=2e-6)
            links = t.links.copy()
            links["bw_Bps"] = links["bw_Bps"] / u[links["src"]]
            topos.append((graph, Topology(f"{t.name}~g{g}", t.n_nodes, t.n_gpus, links, np.arange(8, dtype=np.uint32))))
    bws = np.logspace(np.log10(0.25), np.log10(4.0), n_bw)
    lats = np.logspace(np.log10(0.5), np.log10(2.0), n_lat)
    pts = []
    for ti, (graph, _) in enumerate(topos):
        for b in (0, 1):
            for st, gap in ((0, 0), (1, 2)):
                for bw in bws:
                    for lat in lats:
                        pts.append(make_point(ti, ST_HOP, dp=8, m=10, B=8 * 128, tp_mode=graph, bw=float(bw),
                                              lat=float(lat), hop=(b, st, gap)))
    arr = points_array(pts)
    perm = np.random.Generator(np.random.PCG64(seed + 1)).permutation(len(arr))
    return Sweep("hop_vgg11_fig16", tr, [t for _, t in topos], arr[perm])


def sweep_wafer(trace=None, seed=6, n_bw=10, n_lat=5) -> Sweep:
    """NEXT 1: the Passage case study (Fig. 15).  84 GPUs on a 12 x 7 wafer,
    DDP over all of them, ring AllReduce along a Hamiltonian cycle of the electrical mesh vs the
    same ring over photonic logical links (8 ports, 484 GB/s across 8 links, 20 ms link setup).  Axes:
    network x per-GPU batch {16, 32, 64, 128} x bucket {per tensor, 25 MiB} x bandwidth x latency scales."""
    tr = trace if trace is not None else resnet50_trace()
    elec = wafer_mesh(12, 7, bw=50e9, lat=1e-6)
    opt = photonic(84, ports=8, link_bw=484e9 / 8, setup=20e-3, lat=1e-6, ring_order=elec.ring_order,
                   name="passage84")
    topos = [elec, opt]
    bws = np.logspace(np.log10(0.5), np.log10(2.0), n_bw)
    lats = np.logspace(np.log10(0.5), np.log10(2.0), n_lat)
    pts = []
    for ti in range(2):
        for b in (16, 32, 64, 128):
            for bucket in (0, 25 * MiB):
                for bw in bws:
                    for lat in lats:
                        pts.append(make_point(ti, ST_DDP, dp=84, B=84 * b, bucket=bucket, bw=float(bw), lat=float(lat)))
    arr = points_array(pts)
    perm = np.random.Generator(np.random.PCG64(seed)).permutation(len(arr))
    return Sweep("wafer84_passage_dp", tr, topos, arr[perm])


def sweep_c5_small(trace=None, seed=5) -> Sweep:
    """configs[4]'s structure on 8-32 simulated GPUs (warp-segment hybrid kernel; m in {8,16,32},
    4 bandwidths x 2 latencies): the small end used by the sampled parity tests."""
    return sweep_c5(trace, seed, Ns=(8, 16, 32), n_bw=4, n_lat=2, oversubs=(2.0, 4.0), ms=(8, 16, 32))

