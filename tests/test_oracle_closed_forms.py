"""Pins of the CPU oracle against closed forms the paper and the mathematics fix.

DESIGN.md "Pins" lists each: CF1 identity, CF2 power-of-two batch scaling
(P:178), CF3/CF4 the two cases of Fig. 5, CF5-CF9 ring / star / tree
collective times, CF10-CF11 DataParallel vs DDP overlap (P:176,
P:236), CF12 tensor parallel with blocking collectives, CF13-CF14 the
GPipe bubble formula and the Fig. 4 instance.
"""
import math

import numpy as np
import pytest

import oracle
from paper_conf_isca_libwmvgjbj025_b200 import workloads as W
from tests.helpers import HandGraph, HandTrace, one_wgrad_trace, rel

pytestmark = []


def fold(xs):
    s = 0.0
    for x in xs:
        s = s + x
    return s


# ---------------- CF1 / CF2: operator-time model ----------------
@pytest.mark.parametrize("mk", [W.mlp_trace, W.resnet50_trace])
def test_cf1_identity_single_gpu_trace_batch(mk):
    """same environment as the trace -> the trace time itself; DP on 1 GPU at b0
    takes exactly the left fold of the trace times."""
    tr = mk()
    topo = W.ring(2)
    for st in (W.ST_DP, W.ST_DDP):
        r = oracle.run_point(tr, topo, W.make_point(0, st, dp=1, B=tr.trace_batch))
        assert r["status"] == 0
        assert r["iter_time_s"] == fold(tr.ops["time_s"])
        assert r["compute_busy_max_s"] == r["iter_time_s"]
        assert r["n_collectives"] == 0 and r["n_flows"] == 0 and r["comm_busy_s"] == 0.0
        assert r["n_compute"] == len(tr.ops)


def test_cf2_power_of_two_batch_is_exact():
    """per-GPU batch 4x the trace batch -> batch-scaled ops take exactly 4t."""
    tr = W.resnet50_trace()
    r = oracle.run_point(tr, W.ring(2), W.make_point(0, W.ST_DP, dp=1, B=4 * tr.trace_batch))
    scaled = (tr.ops["flags"] & W.OPF_BATCH_SCALED) != 0
    exp = fold(np.where(scaled, tr.ops["time_s"] * 4.0, tr.ops["time_s"]))
    assert r["iter_time_s"] == exp
    # half batch
    r = oracle.run_point(tr, W.ring(2), W.make_point(0, W.ST_DP, dp=1, B=tr.trace_batch // 2))
    exp = fold(np.where(scaled, tr.ops["time_s"] * 0.5, tr.ops["time_s"]))
    assert r["iter_time_s"] == exp


@pytest.mark.parametrize("k", [-3, 2])
@pytest.mark.parametrize("st", [W.ST_DDP, W.ST_TP, W.ST_PP])
def test_cf2_time_scaling_metamorphic(k, st):
    """Scaling op times and latencies by 2^k and bandwidths by 2^-k scales every output time
    by exactly 2^k (dimensional analysis of the model: bytes fixed)."""
    rng = np.random.Generator(np.random.PCG64(11))
    tr = W.random_trace(rng, n_layers=4)
    topo = W.mesh(2, 2, bw=3e9, lat=1.3e-6)
    pt = {W.ST_DDP: W.make_point(0, st, dp=4, B=8, bucket=1000),
          W.ST_TP: W.make_point(0, st, tp=4, B=4),
          W.ST_PP: W.make_point(0, st, pp=3, m=2, B=8)}[st]
    r0 = oracle.run_point(tr, topo, pt)
    assert r0["status"] == 0
    tr2 = W.Trace(tr.name, tr.ops.copy(), tr.tensors, tr.io, tr.trace_batch, tr.n_layers)
    tr2.ops["time_s"] = tr.ops["time_s"] * 2.0 ** k
    t2 = W.Topology("m", topo.n_nodes, topo.n_gpus, topo.links.copy(), topo.ring_order)
    t2.links["lat_s"] *= 2.0 ** k
    t2.links["bw_Bps"] *= 2.0 ** -k
    if st == W.ST_PP:
        plan = oracle.partition(tr, 3)  # keep the same stages (partition is scale invariant anyway)
        r0 = oracle.run_point(tr, topo, pt, plan)
        r1 = oracle.run_point(tr2, t2, pt, plan)
    else:
        r1 = oracle.run_point(tr2, t2, pt)
    for f in ("iter_time_s", "compute_busy_max_s", "comm_busy_s", "exposed_comm_s"):
        assert r1[f] == r0[f] * 2.0 ** k, f
    for f in ("n_compute", "n_flows", "n_collectives", "n_p2p", "n_instants", "n_wf_calls", "n_wf_rounds",
              "max_active_flows"):
        assert r1[f] == r0[f], f


# ---------------- CF3 / CF4: Fig. 5 ----------------
def test_cf3_fig5_case_a_single_message():
    """Fig. 5 case A: one message alone on the link is delivered at t0 + L + S/B."""
    B, L, S, t0 = 7.5e9, 3e-6, 12345678.0, 1e-3
    g = HandGraph()
    a = g.task(0, t0)
    f = g.flow(0, 1, S, deps=[a])
    r, td = oracle.sim_graph(g.arrays(), W.ring(2, bw=B, lat=L), times=True)
    assert td[f] == (t0 + L) + S / B
    assert r["iter_time_s"] == td[f]
    assert r["n_wf_calls"] == 2 and r["max_active_flows"] == 1  # activation, delivery


def test_cf4_fig5_case_b_two_messages_share_a_link():
    """Fig. 5 case B: orange starts while blue is in transit on the same link; the
    bandwidth is re-allocated; orange arrives at T3 = t_o + L + 2S_o/B and blue's delivery
    moves EARLIER than its tentative T5 to T4 = t_b + L + (S_b + S_o)/B."""
    B, L = 1e9, 1e-6
    t_b, t_o, S_b, S_o = 1e-3, 3e-3, 8e6, 1e6
    g = HandGraph()
    a = g.task(0, t_b)
    blue = g.flow(0, 1, S_b, deps=[a])
    b = g.task(0, t_o - t_b)
    orange = g.flow(0, 1, S_o, deps=[b])
    r, td = oracle.sim_graph(g.arrays(), W.ring(2, bw=B, lat=L), times=True)
    T3 = t_o + L + 2 * S_o / B
    T4 = t_b + L + (S_b + S_o) / B
    rem_b = S_b - B * (t_o - t_b)
    T5 = t_o + L + 2 * rem_b / B
    assert rel(td[orange], T3) < 1e-13
    assert rel(td[blue], T4) < 1e-13
    assert td[blue] < T5
    assert td[orange] < td[blue]
    assert r["max_active_flows"] == 2


# ---------------- CF5 - CF9: collectives ----------------
def _dp_point(p, S, algo=W.ALG_RING, strategy=W.ST_DP):
    return one_wgrad_trace(S), W.make_point(0, strategy, dp=p, B=p, algo=algo)


@pytest.mark.parametrize("p", [2, 3, 4, 8, 16])
def test_cf5_ring_allreduce_uniform(p):
    """Ring AllReduce: 2(p-1) steps of S/p over one link each: 2(p-1)(a + S/(pB))."""
    S, B, a = 100e6, 50e9, 2e-6
    tr, pt = _dp_point(p, int(S))
    r = oracle.run_point(tr, W.ring(p, bw=B, lat=a), pt)
    t_fb = 2.0 ** -10 + 2.0 ** -9
    exp = t_fb + 2 * (p - 1) * (a + S / (p * B))
    assert r["status"] == 0
    assert rel(r["iter_time_s"], exp) < 1e-12
    assert r["n_flows"] == 2 * (p - 1) * p and r["n_collectives"] == 1
    assert r["coll_payload_bytes"] == S


@pytest.mark.parametrize("seed", range(8))
def test_cf6_ring_allreduce_heterogeneous_links(seed):
    """'one link is slower than other links': the ring runs at its slowest hop,
    2(p-1) max_i(a_i + S/(p B_i))."""
    rng = np.random.Generator(np.random.PCG64(seed))
    p = int(rng.integers(2, 9))
    S = 64e6
    topo = W.ring(p)
    topo.links["bw_Bps"] = rng.uniform(5e9, 100e9, len(topo.links))
    topo.links["lat_s"] = rng.uniform(0.0, 2e-4, len(topo.links))
    tr, pt = _dp_point(p, int(S))
    r = oracle.run_point(tr, topo, pt)
    worst = 0.0
    for l in topo.links:
        if (int(l["src"]) + 1) % p == int(l["dst"]):
            worst = max(worst, l["lat_s"] + S / (p * l["bw_Bps"]))
    exp = 2.0 ** -10 + 2.0 ** -9 + 2 * (p - 1) * worst
    assert rel(r["iter_time_s"], exp) < 1e-12


@pytest.mark.parametrize("p", [2, 4, 5, 8])
def test_cf7_ring_allreduce_through_switch(p):
    """NVSwitch-like star: every flow crosses GPU->switch->GPU: 2(p-1)(2a + S/(pB))."""
    S, B, a = 32e6, 100e9, 1e-6
    tr, pt = _dp_point(p, int(S))
    r = oracle.run_point(tr, W.star(p, bw=B, lat=a), pt)
    exp = 2.0 ** -10 + 2.0 ** -9 + 2 * (p - 1) * (2 * a + S / (p * B))
    assert rel(r["iter_time_s"], exp) < 1e-12


@pytest.mark.parametrize("p", [2, 4, 8])
def test_cf8_ring_allgather(p):
    """Ring AllGather of a tensor-parallel layer's output: (p-1)(a + S/(pB))."""
    S, B, a = 16e6, 25e9, 4e-6
    h = HandTrace(b0=1)
    x = h.tensor(64, W.CAT_INPUT)
    y = h.tensor(int(S))
    h.op(0, W.PH_FWD, [x], [y], 2.0 ** -8, role=W.ROLE_GATHER)
    tr = h.build()
    r = oracle.run_point(tr, W.ring(p, bw=B, lat=a), W.make_point(0, W.ST_TP, tp=p, B=1, tp_mode=W.TPM_PAPER))
    exp = 2.0 ** -8 / p + (p - 1) * (a + S / (p * B))
    assert r["n_collectives"] == 1 and r["n_flows"] == (p - 1) * p
    assert rel(r["iter_time_s"], exp) < 1e-12


@pytest.mark.parametrize("k", [2, 3, 4])
def test_cf9_tree_allreduce_on_star(k):
    """Binary-tree AllReduce (extension, reading Q25) through a switch, p = 2^k - 1:
    (k-1) reduce + (k-1) broadcast levels, two flows share a switch port: 4(k-1)(a + S/B)."""
    p = 2 ** k - 1
    S, B, a = 8e6, 40e9, 3e-6
    tr, pt = _dp_point(p, int(S), algo=W.ALG_TREE)
    r = oracle.run_point(tr, W.star(p, bw=B, lat=a), pt)
    exp = 2.0 ** -10 + 2.0 ** -9 + 4 * (k - 1) * (a + S / B)
    assert r["n_flows"] == 2 * (p - 1)
    assert rel(r["iter_time_s"], exp) < 1e-12


# ---------------- CF10 / CF11: DataParallel vs DDP ----------------
def _mlp_parts(tr):
    ph = tr.ops["phase"]
    return tr.ops["time_s"][ph != W.PH_OPT], tr.ops["time_s"][ph == W.PH_OPT]


@pytest.mark.parametrize("p", [2, 4])
def test_cf10_dataparallel_after_backward(p):
    """Standard DataParallel: all gradient AllReduces after the backward pass, in
    FIFO: T = sum t'(fwd,bwd) + sum_c 2(p-1)(a + S_c/(pB)) + sum t'(opt)."""
    tr = W.mlp_trace()
    B, a = 25e9, 5e-6
    r = oracle.run_point(tr, W.ring(p, bw=B, lat=a), W.make_point(0, W.ST_DP, dp=p, B=p * tr.trace_batch))
    fb, opt = _mlp_parts(tr)
    wg = tr.tensors[tr.tensors["category"] == W.CAT_WGRAD]["bytes_b0"].astype(float)
    exp = fold(fb) + sum(2 * (p - 1) * (a + s / (p * B)) for s in wg) + fold(opt)
    assert r["n_collectives"] == len(wg)
    assert rel(r["iter_time_s"], exp) < 1e-12
    assert r["coll_payload_bytes"] == wg.sum()


@pytest.mark.parametrize("bucket", [0, 1 << 30])
@pytest.mark.parametrize("p", [2, 3])
def test_cf11_ddp_overlap_recursion(bucket, p):
    """DDP overlaps each bucket's AllReduce with the rest of the backward:
    c_i = max(g_i, c_{i-1}) + A_i, T = max(g_bwd_end, c_last) + sum t'(opt)."""
    tr = W.mlp_trace()
    B, a = 25e9, 5e-6
    r = oracle.run_point(tr, W.ring(p, bw=B, lat=a),
                         W.make_point(0, W.ST_DDP, dp=p, B=p * tr.trace_batch, bucket=bucket))
    t = tr.ops["time_s"]
    ends = np.cumsum(t)  # dyadic times: exact prefix sums
    cat = tr.tensors["category"]
    prod = {}
    for o, op in enumerate(tr.ops):
        for x in tr.io[op["io_off"] + op["n_in"]: op["io_off"] + op["n_in"] + op["n_out"]]:
            prod[int(x)] = o
    wg = sorted((prod[x], x) for x in range(len(cat)) if cat[x] == W.CAT_WGRAD)
    if bucket == 0:
        buckets = [[w] for w in wg]
    else:
        buckets = [wg]
    c = 0.0
    for bk in buckets:
        S = float(sum(int(tr.tensors["bytes_b0"][x]) for _, x in bk))
        g_i = ends[bk[-1][0]]
        c = max(g_i, c) + 2 * (p - 1) * (a + S / (p * B))
    fb, opt = _mlp_parts(tr)
    exp = max(fold(fb), c) + fold(opt)
    assert rel(r["iter_time_s"], exp) < 1e-12
    assert r["compute_busy_max_s"] == fold(t)


# ---------------- CF12: tensor parallel ----------------
@pytest.mark.parametrize("p", [2, 4])
def test_cf12_tp_blocking_collectives(p):
    """Megatron TP: a row-parallel FWD op's output and a column-parallel BWD
    op's input-gradient are all-reduced and read by the very next op, which therefore waits:
    T = sum t' + sum_c AR_c."""
    B, a = 50e9, 1e-6
    S1, S2 = 4e6, 6e6
    h = HandTrace(b0=1)
    x = h.tensor(64, W.CAT_INPUT)
    y1 = h.tensor(int(S1))
    y2 = h.tensor(64)
    h.op(0, W.PH_FWD, [x], [y1], 2.0 ** -7, role=W.ROLE_ROW)
    h.op(0, W.PH_FWD, [y1], [y2], 2.0 ** -8)
    g1 = h.tensor(int(S2), W.CAT_AGRAD)
    h.op(0, W.PH_BWD, [y2], [g1], 2.0 ** -6, role=W.ROLE_COL)
    g0 = h.tensor(64, W.CAT_AGRAD)
    h.op(0, W.PH_BWD, [g1], [g0], 2.0 ** -9)
    tr = h.build()
    r = oracle.run_point(tr, W.ring(p, bw=B, lat=a), W.make_point(0, W.ST_TP, tp=p, B=1))
    AR = lambda S: 2 * (p - 1) * (a + S / (p * B))
    exp = 2.0 ** -7 / p + AR(S1) + 2.0 ** -8 + 2.0 ** -6 / p + AR(S2) + 2.0 ** -9
    assert r["n_collectives"] == 2
    assert rel(r["iter_time_s"], exp) < 1e-12


# ---------------- CF13 / CF14: GPipe ----------------
def gpipe_trace(S, t_f, t_b, t_opt, A):
    """S single-op layers (one per stage); activation / gradient of A bytes between layers."""
    h = HandTrace(b0=1)
    x = h.tensor(64, W.CAT_INPUT)
    ws = [h.tensor(1024, W.CAT_WEIGHT, scaled=False) for _ in range(S)]
    hs = []
    prev = x
    for l in range(S):
        out = h.tensor(A if l < S - 1 else 4, W.CAT_ACT if l < S - 1 else W.CAT_OTHER, scaled=l < S - 1)
        h.op(l, W.PH_FWD, [prev, ws[l]], [out], t_f)
        hs.append(out)
        prev = out
    gs = {}
    dws = {}
    for l in range(S - 1, -1, -1):
        ins = [hs[l] if l == S - 1 else gs[l]] + ([hs[l - 1]] if l > 0 else [x])
        outs = []
        if l > 0:
            gs[l - 1] = h.tensor(A, W.CAT_AGRAD)
            outs.append(gs[l - 1])
        dws[l] = h.tensor(1024, W.CAT_WGRAD, scaled=False)
        outs.append(dws[l])
        h.op(l, W.PH_BWD, ins, outs, t_b)
    for l in range(S):
        w2 = h.tensor(1024, W.CAT_WEIGHT, scaled=False)
        h.op(l, W.PH_OPT, [ws[l], dws[l]], [w2], t_opt, scaled=False)
    return h.build()


@pytest.mark.parametrize("p,m", [(2, 2), (4, 8), (3, 5), (2, 1), (5, 3)])
def test_cf13_gpipe_bubble(p, m):
    """GPipe (Fig. 4): uniform stages, P2P c = a + A/B <= min(t_f, t_b):
    T = (m+p-1)(t_f+t_b) + (p-1)(c_f+c_b) + t_opt."""
    t_f, t_b, t_opt = 2.0 ** -10, 2.0 ** -9, 2.0 ** -12
    A, B, a = 2 ** 20, 2.0 ** 32, 2.0 ** -16
    tr = gpipe_trace(p, t_f, t_b, t_opt, A)
    r = oracle.run_point(tr, W.ring(p, bw=B, lat=a), W.make_point(0, W.ST_PP, pp=p, m=m, B=m))
    c = a + A / B
    exp = (m + p - 1) * (t_f + t_b) + (p - 1) * (c + c) + t_opt
    assert r["status"] == 0
    assert r["n_p2p"] == 2 * (p - 1) * m
    assert rel(r["iter_time_s"], exp) < 1e-12


def test_cf14_fig4_two_layers_two_gpus_two_microbatches():
    """The Fig. 4 instance: 2 layers on 2 GPUs, 1 mini-batch split into 2
    micro-batches: T = 3(t_f + t_b) + c_f + c_b + t_opt."""
    t_f, t_b, t_opt = 3e-3, 5e-3, 1e-4
    A, B, a = 8e6, 16e9, 2e-6
    tr = gpipe_trace(2, t_f, t_b, t_opt, int(A))
    r = oracle.run_point(tr, W.ring(2, bw=B, lat=a), W.make_point(0, W.ST_PP, pp=2, m=2, B=2))
    c = a + A / B
    assert rel(r["iter_time_s"], 3 * (t_f + t_b) + 2 * c + t_opt) < 1e-12
    assert r["n_compute"] == 2 * (2 * 2 + 1)


def test_cf13_comm_bound_is_not_the_formula():
    """Outside its validity (A/B > t_f) the bubble formula under-predicts."""
    t_f, t_b, t_opt = 2.0 ** -10, 2.0 ** -9, 0.0
    A, B, a = 2 ** 24, 2.0 ** 30, 0.0   # A/B = 1/64 >> t_f
    tr = gpipe_trace(3, t_f, t_b, t_opt, A)
    r = oracle.run_point(tr, W.ring(3, bw=B, lat=a), W.make_point(0, W.ST_PP, pp=3, m=4, B=4))
    c = a + A / B
    assert r["iter_time_s"] > (4 + 2) * (t_f + t_b) + 2 * 2 * c + 1e-9


# ---------------- R24: DDP first-bucket rule ----------------
def _buckets(sizes, first, cap):
    """Plain greedy bucketing of gradient sizes in production order (R24 restated)."""
    out, cur, tot = [], [], 0
    for s in sizes:
        cur.append(s)
        tot += s
        lim = first if (not out and first) else cap
        if tot >= lim:
            out.append(cur)
            cur, tot = [], 0
    if cur:
        out.append(cur)
    return out


def _wgrad_sizes(tr):
    prod = {}
    for o, op in enumerate(tr.ops):
        for k in range(int(op["n_out"])):
            prod[int(tr.io[op["io_off"] + op["n_in"] + k])] = o
    xs = [x for x in range(len(tr.tensors)) if tr.tensors[x]["category"] == W.CAT_WGRAD and x in prod
          and tr.ops[prod[x]]["phase"] != W.PH_OPT]
    xs.sort(key=lambda x: (prod[x], x))
    return [int(tr.tensors[x]["bytes_b0"]) for x in xs]


@pytest.mark.parametrize("first,cap", [(1, 25 << 20), (1 << 20, 25 << 20), (4 << 20, 1 << 20), (1, 1)])
def test_r24_first_bucket_counts_and_payload(first, cap):
    """PyTorch DDP caps the first gradient bucket separately (1 MiB by default, later ones 25 MiB): the
    number of AllReduces is the greedy bucket count with the first cap, and the payload is unchanged."""
    tr = W.resnet50_trace()
    sizes = _wgrad_sizes(tr)
    exp = _buckets(sizes, first, cap)
    r = oracle.run_point(tr, W.ring(4), W.make_point(0, W.ST_DDP, dp=4, B=4 * tr.trace_batch, bucket=cap,
                                                     first_bucket=first))
    assert r["status"] == 0 and r["n_collectives"] == len(exp)
    assert r["coll_payload_bytes"] == float(sum(sizes))
    if first == 1:
        assert len(exp[0]) == 1


@pytest.mark.parametrize("st", [W.ST_DP, W.ST_DDP, W.ST_HYBRID])
def test_r24_first_bucket_equal_to_cap_or_per_tensor_is_the_plain_rule(st):
    """first_bucket_bytes == bucket_bytes, or bucket_bytes == 0 (one tensor per AllReduce), reproduce the
    rule without a first cap bit for bit, order hash included."""
    tr = W.resnet50_trace()
    topo = W.ring(8, 50e9, 2e-6)
    kw = dict(dp=4, B=4 * tr.trace_batch) if st != W.ST_HYBRID else dict(dp=2, tp=2, pp=2, m=2, B=4 * tr.trace_batch)
    for cap, first in ((25 << 20, 25 << 20), (0, 1 << 20)):
        a = oracle.run_point(tr, topo, W.make_point(0, st, bucket=cap, **kw))
        b = oracle.run_point(tr, topo, W.make_point(0, st, bucket=cap, first_bucket=first, **kw))
        assert a.tobytes() == b.tobytes()


def test_r24_small_first_bucket_starts_communication_earlier():
    """A small first bucket launches its AllReduce as soon as its few gradients exist, so on a fast link
    the iteration is not slower and the first collective starts before the 25 MiB-only case's."""
    tr = W.resnet50_trace()
    topo = W.ring(4, 100e9, 1e-6)
    a, ta, fa = oracle.run_point(tr, topo, W.make_point(0, W.ST_DDP, dp=4, B=256, bucket=25 << 20), timeline=True)
    b, tb, fb = oracle.run_point(tr, topo, W.make_point(0, W.ST_DDP, dp=4, B=256, bucket=25 << 20,
                                                        first_bucket=1 << 20), timeline=True)
    assert fb["release_s"].min() < fa["release_s"].min()
    assert b["n_collectives"] >= a["n_collectives"]
