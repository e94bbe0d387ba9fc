"""Absolute pins of the oracle's R19 outputs: order_hash, n_instants, n_wf_calls, n_wf_rounds and
max_active_flows (R19; "it shows the timeline of the communication process among
GPUs or the computation process on each GPU" -- these counters and the hash summarise that timeline).

Each case lists its boundary events BY HAND from the closed-form schedule (Fig. 5 cases A/B, P:214;
ring AllReduce, P:87 / P:192; the Fig. 4 GPipe instance), with dyadic inputs so that
every event time is exact in binary64 whatever order the simulator adds in.  The hash is then
recomputed here from R19's definition alone:

    order_hash = sum over events e of mix64(mix64(bits(t_e)) XOR (kind_e << 60 | code_e))  (mod 2^64)

with mix64 the SplitMix64 finaliser (Steele, Lea & Flood, OOPSLA 2014) and the R19 event kinds
COLL_START 1, RELEASE 2, ACTIVATE 3, DELIVER 4, TASK_START 5, TASK_END 6.  Nothing here calls the
oracle's hash code: a dropped / extra event, a wrong code field, a wrong time or a wrong kind fails.
"""
import struct

import oracle
from paper_conf_isca_libwmvgjbj025_b200 import workloads as W
from tests.helpers import HandGraph, HandTrace, one_wgrad_trace

M64 = (1 << 64) - 1
COLL_START, RELEASE, ACTIVATE, DELIVER, TASK_START, TASK_END = 1, 2, 3, 4, 5, 6


def mix64(z):
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & M64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & M64
    return z ^ (z >> 31)


def bits(t):
    return struct.unpack("<Q", struct.pack("<d", t))[0]


def r19_hash(events):
    """events: iterable of (time, kind, code)."""
    h = 0
    for t, kind, code in events:
        h = (h + mix64(mix64(bits(t)) ^ ((kind << 60) | code))) & M64
    return h


def n_instants(events):
    return len({t for t, _, _ in events})


def task_code(gpu, prog):
    return (gpu << 40) | prog


def coll_flow_code(c, step, member):
    return (c << 32) | (step << 16) | member


def p2p_code(x, j, dst):
    return (1 << 59) | (x << 32) | (j << 16) | dst


def test_sanity_mix64_reference_values():
    # SplitMix64: the generator state advances by 0x9E3779B97F4A7C15 and mix64 is applied to it;
    # the first outputs for seed 0 are published widely (e.g. the xoshiro reference seeding)
    g = 0x9E3779B97F4A7C15
    assert mix64(g) == 0xE220A8397B1DCDAF
    assert mix64((2 * g) & M64) == 0x6E789E6AA1B965F4


def test_cf3_case_a_hash_and_counts():
    """Fig. 5 case A: a task on GPU 0 ends at t0, its message is released, activates after L and
    drains alone at the link bandwidth."""
    B, L, S, t0 = 2.0 ** 30, 2.0 ** -20, 2.0 ** 22, 2.0 ** -10
    g = HandGraph()
    a = g.task(0, t0)
    f = g.flow(0, 1, S, deps=[a])
    r, td = oracle.sim_graph(g.arrays(), W.ring(2, bw=B, lat=L), times=True)
    T1 = t0 + L + S / B
    ev = [(t0, TASK_END, a), (t0, RELEASE, f), (t0 + L, ACTIVATE, f), (T1, DELIVER, f)]
    assert td[f] == T1
    assert r["order_hash"] == r19_hash(ev)
    assert r["n_instants"] == n_instants(ev) == 3
    assert r["n_wf_calls"] == 2 and r["n_wf_rounds"] == 1 and r["max_active_flows"] == 1


def test_cf4_case_b_hash_and_counts():
    """Fig. 5 case B with dyadic sizes: blue (8 MiB) alone, orange (1 MiB) joins at t_o + L, both at
    B/2; orange arrives at T3 = t_o + L + 2 S_o / B, blue at T4 = t_b + L + (S_b + S_o) / B."""
    B, L = 2.0 ** 30, 2.0 ** -20
    t_b, t_o, S_b, S_o = 2.0 ** -10, 3 * 2.0 ** -10, 2.0 ** 23, 2.0 ** 20
    g = HandGraph()
    a = g.task(0, t_b)
    blue = g.flow(0, 1, S_b, deps=[a])
    b = g.task(0, t_o - t_b)
    orange = g.flow(0, 1, S_o, deps=[b])
    r, td = oracle.sim_graph(g.arrays(), W.ring(2, bw=B, lat=L), times=True)
    T3 = t_o + L + 2 * S_o / B
    T4 = t_b + L + (S_b + S_o) / B
    assert td[orange] == T3 and td[blue] == T4
    ev = [(t_b, TASK_END, a), (t_b, RELEASE, blue), (t_b + L, ACTIVATE, blue),
          (t_o, TASK_END, b), (t_o, RELEASE, orange), (t_o + L, ACTIVATE, orange),
          (T3, DELIVER, orange), (T4, DELIVER, blue)]
    assert r["order_hash"] == r19_hash(ev)
    assert r["n_instants"] == n_instants(ev) == 6
    # water-filling at both activations and both deliveries; rounds: 1 (blue alone), 1 (two flows,
    # one shared link, one bottleneck), 1 (blue alone again), 0 (nothing active)
    assert r["n_wf_calls"] == 4 and r["n_wf_rounds"] == 3
    assert r["max_active_flows"] == 2


def test_cf5_ring_p3_hash_and_counts():
    """DataParallel on a uniform 3-GPU ring: at t_fb every rank's backward op ends (it triggers the
    AllReduce), the collective starts and the three step-0 flows are released; each of the 2(p-1) = 4
    steps activates after alpha and drains S/(pB) later, releasing the next step (R10, Q21)."""
    p, K = 3, 4
    S, B, al = 3 * 2 ** 20, 2.0 ** 30, 2.0 ** -20
    t_f, t_b = 2.0 ** -10, 2.0 ** -9
    tr = one_wgrad_trace(S, t_f=t_f, t_b=t_b)
    r = oracle.run_point(tr, W.ring(p, bw=B, lat=al), W.make_point(0, W.ST_DP, dp=p, B=p))
    t0 = t_f + t_b
    x = (S / p) / B   # 2^-10
    ev = [(t0, TASK_END, task_code(g, 1)) for g in range(p)] + [(t0, COLL_START, 0)]
    t = t0
    for k in range(K):
        ev += [(t, RELEASE, coll_flow_code(0, k, i)) for i in range(p)]
        t = t + al
        ev += [(t, ACTIVATE, coll_flow_code(0, k, i)) for i in range(p)]
        t = t + x
        ev += [(t, DELIVER, coll_flow_code(0, k, i)) for i in range(p)]
    assert r["iter_time_s"] == t0 + K * (al + x)
    assert r["order_hash"] == r19_hash(ev)
    assert r["n_instants"] == n_instants(ev) == 1 + 2 * K
    assert r["n_wf_calls"] == 2 * K and r["n_wf_rounds"] == K
    assert r["max_active_flows"] == p
    assert r["n_flows"] == K * p


def test_cf14_gpipe_fig4_hash_and_counts():
    """The Fig. 4 instance with dyadic times: 2 layers on 2 GPUs, 2 micro-batches (R8: FWD j = 0, 1,
    BWD j = 1, 0, OPT once).  Tensor ids of the hand trace: h0 = 3 (layer-0 activation, read by F1
    and B1 on stage 1), g0 = 5 (activation gradient of layer 0, produced by B1, read by B0)."""
    t_f, t_b, t_opt = 2.0 ** -10, 2.0 ** -9, 2.0 ** -12
    A, B, a = 2 ** 20, 2.0 ** 32, 2.0 ** -16
    c = a + A / B
    h = HandTrace(b0=1)
    x = h.tensor(64, W.CAT_INPUT)
    w0, w1 = h.tensor(1024, W.CAT_WEIGHT, scaled=False), h.tensor(1024, W.CAT_WEIGHT, scaled=False)
    h0 = h.tensor(A)
    h1 = h.tensor(4, W.CAT_OTHER)
    h.op(0, W.PH_FWD, [x, w0], [h0], t_f)
    h.op(1, W.PH_FWD, [h0, w1], [h1], t_f)
    g0 = h.tensor(A, W.CAT_AGRAD)
    d1 = h.tensor(1024, W.CAT_WGRAD, scaled=False)
    h.op(1, W.PH_BWD, [h1, h0], [g0, d1], t_b)
    d0 = h.tensor(1024, W.CAT_WGRAD, scaled=False)
    h.op(0, W.PH_BWD, [g0, x], [d0], t_b)
    for w, d in ((w0, d0), (w1, d1)):
        w2 = h.tensor(1024, W.CAT_WEIGHT, scaled=False)
        h.op(0 if w == w0 else 1, W.PH_OPT, [w, d], [w2], t_opt, scaled=False)
    tr = h.build()
    assert (h0, g0) == (3, 5)
    r = oracle.run_point(tr, W.ring(2, bw=B, lat=a), W.make_point(0, W.ST_PP, pp=2, m=2, B=2), plan=[0, 1])
    # programs: stage 0 (GPU 0) F0(0) F0(1) B0(1) B0(0) O0; stage 1 (GPU 1) F1(0) F1(1) B1(1) B1(0) O1
    ev = []
    # F0(j) ends at (j+1) t_f and pushes h0(j) to GPU 1
    for j in range(2):
        te = (j + 1) * t_f
        ev += [(te, TASK_END, task_code(0, j)), (te, RELEASE, p2p_code(h0, j, 1)),
               (te + a, ACTIVATE, p2p_code(h0, j, 1)), (te + c, DELIVER, p2p_code(h0, j, 1))]
    # F1(0) starts on delivery at t_f + c; F1(1) at 2 t_f + c (= its delivery = F1(0)'s end)
    ev += [(t_f + c, TASK_START, task_code(1, 0)), (2 * t_f + c, TASK_START, task_code(1, 1))]
    # B1(1) starts at 3 t_f + c (reads h0(1), already delivered), ends t_b later and pushes g0(1);
    # B1(0) starts right after it (reads h0(0)) and pushes g0(0) at its end
    tb1 = 3 * t_f + c
    ev += [(tb1, TASK_START, task_code(1, 2))]
    for k, j in enumerate((1, 0)):
        te = tb1 + (k + 1) * t_b
        ev += [(te, TASK_END, task_code(1, 2 + k)), (te, RELEASE, p2p_code(g0, j, 0)),
               (te + a, ACTIVATE, p2p_code(g0, j, 0)), (te + c, DELIVER, p2p_code(g0, j, 0))]
    ev += [(tb1 + t_b, TASK_START, task_code(1, 3))]
    # B0(1) starts on g0(1)'s delivery, B0(0) on g0(0)'s delivery (= B0(1)'s end)
    ev += [(tb1 + t_b + c, TASK_START, task_code(0, 2)), (tb1 + 2 * t_b + c, TASK_START, task_code(0, 3))]
    T = 3 * (t_f + t_b) + 2 * c + t_opt
    assert r["iter_time_s"] == T
    assert r["order_hash"] == r19_hash(ev)
    assert r["n_instants"] == n_instants(ev) == 13
    assert r["n_wf_calls"] == 8 and r["n_wf_rounds"] == 4 and r["max_active_flows"] == 1
    assert r["n_p2p"] == 4


def test_hash_differs_under_a_single_event_change():
    """The pins above would catch a one-event slip: moving one event by one ulp, or changing one
    code bit, changes the hash (a property of the definition, checked on the CF5 event set)."""
    ev = [(1.0, RELEASE, 7), (2.0, DELIVER, 7)]
    h = r19_hash(ev)
    assert r19_hash([(1.0, RELEASE, 7), (2.0000000000000004, DELIVER, 7)]) != h
    assert r19_hash([(1.0, RELEASE, 6), (2.0, DELIVER, 7)]) != h
    assert r19_hash([(1.0, ACTIVATE, 7), (2.0, DELIVER, 7)]) != h
