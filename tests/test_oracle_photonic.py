"""Oracle pins for the photonic circuit-switched network model (R20): link setup,
port limit with teardown of the link idle the longest, destination receive buffers, dedicated
bandwidth -- by closed forms on hand-built graphs and by reduction to the flow network where the two
must coincide."""
import numpy as np
import pytest

import oracle
from paper_conf_isca_libwmvgjbj025_b200 import workloads as W
from tests.helpers import HandGraph, one_wgrad_trace, rel

B, L, SET = 2.0 ** 33, 2.0 ** -20, 2.0 ** -6      # dyadic: every closed form below is exact


def ph(n, ports=8, setup=SET, lat=L, bw=B, buf=0):
    return W.photonic(n, ports=ports, link_bw=bw, setup=setup, lat=lat, buf_slots=buf)


def test_single_transfer_pays_setup_latency_and_size_over_bandwidth():
    """no link yet -> establish it (setup), reserve the buffer, deliver after size / bw."""
    S, t0 = 2.0 ** 28, 2.0 ** -8
    g = HandGraph()
    a = g.task(0, t0)
    f = g.flow(0, 1, S, deps=[a])
    r, td = oracle.sim_graph(g.arrays(), ph(2), times=True)
    assert td[f] == ((t0 + SET) + L) + S / B
    assert r["iter_time_s"] == td[f] and r["status"] == 0
    assert r["n_wf_calls"] == 0 and r["n_wf_rounds"] == 0 and r["max_active_flows"] == 1
    assert r["comm_busy_s"] == td[f] - t0


def test_established_link_is_reused():
    """P:336 'check if there is already a link established': the second send on the same pair pays no setup."""
    S = 2.0 ** 26
    g = HandGraph()
    f1 = g.flow(0, 1, S)
    f2 = g.flow(0, 1, S, deps=[f1])
    r, td = oracle.sim_graph(g.arrays(), ph(2), times=True)
    assert td[f1] == (SET + L) + S / B
    assert td[f2] == (td[f1] + L) + S / B


def _chain(dsts, S=2.0 ** 24):
    g = HandGraph()
    prev = None
    fl = []
    for d in dsts:
        prev = g.flow(0, d, S, deps=[] if prev is None else [prev])
        fl.append(prev)
    return g, fl


@pytest.mark.parametrize("ports,dsts,setups", [
    (1, [1, 2, 1], 3),            # one port: every change of destination tears the link down
    (2, [1, 2, 1], 2),            # two ports: the third send reuses the link to 1
    (2, [1, 2, 1, 3, 2], 4),      # LRU: the send to 3 evicts the link to 2 (idle longest), so 2 is set up again
    (3, [1, 2, 1, 3, 2], 3),
    (1, [1, 1, 1], 1),
])
def test_port_limit_tears_down_the_link_idle_longest(ports, dsts, setups):
    """'we destroy the unused links that have been idle for the longest time if there is no port
    available'.  A sequential chain of sends from GPU 0 costs one setup per link (re-)establishment; an
    eviction policy other than least-recently-used gives a different count on the 5-send case."""
    S = 2.0 ** 24
    g, fl = _chain(dsts, S)
    r, td = oracle.sim_graph(g.arrays(), ph(4, ports=ports), times=True)
    assert r["iter_time_s"] == setups * SET + len(dsts) * (L + S / B)
    assert td[fl[-1]] == r["iter_time_s"]


@pytest.mark.parametrize("buf,expect_serial", [(1, True), (2, False), (0, False)])
def test_destination_buffer_serialises_concurrent_senders(buf, expect_serial):
    """'the sender waits until the destination has buffer space available'.  Two GPUs send to GPU 2
    at once; with one receive buffer the second (by release order, then canonical id) starts when the
    first is delivered."""
    S = 2.0 ** 27
    g = HandGraph()
    f1 = g.flow(0, 2, S)
    f2 = g.flow(1, 2, S)
    r, td = oracle.sim_graph(g.arrays(), ph(3, buf=buf), times=True)
    one = (SET + L) + S / B
    assert td[f1] == one
    assert td[f2] == ((one + L) + S / B if expect_serial else one)
    assert r["max_active_flows"] == (1 if expect_serial else 2)


def test_dedicated_bandwidth_no_sharing():
    """Circuit switching: concurrent transfers on different logical links each get the full link
    bandwidth (no max-min sharing), unlike the flow network's shared physical link."""
    S = 2.0 ** 27
    g = HandGraph()
    fs = [g.flow(0, d, S) for d in (1, 2, 3)]
    r, td = oracle.sim_graph(g.arrays(), ph(4, ports=4), times=True)
    for f in fs:
        assert td[f] == (SET + L) + S / B


@pytest.mark.parametrize("p", [2, 3, 4, 8, 16])
def test_ring_allreduce_closed_form(p):
    """Ring AllReduce over logical links: one setup per GPU (successor link), then 2(p-1) steps of
    L + S/(pB): T = t_fb + setup + 2(p-1)(L + S/(pB))."""
    S = 100e6
    tr = one_wgrad_trace(int(S))
    pt = W.make_point(0, W.ST_DP, dp=p, B=p)
    r = oracle.run_point(tr, ph(p, bw=50e9, lat=2e-6, setup=20e-3), pt)
    t_fb = 2.0 ** -10 + 2.0 ** -9
    assert r["status"] == 0
    assert rel(r["iter_time_s"], t_fb + 20e-3 + 2 * (p - 1) * (2e-6 + S / (p * 50e9))) < 1e-12
    assert r["n_flows"] == 2 * (p - 1) * p


def test_scales_apply_to_photonic_parameters():
    """bw_scale multiplies the logical-link bandwidth, lat_scale the setup and transfer latencies (R2)."""
    S = 2.0 ** 28
    tr = one_wgrad_trace(int(S))
    base = oracle.run_point(tr, ph(4), W.make_point(0, W.ST_DP, dp=4, B=4))
    sc = oracle.run_point(tr, ph(4, bw=B / 2, lat=L * 4, setup=SET * 4), W.make_point(0, W.ST_DP, dp=4, B=4))
    pt = W.make_point(0, W.ST_DP, dp=4, B=4, bw=0.5, lat=4.0)
    r = oracle.run_point(tr, ph(4), pt)
    assert r["iter_time_s"] == sc["iter_time_s"] != base["iter_time_s"]


def _ring_equivalence_points(rng, tr):
    P = W.make_point
    pts = []
    for _ in range(6):
        p = int(rng.integers(2, 7))
        pts.append((p, P(0, W.ST_DDP, dp=p, B=p * 2, bucket=int(rng.choice([0, 1 << 12])))))
        pts.append((p, P(0, W.ST_DP, dp=p, B=p)))
        pts.append((p, P(0, W.ST_TP, tp=p, B=2, tp_mode=int(rng.integers(0, 2)))))
        pp = min(p, tr.n_layers)
        pts.append((pp, P(0, W.ST_PP, pp=pp, m=int(rng.integers(1, 4)) * 1, B=6)))
    return pts


@pytest.mark.parametrize("seed", range(6))
def test_reduces_to_flow_network_on_a_ring_without_contention(seed):
    """With zero setup, unlimited buffers and ports for both ring neighbours, a logical link behaves like a
    dedicated physical link: on a ring topology where ring collectives and GPipe P2P never put two flows on
    one link at once, every time output equals the flow network's (latency-first, R13) -- a pin of the
    whole photonic path against the independently pinned flow network."""
    rng = np.random.Generator(np.random.PCG64(4200 + seed))
    tr = W.random_trace(rng, n_layers=4, max_ops_per_layer=3, dyadic=True)
    for p, pt in _ring_equivalence_points(rng, tr):
        if pt["strategy"] == W.ST_PP and pt["global_batch"] % pt["microbatches"]:
            continue
        bw, lat = 2.0 ** int(rng.integers(30, 36)), 2.0 ** -int(rng.integers(16, 24))
        e = oracle.run_point(tr, W.ring(p, bw=bw, lat=lat), pt)
        o = oracle.run_point(tr, W.photonic(p, ports=2, link_bw=bw, setup=0.0, lat=lat), pt)
        assert e["status"] == o["status"]
        for f in ("iter_time_s", "compute_busy_max_s", "comm_busy_s", "exposed_comm_s", "coll_payload_bytes"):
            assert o[f] == e[f], (f, pt)
        for f in ("n_compute", "n_flows", "n_collectives", "n_p2p"):
            assert o[f] == e[f], (f, pt)
        assert o["n_wf_calls"] == 0


def test_invalid_photonic_parameters_are_rejected():
    tr = one_wgrad_trace(1 << 20)
    for bad in (dict(ports=0), dict(bw=0.0), dict(setup=-1.0), dict(lat=float("inf"))):
        kw = dict(ports=8, bw=B, setup=SET, lat=L)
        kw.update(bad)
        with pytest.raises(oracle.OracleError):
            oracle.run_point(tr, ph(2, **kw), W.make_point(0, W.ST_DP, dp=2, B=2))
