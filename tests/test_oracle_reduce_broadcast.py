"""Pins for R26: AllReduce as ring Reduce to member 0 + ring Broadcast from member 0, pipelined in
chunks (NEXT 3; "NCCL-style collective communication, including reduce, scatter, and gather",
P:398; R26).

* uniform ring closed form (c <= p): the reduce chain fills in p-1 chunk times, the broadcast chain
  adds p-1 more, the c chunks one each: (2p + c - 3)(a + S/(c B));
* an independently built reduce + broadcast task graph (the R26 rule written out here) re-simulated in
  exact rational arithmetic (tests/ratsim.py) reproduces the oracle on heterogeneous rings and stars;
* structure: 2(p-1)c flows of S/c, payload S; AllGather / ReduceScatter keep the plain ring.
"""
import numpy as np
import pytest

import oracle
from paper_conf_isca_libwmvgjbj025_b200 import workloads as W
from tests import ratsim
from tests.helpers import HandGraph, links_of, one_wgrad_trace, rel

T_F, T_B = 2.0 ** -10, 2.0 ** -9


def _pt(p, c, strategy=W.ST_DP):
    return W.make_point(0, strategy, dp=p, B=p, chunks=c, algo=W.ALG_REDBCAST)


@pytest.mark.parametrize("p,c", [(2, 1), (3, 1), (4, 2), (8, 1), (8, 8), (16, 4)])
def test_uniform_ring_closed_form(p, c):
    S, B, a = 64e6, 50e9, 3e-6
    tr = one_wgrad_trace(int(S), T_F, T_B)
    r = oracle.run_point(tr, W.ring(p, bw=B, lat=a), _pt(p, c))
    assert r["status"] == 0
    exp = T_F + T_B + (2 * p + c - 3) * (a + S / (c * B))
    assert rel(r["iter_time_s"], exp) < 1e-12
    assert r["n_flows"] == 2 * (p - 1) * c and r["n_collectives"] == 1 and r["coll_payload_bytes"] == S


def _reduce_bcast_graph(p, c, S, members):
    """Written from R26: member i sends one flow at a time to member i+1; reduce chunks (i >= 1) first,
    then broadcast chunks (i <= p-2)."""
    g = HandGraph()
    bw = []
    for i in range(p):
        g.task(members[i], T_F)
        bw.append(g.task(members[i], T_B))
    start = g.barrier(bw, coll_start=True)
    red, bc, last = {}, {}, {}
    for j in range(c):
        for i in range(1, p):
            deps = []
            if i in last:
                deps.append(last[i])
            if i >= 2:
                deps.append(red[(i - 1, j)])
            if not deps:
                deps = [start]
            red[(i, j)] = last[i] = g.flow(members[i], members[(i + 1) % p], S / c, deps)
    for j in range(c):
        for i in range(0, p - 1):
            deps = [last[i]] if i in last else []
            deps.append(red[(p - 1, j)] if i == 0 else bc[(i - 1, j)])
            bc[(i, j)] = last[i] = g.flow(members[i], members[i + 1], S / c, deps)
    return g.arrays()


@pytest.mark.parametrize("seed", range(8))
def test_heterogeneous_matches_hand_built_graph(seed):
    rng = np.random.Generator(np.random.PCG64(300 + seed))
    p = int(rng.integers(2, 6))
    c = int(rng.integers(1, 5))
    S = float(2 ** int(rng.integers(16, 24)))
    topo = W.star(p) if seed % 3 == 2 else W.ring(p)
    topo.links["bw_Bps"] = rng.uniform(5e9, 100e9, len(topo.links))
    topo.links["lat_s"] = rng.uniform(0.0, 2e-5, len(topo.links))
    tr = one_wgrad_trace(int(S), T_F, T_B)
    r = oracle.run_point(tr, topo, _pt(p, c))
    assert r["status"] == 0
    members = [int(x) for x in topo.ring_order[:p]]
    T, _, _ = ratsim.simulate(_reduce_bcast_graph(p, c, S, members), topo.n_nodes, links_of(topo))
    assert rel(r["iter_time_s"], float(T)) < 1e-12


def test_allgather_keeps_the_ring_and_limits():
    """PAPER-mode TP all-gathers with the ring whatever the AllReduce algorithm; its AllReduces follow R26."""
    tr = W.mlp_trace()
    topo = W.ring(4, bw=25e9, lat=1e-6)
    mk = lambda algo: W.make_point(0, W.ST_TP, tp=4, B=64, tp_mode=W.TPM_PAPER, algo=algo)
    r_ring, r_rb = oracle.run_point(tr, topo, mk(W.ALG_RING)), oracle.run_point(tr, topo, mk(W.ALG_REDBCAST))
    assert r_ring["status"] == 0 and r_rb["status"] == 0
    assert r_rb["coll_payload_bytes"] == r_ring["coll_payload_bytes"]
    assert r_rb["n_collectives"] == r_ring["n_collectives"]
    assert oracle.run_point(tr, topo, W.make_point(0, W.ST_DDP, dp=4, B=64, algo=7))["status"] == W.PT_BAD_CONFIG


def test_hybrid_and_degenerate_groups():
    tr = W.mlp_trace()
    topo = W.ring(8, bw=25e9, lat=1e-6)
    for pt in (W.make_point(0, W.ST_HYBRID, dp=2, tp=2, pp=2, m=2, B=128, algo=W.ALG_REDBCAST, chunks=2),
               W.make_point(0, W.ST_DDP, dp=1, B=64, algo=W.ALG_REDBCAST)):
        r = oracle.run_point(tr, topo, pt)
        assert r["status"] == 0
