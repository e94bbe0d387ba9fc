"""Pins for R25, the pipelined (chunked) ring (NEXT 3; "recreates the behavior of the
open-sourced NCCL implementation"; R25).

* c <= 1 is R10 bit for bit (result record and order hash);
* uniform ring closed form 2(p-1) c (a + S/(p c B)) -- every member moves in lockstep;
* an independently built chunked-ring task graph (the R25 dependency rule written out here, not the
  oracle's expansion) re-simulated in exact rational arithmetic (tests/ratsim.py) reproduces the
  oracle's iteration time on heterogeneous rings and through a switch;
* structural counts: c times the flows, same payload; chunking never slows a latency-free ring.
"""
import numpy as np
import pytest

import oracle
from paper_conf_isca_libwmvgjbj025_b200 import workloads as W
from tests import ratsim
from tests.helpers import HandGraph, links_of, one_wgrad_trace, rel

T_F, T_B = 2.0 ** -10, 2.0 ** -9


def _pt(p, c, strategy=W.ST_DP, **kw):
    return W.make_point(0, strategy, dp=p, B=p, chunks=c, **kw)


@pytest.mark.parametrize("strategy", [W.ST_DP, W.ST_DDP])
@pytest.mark.parametrize("p", [2, 3, 5])
def test_one_chunk_is_the_plain_ring(strategy, p):
    rng = np.random.Generator(np.random.PCG64(p))
    tr = W.resnet50_trace() if p == 2 else W.mlp_trace()
    topo = W.ring(p)
    topo.links["bw_Bps"] = rng.uniform(5e9, 100e9, len(topo.links))
    topo.links["lat_s"] = rng.uniform(0.0, 2e-5, len(topo.links))
    base = oracle.run_point(tr, topo, W.make_point(0, strategy, dp=p, B=p * 16, bucket=1 << 22))
    for c in (0, 1):
        r = oracle.run_point(tr, topo, W.make_point(0, strategy, dp=p, B=p * 16, bucket=1 << 22, chunks=c))
        assert r == base


@pytest.mark.parametrize("p,c", [(2, 2), (3, 4), (4, 3), (8, 8), (16, 2)])
def test_uniform_ring_closed_form(p, c):
    """Lockstep members: 2(p-1)c flows in sequence on every member, each a + S/(p c B)."""
    S, B, a = 96e6, 50e9, 2e-6
    tr = one_wgrad_trace(int(S), T_F, T_B)
    r = oracle.run_point(tr, W.ring(p, bw=B, lat=a), _pt(p, c))
    assert r["status"] == 0
    exp = T_F + T_B + 2 * (p - 1) * c * (a + S / (p * c * B))
    assert rel(r["iter_time_s"], exp) < 1e-12
    assert r["n_flows"] == 2 * (p - 1) * p * c and r["n_collectives"] == 1
    assert r["coll_payload_bytes"] == S


def _chunked_ring_graph(p, c, S, members):
    """Compute (F, B per GPU) -> one ring AllReduce with c chunks per step, written from R25:
    member i sends q = k c + j (k < 2(p-1), j < c) one at a time; flow (i, q) waits for (i, q-1) and,
    when k >= 1, for (i-1, q-c)."""
    g = HandGraph()
    bw = []
    for i in range(p):
        g.task(members[i], T_F)
        bw.append(g.task(members[i], T_B))
    start = g.barrier(bw, coll_start=True)
    K = 2 * (p - 1) * c
    fid = {}
    for q in range(K):
        for i in range(p):
            deps = [start] if q == 0 else [fid[(i, q - 1)]]
            if q >= c:
                deps.append(fid[((i - 1) % p, q - c)])
            fid[(i, q)] = g.flow(members[i], members[(i + 1) % p], S / p / c, deps)
    return g.arrays()


@pytest.mark.parametrize("seed", range(8))
def test_heterogeneous_ring_matches_hand_built_graph(seed):
    rng = np.random.Generator(np.random.PCG64(100 + seed))
    p = int(rng.integers(2, 6))
    c = int(rng.integers(2, 5))
    S = float(2 ** int(rng.integers(16, 24)))
    star = seed % 3 == 2
    topo = W.star(p) if star else W.ring(p)
    topo.links["bw_Bps"] = rng.uniform(5e9, 100e9, len(topo.links))
    topo.links["lat_s"] = rng.uniform(0.0, 2e-5, len(topo.links))
    tr = one_wgrad_trace(int(S), T_F, T_B)
    r = oracle.run_point(tr, topo, _pt(p, c))
    assert r["status"] == 0
    members = [int(x) for x in topo.ring_order[:p]]
    T, _, _ = ratsim.simulate(_chunked_ring_graph(p, c, S, members), topo.n_nodes, links_of(topo))
    assert rel(r["iter_time_s"], float(T)) < 1e-12
    assert r["n_flows"] == 2 * (p - 1) * p * c


@pytest.mark.parametrize("seed", range(6))
def test_chunking_structure_and_latency_free_speedup(seed):
    """More chunks: c times the flows, the same payload; with zero latency a chunked ring is never
    slower than the plain one (its dependencies are a subset once scaled to chunk granularity)."""
    rng = np.random.Generator(np.random.PCG64(200 + seed))
    p = int(rng.integers(3, 7))
    topo = W.ring(p)
    topo.links["bw_Bps"] = rng.uniform(5e9, 100e9, len(topo.links))
    topo.links["lat_s"] = 0.0
    tr = one_wgrad_trace(1 << 22, T_F, T_B)
    r1 = oracle.run_point(tr, topo, _pt(p, 1))
    for c in (2, 4):
        rc = oracle.run_point(tr, topo, _pt(p, c))
        assert rc["n_flows"] == c * r1["n_flows"]
        assert rc["coll_payload_bytes"] == r1["coll_payload_bytes"]
        assert rc["iter_time_s"] <= r1["iter_time_s"] * (1 + 1e-12)


def test_tp_allgather_and_hybrid_chunked_counts():
    """Chunks apply to every ring collective (AllGather / ReduceScatter / AllReduce), in TP and HYBRID."""
    tr = W.mlp_trace()
    topo = W.ring(4, bw=25e9, lat=1e-6)
    for mk in (lambda c: W.make_point(0, W.ST_TP, tp=4, B=64, tp_mode=W.TPM_PAPER, chunks=c),
               lambda c: W.make_point(0, W.ST_HYBRID, dp=2, tp=2, pp=1, m=2, B=128, chunks=c)):
        r1, r3 = oracle.run_point(tr, topo, mk(1)), oracle.run_point(tr, topo, mk(3))
        assert r1["status"] == 0 and r3["status"] == 0
        assert r3["n_flows"] - r3["n_p2p"] == 3 * (r1["n_flows"] - r1["n_p2p"])
        assert r3["coll_payload_bytes"] == r1["coll_payload_bytes"]


def test_tree_ignores_chunks_and_limit():
    tr = W.mlp_trace()
    topo = W.star(4, bw=25e9, lat=1e-6)
    r1 = oracle.run_point(tr, topo, W.make_point(0, W.ST_DDP, dp=4, B=256, algo=W.ALG_TREE))
    r4 = oracle.run_point(tr, topo, W.make_point(0, W.ST_DDP, dp=4, B=256, algo=W.ALG_TREE, chunks=4))
    assert r1 == r4
    bad = oracle.run_point(tr, topo, W.make_point(0, W.ST_DDP, dp=4, B=256, chunks=17))
    assert bad["status"] == W.PT_BAD_CONFIG
