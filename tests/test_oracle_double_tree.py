"""Pins for R27: double binary tree AllReduce (NEXT 3; NCCL's trees, "NCCL-style collective
communication"; R27).

* closed forms on fully connected uniform topologies, where the two trees' flows never share a directed
  link at the same time: p = 2 and p = 3 finish in 2(a + S/(2B)) — half the payload per tree, one
  reduce level and one broadcast level — against 2(a + S/B) for the single tree;
* the complement property the mirrored tree is chosen for: for even p every member is interior in at
  most one of the two trees (checked on the oracle's own flow list through the timeline);
* an independently built two-tree task graph (the R27 rule written out here) re-simulated in exact
  rational arithmetic (tests/ratsim.py) reproduces the oracle on heterogeneous rings, stars and meshes;
* structure: 4(p-1) flows of S/2, payload S; p = 1 has no flows; AllGather keeps the ring.
"""
import numpy as np
import pytest

import oracle
from paper_conf_isca_libwmvgjbj025_b200 import workloads as W
from tests import ratsim
from tests.helpers import HandGraph, links_of, one_wgrad_trace, rel

T_F, T_B = 2.0 ** -10, 2.0 ** -9


def _full(p, bw, lat):
    return W._mk(f"full{p}", p, p, [(i, j, bw, lat) for i in range(p) for j in range(p) if i != j],
                 list(range(p)), bidir=False)


def _pt(p, algo=W.ALG_DBTREE):
    return W.make_point(0, W.ST_DP, dp=p, B=p, algo=algo)


@pytest.mark.parametrize("p", [2, 3])
def test_fully_connected_closed_form(p):
    S, B, a = 64e6, 50e9, 3e-6
    tr = one_wgrad_trace(int(S), T_F, T_B)
    topo = _full(p, B, a)
    r = oracle.run_point(tr, topo, _pt(p))
    assert r["status"] == 0
    assert rel(r["iter_time_s"], T_F + T_B + 2 * (a + S / (2 * B))) < 1e-12
    r1 = oracle.run_point(tr, topo, _pt(p, W.ALG_TREE))
    assert rel(r1["iter_time_s"], T_F + T_B + 2 * (a + S / B)) < 1e-12
    assert r["n_flows"] == 4 * (p - 1) and r["n_collectives"] == 1 and r["coll_payload_bytes"] == S


@pytest.mark.parametrize("p", [2, 4, 6, 8, 16])
def test_even_p_interior_nodes_are_complementary(p):
    """Senders of broadcast (down) flows are the interior nodes of a tree; for even p no member is
    interior in both (the mirrored heap), which is why NCCL pairs the trees."""
    tr = one_wgrad_trace(1 << 20, T_F, T_B)
    _, _, fl = oracle.run_point(tr, W.ring(p), _pt(p), timeline=True)
    step = (fl["code"] >> 16) & 0xFFFF
    interior = [set(int(s) for s in fl["src"][step == st]) for st in (1, 3)]
    assert not (interior[0] & interior[1])
    assert len(fl) == 4 * (p - 1)
    assert set(np.unique(fl["bytes"]).tolist()) == {float(1 << 19)}


def _double_tree_graph(p, S, members):
    """Written from R27: two heap trees over positions 0..p-1; tree A puts member h at position h,
    tree B member p-1-h; each child reduces to its parent after its own children's reduces, each
    parent broadcasts back after it holds the result (the root: after both children's reduces)."""
    g = HandGraph()
    bw = []
    for i in range(p):
        g.task(members[i], T_F)
        bw.append(g.task(members[i], T_B))
    start = g.barrier(bw, coll_start=True)
    for mirror in (0, 1):
        mem = (lambda h: p - 1 - h) if mirror else (lambda h: h)
        up, dn = {}, {}
        for h in range(p - 1, 0, -1):
            kids = [up[c] for c in (2 * h + 1, 2 * h + 2) if c < p]
            up[h] = g.flow(members[mem(h)], members[mem((h - 1) // 2)], S / 2, kids or [start])
        for h in range(1, p):
            par = (h - 1) // 2
            deps = [up[c] for c in (1, 2) if c < p] if par == 0 else [dn[par]]
            dn[h] = g.flow(members[mem(par)], members[mem(h)], S / 2, deps)
    return g.arrays()


@pytest.mark.parametrize("seed", range(9))
def test_heterogeneous_matches_hand_built_graph(seed):
    rng = np.random.Generator(np.random.PCG64(700 + seed))
    p = int(rng.integers(2, 8))
    S = float(2 ** int(rng.integers(16, 24)))
    topo = [W.ring, W.star, lambda q: W.mesh(2, (q + 1) // 2)][seed % 3](p)
    topo.links["bw_Bps"] = rng.uniform(5e9, 100e9, len(topo.links))
    topo.links["lat_s"] = rng.uniform(0.0, 2e-5, len(topo.links))
    tr = one_wgrad_trace(int(S), T_F, T_B)
    r = oracle.run_point(tr, topo, _pt(p))
    assert r["status"] == 0
    members = [int(x) for x in topo.ring_order[:p]]
    T, _, _ = ratsim.simulate(_double_tree_graph(p, S, members), topo.n_nodes, links_of(topo))
    assert rel(r["iter_time_s"], float(T)) < 1e-12


def test_degenerate_and_other_collectives():
    tr = W.mlp_trace()
    topo = W.ring(8, bw=25e9, lat=1e-6)
    r = oracle.run_point(tr, topo, W.make_point(0, W.ST_DDP, dp=1, B=64, algo=W.ALG_DBTREE))
    assert r["status"] == 0 and r["n_flows"] == 0
    # PAPER-mode TP all-gathers keep the ring; its AllReduces are double trees
    mk = lambda algo: W.make_point(0, W.ST_TP, tp=4, B=64, tp_mode=W.TPM_PAPER, algo=algo)
    r_ring, r_dt = oracle.run_point(tr, topo, mk(W.ALG_RING)), oracle.run_point(tr, topo, mk(W.ALG_DBTREE))
    assert r_dt["status"] == 0 and r_dt["coll_payload_bytes"] == r_ring["coll_payload_bytes"]
    assert r_dt["n_collectives"] == r_ring["n_collectives"]
    r = oracle.run_point(tr, topo, W.make_point(0, W.ST_HYBRID, dp=2, tp=2, pp=2, m=2, B=128, algo=W.ALG_DBTREE))
    assert r["status"] == 0
