"""Pins of the oracle's Hop decentralized-training model (NEXT 4, R28, Hop [42]).

* the communication graphs of Fig. 16a (ring-based, double ring), read off the exported task graph;
* closed forms on two workers: synchronous iterations K (t_fb + c + t_opt), and with staleness 1
  (K - 1)(t_fb + t_opt) + t_fb + max(t_opt, c);
* an independent max-plus recursion of the R28 rules (update queues with backup workers b and staleness s,
  token queues with iteration gap g, FIFO send streams) on contention-free topologies -- every update on
  its own link -- over a (b, s, g) grid with the paper's random 1-10x per-GPU slowdowns;
* the exact-rational re-simulation (tests/ratsim.py, threshold barriers) of the exported graphs on a
  switch star, where updates share links;
* counts, statuses and invariants (a backup worker is never slower when links are not shared).
"""
import itertools

import numpy as np
import pytest

import oracle
from paper_conf_isca_libwmvgjbj025_b200 import workloads as W
from tests import ratsim
from tests.helpers import links_of, one_wgrad_trace, rel


def fig16a_edges(n, graph):
    """Undirected edges of Fig. 16a's graphs, built as edge sets (not neighbour lists)."""
    def ring_based(nodes):
        m = len(nodes)
        e = {frozenset((nodes[i], nodes[(i + 1) % m])) for i in range(m)}
        e |= {frozenset((nodes[i], nodes[(i + m // 2) % m])) for i in range(m)}
        return {x for x in e if len(x) == 2}
    if graph == W.HOP_RING_BASED:
        return ring_based(list(range(n)))
    h = n // 2
    return ring_based(list(range(h))) | ring_based(list(range(h, n))) | {frozenset((i, i + h)) for i in range(h)}


def identity_order(topo):
    return W.Topology(topo.name, topo.n_nodes, topo.n_gpus, topo.links.copy(), np.arange(topo.n_gpus, dtype=np.uint32))


def slowed(topo, seed):
    """every GPU's communication bandwidth divided by a random factor in [1, 10]."""
    rng = np.random.Generator(np.random.PCG64(seed))
    u = rng.uniform(1.0, 10.0, topo.n_nodes)
    t = identity_order(topo)
    t.links["bw_Bps"] = t.links["bw_Bps"] / u[t.links["src"]]
    return t


def hop_point(n, K, b=0, s=0, g=0, graph=W.HOP_RING_BASED, B=None):
    return W.make_point(0, W.ST_HOP, dp=n, m=K, B=B or n, tp_mode=graph, hop=(b, s, g))


def maxplus(n, graph, K, b, s, g, t_f, t_b, t_opt, alpha, S, bw):
    """R28 as a max-plus recursion, valid when every update has its own link (no bandwidth sharing):
    bw[(src, dst)] is that link's bandwidth.  Returns the makespan."""
    E = fig16a_edges(n, graph)
    nb = {r: sorted(j for e in E if r in e for j in e if j != r) for r in range(n)}
    end_bwd, end_opt, sdone = {}, {}, {}
    last = {r: 0.0 for r in range(n)}
    T = 0.0
    for k in range(K):
        for r in range(n):
            st = end_opt.get((r, k - 1), 0.0)
            if g > 0 and k >= g:
                st = max([st] + [end_bwd[(j, k - g)] for j in nb[r]])
            end_bwd[(r, k)] = (st + t_f) + t_b
        for r in range(n):
            for j in nb[r]:
                rel_t = max(end_bwd[(r, k)], last[r])
                last[r] = sdone[(r, k, j)] = (rel_t + alpha) + S / bw[(r, j)]
                T = max(T, last[r])
        for r in range(n):
            need = len(nb[r]) - b
            ap = -np.inf
            if k >= s and need > 0:
                ap = sorted(sdone[(j, k - s, r)] for j in nb[r])[need - 1]
            end_opt[(r, k)] = max(end_bwd[(r, k)], ap) + t_opt
            T = max(T, end_opt[(r, k)])
    return T


def link_bw(topo):
    return {(int(l["src"]), int(l["dst"])): float(l["bw_Bps"]) for l in topo.links}


@pytest.mark.parametrize("n,graph", [(8, W.HOP_RING_BASED), (8, W.HOP_DOUBLE_RING), (4, W.HOP_RING_BASED),
                                     (2, W.HOP_RING_BASED), (12, W.HOP_DOUBLE_RING), (16, W.HOP_RING_BASED)])
def test_update_flows_follow_fig16a(n, graph):
    tr = one_wgrad_trace(4096, n_opt=1)
    topo = W.ring(n)
    K = 2
    g = oracle.export_graph(tr, topo, hop_point(n, K, graph=graph))
    assert g["status"] == 0
    flows = [(int(a), int(b)) for t, a, b in zip(g["type"], g["src"], g["dst"]) if t == 1]
    E = fig16a_edges(n, graph)
    assert sorted(flows) == sorted([(a, b) for e in E for a in e for b in e if a != b] * K)
    r = oracle.run_point(tr, topo, hop_point(n, K, graph=graph))
    assert r["n_p2p"] == r["n_flows"] == 2 * len(E) * K and r["n_collectives"] == 0
    assert r["n_compute"] == n * K * len(tr.ops)


@pytest.mark.parametrize("K", [1, 2, 5])
def test_two_workers_synchronous_closed_form(K):
    """n = 2, no backup, no staleness: every iteration is compute, one update each way, apply."""
    t_f, t_b, t_o = 2.0 ** -10, 2.0 ** -9, 2.0 ** -12
    S, B, a = 2 ** 20, 2.0 ** 30, 2.0 ** -16
    tr = one_wgrad_trace(S, t_f=t_f, t_b=t_b, t_o=t_o, n_opt=1)
    r = oracle.run_point(tr, W.ring(2, bw=B, lat=a), hop_point(2, K))
    assert r["status"] == 0
    assert r["iter_time_s"] == K * ((t_f + t_b) + (a + S / B) + t_o)


@pytest.mark.parametrize("K", [1, 3, 6])
@pytest.mark.parametrize("slow", [False, True])
def test_two_workers_staleness_one_closed_form(K, slow):
    """Staleness 1: iteration k applies the neighbour's update of k - 1, so communication hides behind the
    next iteration: (K-1)(t_fb + t_opt) + t_fb + max(t_opt, c) while c <= t_fb + t_opt."""
    t_f, t_b, t_o = 2.0 ** -10, 2.0 ** -9, 2.0 ** -12
    S, a = 2 ** 20, 2.0 ** -16
    B = 2.0 ** 31 if not slow else 2.0 ** 30   # c = 2^-16 + 2^-11 (> t_opt) or + 2^-10
    tr = one_wgrad_trace(S, t_f=t_f, t_b=t_b, t_o=t_o, n_opt=1)
    r = oracle.run_point(tr, W.ring(2, bw=B, lat=a), hop_point(2, K, s=1))
    c = a + S / B
    assert c <= t_f + t_b + t_o
    assert r["iter_time_s"] == (K - 1) * ((t_f + t_b) + t_o) + (t_f + t_b) + max(t_o, c)


GRID = list(itertools.product([0, 1, 2], [0, 1, 2], [0, 1, 3]))


@pytest.mark.parametrize("graph,topo_fn", [(W.HOP_RING_BASED, W.ring_graph), (W.HOP_DOUBLE_RING, W.double_ring)])
@pytest.mark.parametrize("seed", range(3))
def test_maxplus_recursion_on_dedicated_links(graph, topo_fn, seed):
    """Fig. 16's setting -- 8 workers, each update on its own link of the ring-based / double-ring graph, the
    GPUs' bandwidths slowed by random 1-10x factors -- against the max-plus recursion, over backup workers,
    staleness and the iteration gap."""
    t_f, t_b, t_o = 3.1e-3, 5.3e-3, 0.7e-3
    S, a = 40e6, 2e-6
    tr = one_wgrad_trace(int(S), t_f=t_f, t_b=t_b, t_o=t_o, n_opt=1)
    topo = slowed(topo_fn(8, bw=25e9, lat=a), 100 + seed)
    bw = link_bw(topo)
    K = 5
    for b, s, g in GRID:
        r = oracle.run_point(tr, topo, hop_point(8, K, b, s, g, graph))
        assert r["status"] == 0
        T = maxplus(8, graph, K, b, s, g, t_f, t_b, t_o, a, float(S), bw)
        assert rel(r["iter_time_s"], T) < 1e-12, (b, s, g, r["iter_time_s"], T)


@pytest.mark.parametrize("seed", range(4))
def test_backup_worker_never_slower_without_sharing(seed):
    """With updates on their own links, needing fewer updates (one backup worker) or older ones (staleness)
    can only move every event earlier; a tighter iteration gap only later."""
    t_f, t_b, t_o = 2e-3, 4e-3, 1e-3
    tr = one_wgrad_trace(int(60e6), t_f=t_f, t_b=t_b, t_o=t_o, n_opt=1)
    topo = slowed(W.ring_graph(8, bw=20e9, lat=3e-6), 7 + seed)
    T = {}
    for b, s, g in itertools.product([0, 1], [0, 1], [0, 1]):
        T[(b, s, g)] = oracle.run_point(tr, topo, hop_point(8, 6, b, s, g))["iter_time_s"]
    eps = 1e-12   # equal in exact arithmetic: rounding of the progress updates only
    for s, g in itertools.product([0, 1], [0, 1]):
        assert T[(1, s, g)] <= T[(0, s, g)] * (1 + eps)
    for b, g in itertools.product([0, 1], [0, 1]):
        assert T[(b, 1, g)] <= T[(b, 0, g)] * (1 + eps)
    for b, s in itertools.product([0, 1], [0, 1]):
        assert T[(b, s, 1)] >= T[(b, s, 0)] * (1 - eps)


@pytest.mark.parametrize("seed", range(6))
def test_exact_rational_resimulation_with_shared_links(seed):
    """Hop graphs on a switch star: every update crosses the shared switch links, so bandwidth is shared and
    re-allocated (R14); the exported graph (with its threshold barriers) re-simulated in exact rationals."""
    rng = np.random.Generator(np.random.PCG64(300 + seed))
    n = [2, 4, 8][seed % 3]
    graph = W.HOP_DOUBLE_RING if (seed % 2 and n % 4 == 0) else W.HOP_RING_BASED
    tr = one_wgrad_trace(2 ** int(rng.integers(8, 12)), t_f=2.0 ** -12, t_b=2.0 ** -11, t_o=2.0 ** -13, n_opt=1)
    topo = W.star(n, bw=2.0 ** int(rng.integers(18, 21)), lat=2.0 ** -20)
    b, s, g = int(rng.integers(0, 2)), int(rng.integers(0, 2)), int(rng.integers(0, 3))
    pt = hop_point(n, 3, b, s, g, graph)
    r = oracle.run_point(tr, topo, pt)
    assert r["status"] == 0
    ge = oracle.export_graph(tr, topo, pt)
    T, done, st = ratsim.simulate(ge, topo.n_nodes, links_of(topo))
    assert rel(r["iter_time_s"], float(T)) < 1e-12   # shares of 2^k / 3 are not dyadic: rounding only
    r2, td = oracle.sim_graph(ge, topo, times=True)
    for i in range(len(done)):
        assert abs(td[i] - float(done[i])) <= 1e-12 * float(T), i


def test_statuses():
    tr = one_wgrad_trace(4096, n_opt=1)
    topo = W.ring(8)
    assert oracle.run_point(tr, topo, hop_point(8, 2))["status"] == W.PT_OK
    assert oracle.run_point(tr, topo, hop_point(7, 2))["status"] == W.PT_BAD_DEGREES        # odd worker count
    assert oracle.run_point(tr, topo, hop_point(6, 2, graph=W.HOP_DOUBLE_RING))["status"] == W.PT_BAD_DEGREES
    assert oracle.run_point(tr, topo, hop_point(8, 0))["status"] == W.PT_BAD_DEGREES        # no iteration
    assert oracle.run_point(tr, topo, hop_point(16, 2))["status"] == W.PT_BAD_DEGREES       # > GPUs
    assert oracle.run_point(tr, topo, hop_point(8, 2, B=12))["status"] == W.PT_BAD_BATCH
    assert oracle.run_point(tr, topo, hop_point(8, 2, graph=2))["status"] == W.PT_BAD_CONFIG
    no_opt = one_wgrad_trace(4096, n_opt=0)
    assert oracle.run_point(no_opt, topo, hop_point(8, 2))["status"] == W.PT_BAD_CONFIG


def test_all_backups_means_no_waiting():
    """b = degree: nobody waits for an update; with fast links the workers run back to back and the last
    iteration's updates are the tail."""
    t_f, t_b, t_o = 2.0 ** -10, 2.0 ** -9, 2.0 ** -11
    S, B, a = 2 ** 16, 2.0 ** 34, 2.0 ** -20
    tr = one_wgrad_trace(S, t_f=t_f, t_b=t_b, t_o=t_o, n_opt=1)
    K = 4
    r = oracle.run_point(tr, W.ring_graph(8, bw=B, lat=a), hop_point(8, K, b=3))
    c = a + S / B
    # the last iteration's three sends (FIFO) end 3c after its backward pass
    assert r["iter_time_s"] == max(K * ((t_f + t_b) + t_o), (K - 1) * ((t_f + t_b) + t_o) + (t_f + t_b) + 3 * c)
