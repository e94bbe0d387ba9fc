"""The oracle's explicit task graphs re-simulated in exact rational arithmetic
(tests/ratsim.py), plus metamorphic checks of the discrete-event engine:
processing-order independence (permuting node ids) and structural counts."""
import numpy as np
import pytest

import oracle
from paper_conf_isca_libwmvgjbj025_b200 import workloads as W
from tests import ratsim
from tests.helpers import HandGraph, links_of, rel

STRATS = [
    ("dp", lambda p: W.make_point(0, W.ST_DP, dp=p, B=2 * p)),
    ("ddp", lambda p: W.make_point(0, W.ST_DDP, dp=p, B=2 * p, bucket=0)),
    ("ddp_bucket", lambda p: W.make_point(0, W.ST_DDP, dp=p, B=2 * p, bucket=3000)),
    ("ddp_tree", lambda p: W.make_point(0, W.ST_DDP, dp=p, B=2 * p, algo=W.ALG_TREE)),
    ("tp_meg", lambda p: W.make_point(0, W.ST_TP, tp=p, B=4)),
    ("tp_paper", lambda p: W.make_point(0, W.ST_TP, tp=p, B=4, tp_mode=W.TPM_PAPER)),
    ("tp_tree", lambda p: W.make_point(0, W.ST_TP, tp=p, B=4, algo=W.ALG_TREE)),
    ("pp", lambda p: W.make_point(0, W.ST_PP, pp=min(p, 3), m=2, B=4)),
    ("hybrid", lambda p: W.make_point(0, W.ST_HYBRID, dp=2 if p >= 4 else 1, tp=2, pp=1, m=2, B=8)),
]


def _case(seed, dyadic):
    rng = np.random.Generator(np.random.PCG64(seed))
    tr = W.random_trace(rng, n_layers=int(rng.integers(3, 5)), max_ops_per_layer=2, b0=2, dyadic=dyadic,
                        bytes_hi=1 << 12)
    p = int(rng.integers(2, 5))
    topo = W.random_topology(rng, n_gpus=p, n_switch=int(rng.integers(0, 2)), p_edge=0.3, dyadic=dyadic)
    if dyadic:
        tr.tensors["bytes_b0"] = 2 ** rng.integers(4, 12, len(tr.tensors))
    return tr, topo, p


@pytest.mark.parametrize("name,mk", STRATS)
@pytest.mark.parametrize("seed", range(6))
def test_oracle_matches_exact_rational_resimulation(name, mk, seed):
    dyadic = seed % 2 == 0
    tr, topo, p = _case(1000 * seed + len(name), dyadic)
    pt = mk(p)
    r = oracle.run_point(tr, topo, pt)
    assert r["status"] == 0, r["status"]
    g = oracle.export_graph(tr, topo, pt)
    T, done, st = ratsim.simulate(g, topo.n_nodes, links_of(topo))
    assert rel(r["iter_time_s"], float(T)) < 1e-12
    r2, td = oracle.sim_graph(g, topo, times=True, n_coll=r["n_collectives"], coll_payload=r["coll_payload_bytes"])
    for i in range(len(done)):
        assert abs(td[i] - float(done[i])) <= 1e-12 * max(float(T), 1e-30), i
    if dyadic and p in (2, 4) and name != "pp":
        # power-of-two sizes, rates and times: fp64 is exact, so is everything derived
        assert r["iter_time_s"] == float(T)
        assert r["n_wf_calls"] == st["wf_calls"] and r["n_wf_rounds"] == st["rounds"]
    assert r["max_active_flows"] >= 0


@pytest.mark.parametrize("seed", range(10))
def test_processing_order_independence(seed):
    """Relabelling the graph's nodes (keeping each GPU's program order) changes nothing:
    same times bit for bit, same counts, same order hash (R17/R19)."""
    tr, topo, p = _case(77 + seed, False)
    pt = STRATS[seed % len(STRATS)][1](p)
    g = oracle.export_graph(tr, topo, pt)
    r0 = oracle.sim_graph(g, topo)
    rng = np.random.Generator(np.random.PCG64(seed))
    n = len(g["type"])
    perm = rng.permutation(n)
    # restore per-GPU program order among tasks
    tasks = [i for i in range(n) if g["type"][i] == 0]
    pos = {i: q for q, i in enumerate(perm)}
    by_gpu = {}
    for i in tasks:
        by_gpu.setdefault(int(g["gpu"][i]), []).append(i)
    for gpu, lst in by_gpu.items():
        slots = sorted(pos[i] for i in lst)
        for i, s in zip(lst, slots):
            perm[s] = i
    inv = np.empty(n, np.int64)
    inv[perm] = np.arange(n)
    h = {k: g[k][perm] for k in ("type", "gpu", "dur", "src", "dst", "bytes", "code", "flags")}
    deps = [[int(inv[d]) for d in g["dep_ids"][g["dep_off"][i]:g["dep_off"][i + 1]]] for i in perm]
    off = np.zeros(n + 1, np.int64)
    flat = []
    for q, d in enumerate(deps):
        rng.shuffle(d)
        flat += d
        off[q + 1] = len(flat)
    h["dep_off"], h["dep_ids"] = off, np.asarray(flat if flat else [0], np.int32)
    r1 = oracle.sim_graph(h, topo)
    for f in r0.dtype.names:
        assert r1[f] == r0[f], f


def test_structural_counts_and_payload_conservation():
    tr = W.resnet50_trace()
    wsum = float(tr.tensors["bytes_b0"][tr.tensors["category"] == W.CAT_WGRAD].sum())
    for p in (2, 4):
        for bucket in (0, 1 << 20, 25 << 20, 1 << 40):
            r = oracle.run_point(tr, W.ring(p), W.make_point(0, W.ST_DDP, dp=p, B=p * 64, bucket=bucket,
                                                           bw=100e9, lat=1e-6))
            assert r["coll_payload_bytes"] == wsum  # every gradient byte reduced exactly once
            assert r["n_flows"] == r["n_collectives"] * 2 * (p - 1) * p
            assert r["n_compute"] == p * len(tr.ops)
        r = oracle.run_point(tr, W.ring(p), W.make_point(0, W.ST_DDP, dp=p, B=p * 64, bucket=0, algo=W.ALG_TREE))
        assert r["n_flows"] == r["n_collectives"] * 2 * (p - 1)
        assert r["n_collectives"] == 161


def test_point_statuses():
    tr = W.mlp_trace()
    t = W.ring(4)
    assert oracle.run_point(tr, t, W.make_point(0, W.ST_DP, dp=3, B=64))["status"] == W.PT_BAD_BATCH
    assert oracle.run_point(tr, t, W.make_point(0, W.ST_DP, dp=5, B=5))["status"] == W.PT_BAD_DEGREES
    assert oracle.run_point(tr, t, W.make_point(0, W.ST_DP, dp=2, tp=2, B=4))["status"] == W.PT_BAD_DEGREES
    assert oracle.run_point(tr, t, W.make_point(0, W.ST_PP, pp=5, m=1, B=4))["status"] == W.PT_BAD_DEGREES
    assert oracle.run_point(tr, t, W.make_point(0, W.ST_PP, pp=2, m=0, B=4))["status"] == W.PT_BAD_DEGREES
    assert oracle.run_point(tr, t, W.make_point(0, W.ST_PP, pp=2, m=3, B=4))["status"] == W.PT_BAD_BATCH
    assert oracle.run_point(tr, t, W.make_point(0, 9, dp=1, B=4))["status"] == W.PT_BAD_CONFIG
    assert oracle.run_point(tr, t, W.make_point(0, W.ST_DP, dp=1, B=4, bw=0.0))["status"] == W.PT_BAD_CONFIG
    assert oracle.run_point(tr, t, W.make_point(0, W.ST_PP, pp=2, m=1, B=4), plan=[0, 0])["status"] == W.PT_BAD_PLAN
    assert oracle.run_point(tr, t, W.make_point(0, W.ST_PP, pp=2, m=1, B=4), plan=[1, 2])["status"] == W.PT_BAD_PLAN
    assert oracle.run_point(tr, t, W.make_point(0, W.ST_PP, pp=2, m=1, B=4), plan=[0, 2])["status"] == 0
    # disconnected: two GPUs, one directed link only -> the reverse ring step has no route
    links = np.zeros(1, W.LINK_DTYPE)
    links[0] = (0, 1, 1.0, 0.0)
    one_way = W.Topology("oneway", 2, 2, links, np.arange(2, dtype=np.uint32))
    assert oracle.run_point(tr, one_way, W.make_point(0, W.ST_DP, dp=2, B=128))["status"] == W.PT_NO_ROUTE


def test_deadlock_is_reported():
    g = HandGraph()
    # task waits for a flow that waits for a later task on the same GPU
    a = g.task(0, 1.0, deps=[2])
    b = g.task(0, 1.0)
    f = g.flow(0, 1, 10.0, deps=[b])
    assert (a, b, f) == (0, 1, 2)
    r = oracle.sim_graph(g.arrays(), W.ring(2))
    assert r["status"] == W.PT_DEADLOCK


def test_zero_byte_and_local_flows():
    g = HandGraph()
    a = g.task(0, 0.25)
    f0 = g.flow(0, 1, 0.0, deps=[a])      # zero bytes: delivered after the latency
    f1 = g.flow(1, 1, 100.0, deps=[a])    # same node: empty route, delivered at release
    r, td = oracle.sim_graph(g.arrays(), W.ring(2, bw=10.0, lat=0.5), times=True)
    assert td[f0] == 0.75 and td[f1] == 0.25 and r["iter_time_s"] == 0.75
