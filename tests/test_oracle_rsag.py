"""Pins of R29 (NEXT 3; "NCCL-style collective communication, including reduce, scatter, and gather";
DESIGN.md R29): coll_algo = RSAG runs every AllReduce as a ring ReduceScatter followed by a ring AllGather of
the same payload, two collectives of the group, the AllGather starting once every member has finished the
ReduceScatter.

* CF8 for each half: (p - 1)(alpha + S/(pB)); on a uniform ring the pair costs exactly the ring AllReduce
  (CF5) -- the members are in lockstep, the barrier between the halves is free;
* on heterogeneous rings the barrier can only delay: never faster than the pipelined ring AllReduce;
* counts: twice the collectives and the payload, the same flows;
* exact-rational re-simulation of the exported graphs (DP, DDP, TP, HYBRID) on random topologies.
"""
import numpy as np
import pytest

import oracle
from paper_conf_isca_libwmvgjbj025_b200 import workloads as W
from tests import ratsim
from tests.helpers import links_of, one_wgrad_trace, rel


@pytest.mark.parametrize("p", [2, 3, 4, 8])
def test_uniform_ring_equals_ring_allreduce(p):
    S, B, a = 96e6, 50e9, 2e-6
    tr = one_wgrad_trace(int(S))
    topo = W.ring(p, bw=B, lat=a)
    r = oracle.run_point(tr, topo, W.make_point(0, W.ST_DP, dp=p, B=p, algo=W.ALG_RSAG))
    r0 = oracle.run_point(tr, topo, W.make_point(0, W.ST_DP, dp=p, B=p, algo=W.ALG_RING))
    t_fb = 2.0 ** -10 + 2.0 ** -9
    half = (p - 1) * (a + S / (p * B))
    assert rel(r["iter_time_s"], t_fb + half + half) < 1e-12
    assert rel(r["iter_time_s"], r0["iter_time_s"]) < 1e-12
    assert r["n_collectives"] == 2 and r["coll_payload_bytes"] == 2 * S
    assert r["n_flows"] == r0["n_flows"] == 2 * (p - 1) * p


def test_reduce_scatter_half_closed_form():
    """The ReduceScatter half alone: a single-op trace whose OPT waits for the AllGather; its start time is
    t_fb + (p - 1)(alpha + S/(pB)) (read off the timeline: the AllGather's first flows' release)."""
    p, S, B, a = 4, 64e6, 25e9, 3e-6
    tr = one_wgrad_trace(int(S))
    r, tasks, flows = oracle.run_point(tr, W.ring(p, bw=B, lat=a), W.make_point(0, W.ST_DP, dp=p, B=p, algo=W.ALG_RSAG),
                                       timeline=True)
    ag = flows[(flows["code"] >> np.uint64(32)) == 1]   # collective 1 = the AllGather
    t_fb = 2.0 ** -10 + 2.0 ** -9
    assert len(ag) == (p - 1) * p
    assert rel(float(ag["release_s"].min()), t_fb + (p - 1) * (a + S / (p * B))) < 1e-12


@pytest.mark.parametrize("seed", range(5))
def test_heterogeneous_ring_never_faster(seed):
    rng = np.random.Generator(np.random.PCG64(40 + seed))
    p = int(rng.integers(3, 9))
    tr = one_wgrad_trace(int(rng.uniform(1e6, 1e8)))
    topo = W.ring(p, bw=20e9, lat=float(rng.uniform(0, 5e-6)))
    topo.links["bw_Bps"] /= rng.uniform(1, 10, len(topo.links))
    for st in (W.ST_DP, W.ST_DDP):
        t_ar = oracle.run_point(tr, topo, W.make_point(0, st, dp=p, B=p, algo=W.ALG_RING))["iter_time_s"]
        t_rs = oracle.run_point(tr, topo, W.make_point(0, st, dp=p, B=p, algo=W.ALG_RSAG))["iter_time_s"]
        assert t_rs >= t_ar * (1 - 1e-12)


MK = [
    lambda p: W.make_point(0, W.ST_DP, dp=p, B=2 * p, algo=W.ALG_RSAG),
    lambda p: W.make_point(0, W.ST_DDP, dp=p, B=2 * p, bucket=3000, algo=W.ALG_RSAG, chunks=2),
    lambda p: W.make_point(0, W.ST_TP, tp=p, B=4, algo=W.ALG_RSAG),
    lambda p: W.make_point(0, W.ST_TP, tp=p, B=4, tp_mode=W.TPM_PAPER, algo=W.ALG_RSAG),
    lambda p: W.make_point(0, W.ST_HYBRID, dp=2 if p >= 4 else 1, tp=2, pp=1, m=2, B=8, algo=W.ALG_RSAG),
]


@pytest.mark.parametrize("k", range(len(MK)))
@pytest.mark.parametrize("seed", range(4))
def test_exact_rational_resimulation(k, seed):
    rng = np.random.Generator(np.random.PCG64(7000 + 10 * seed + k))
    tr = W.random_trace(rng, n_layers=int(rng.integers(3, 5)), max_ops_per_layer=2, b0=2, bytes_hi=1 << 12)
    p = int(rng.integers(2, 5))
    topo = W.random_topology(rng, n_gpus=p, n_switch=int(rng.integers(0, 2)), p_edge=0.3)
    pt = MK[k](p)
    r = oracle.run_point(tr, topo, pt)
    assert r["status"] == 0
    g = oracle.export_graph(tr, topo, pt)
    T, done, st = ratsim.simulate(g, topo.n_nodes, links_of(topo))
    assert rel(r["iter_time_s"], float(T)) < 1e-12
    pr = np.array(pt, W.POINT_DTYPE).copy()
    pr["coll_algo"] = W.ALG_RING
    ring = oracle.run_point(tr, topo, pr)
    assert ring["n_flows"] == r["n_flows"]                      # the same ring flows ...
    n_ar = r["n_collectives"] - ring["n_collectives"]            # ... every AllReduce split in two
    assert n_ar >= 0 and r["coll_payload_bytes"] >= ring["coll_payload_bytes"]
