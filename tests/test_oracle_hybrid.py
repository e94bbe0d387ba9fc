"""Oracle pins for HYBRID DP x TP x PP (R9; Table 1, reading Q26):
degenerate degrees reduce bit-exactly (every output incl. the order hash) to DDP / TP / PP,
the exported graphs re-simulate exactly in rational arithmetic, and structural counts follow
from the composition."""
import numpy as np
import pytest

import oracle
from paper_conf_isca_libwmvgjbj025_b200 import workloads as W
from tests import ratsim
from tests.helpers import links_of, rel


def _case(seed, n_gpus=8):
    rng = np.random.Generator(np.random.PCG64(seed))
    tr = W.random_trace(rng, n_layers=int(rng.integers(3, 6)), max_ops_per_layer=3, b0=2)
    topo = W.random_topology(rng, n_gpus=n_gpus, n_switch=int(rng.integers(0, 2)), p_edge=0.2)
    return rng, tr, topo


def same(a, b):
    return all(a[f] == b[f] for f in W.RESULT_DTYPE.names)


@pytest.mark.parametrize("seed", range(10))
def test_hybrid_reduces_to_ddp(seed):
    rng, tr, topo = _case(seed)
    for d in (2, 3, 4):
        for bucket in (0, 3000):
            for algo in (W.ALG_RING, W.ALG_TREE):
                h = oracle.run_point(tr, topo, W.make_point(0, W.ST_HYBRID, dp=d, tp=1, pp=1, m=1, B=2 * d,
                                                            bucket=bucket, algo=algo))
                r = oracle.run_point(tr, topo, W.make_point(0, W.ST_DDP, dp=d, B=2 * d, bucket=bucket, algo=algo))
                assert h["status"] == 0 and same(h, r)


@pytest.mark.parametrize("seed", range(10))
def test_hybrid_reduces_to_tp(seed):
    rng, tr, topo = _case(100 + seed)
    for t in (2, 4):
        for mode in (W.TPM_PAPER, W.TPM_MEGATRON):
            for algo in (W.ALG_RING, W.ALG_TREE):
                h = oracle.run_point(tr, topo, W.make_point(0, W.ST_HYBRID, dp=1, tp=t, pp=1, m=1, B=4,
                                                            tp_mode=mode, algo=algo))
                r = oracle.run_point(tr, topo, W.make_point(0, W.ST_TP, tp=t, B=4, tp_mode=mode, algo=algo))
                assert h["status"] == 0 and same(h, r)


@pytest.mark.parametrize("seed", range(10))
def test_hybrid_reduces_to_pp(seed):
    rng, tr, topo = _case(200 + seed)
    for s in range(1, min(4, tr.n_layers) + 1):
        for m in (1, 2, 3):
            h = oracle.run_point(tr, topo, W.make_point(0, W.ST_HYBRID, dp=1, tp=1, pp=s, m=m, B=2 * m))
            r = oracle.run_point(tr, topo, W.make_point(0, W.ST_PP, pp=s, m=m, B=2 * m))
            assert h["status"] == 0 and same(h, r)


@pytest.mark.parametrize("seed", range(8))
def test_hybrid_exact_rational(seed):
    rng, tr, topo = _case(300 + seed, n_gpus=8)
    dp, tp, pp = [(2, 2, 2), (2, 2, 1), (1, 2, 2), (2, 1, 2), (2, 2, 2), (1, 2, 3), (2, 1, 3), (2, 2, 2)][seed]
    pp = min(pp, tr.n_layers)
    m = 2
    pt = W.make_point(0, W.ST_HYBRID, dp=dp, tp=tp, pp=pp, m=m, B=dp * m * 2, bucket=int(rng.choice([0, 2000])),
                      tp_mode=int(rng.integers(0, 2)), algo=int(rng.integers(0, 2)))
    r = oracle.run_point(tr, topo, pt)
    assert r["status"] == 0
    g = oracle.export_graph(tr, topo, pt)
    T, done, st = ratsim.simulate(g, topo.n_nodes, links_of(topo))
    assert rel(r["iter_time_s"], float(T)) < 1e-12


def test_hybrid_structure_on_a_transformer():
    """GPT-like trace, Megatron roles: per TP group 2 AllReduces per block per micro-batch in FWD and
    2 in BWD; P2P of the residual stream (and its gradient) between consecutive stages; DP payload =
    the TP-sharded gradient bytes of every stage."""
    tr = W.transformer_trace("tiny-gpt", 4, 64, 4, 256, 16, 100, 2, 9)
    topo = W.star(8, 100e9, 1e-6)
    dp, tp, pp, m = 2, 2, 2, 3
    pt = W.make_point(0, W.ST_HYBRID, dp=dp, tp=tp, pp=pp, m=m, B=dp * m * 2, bucket=0)
    r = oracle.run_point(tr, topo, pt)
    assert r["status"] == 0
    n_blocks = 4
    n_wgrad = int((tr.tensors["category"] == W.CAT_WGRAD).sum())
    assert r["n_collectives"] == dp * pp * 0 + dp * (4 * n_blocks * m) + tp * pp * 0 + tp * n_wgrad
    assert r["n_p2p"] > 0
    # the same point without TP has no TP collectives and full-size gradients
    r1 = oracle.run_point(tr, topo, W.make_point(0, W.ST_HYBRID, dp=dp, tp=1, pp=pp, m=m, B=dp * m * 2, bucket=0))
    assert r1["n_collectives"] == n_wgrad
    assert r1["coll_payload_bytes"] == float(tr.tensors["bytes_b0"][tr.tensors["category"] == W.CAT_WGRAD].sum())


def test_hybrid_statuses():
    tr = W.mlp_trace()
    t = W.ring(8)
    P = W.make_point
    assert oracle.run_point(tr, t, P(0, W.ST_HYBRID, dp=2, tp=2, pp=3, m=1, B=8))["status"] == W.PT_BAD_DEGREES
    assert oracle.run_point(tr, t, P(0, W.ST_HYBRID, dp=2, tp=2, pp=2, m=3, B=8))["status"] == W.PT_BAD_BATCH
    assert oracle.run_point(tr, t, P(0, W.ST_HYBRID, dp=2, tp=2, pp=2, m=0, B=8))["status"] == W.PT_BAD_DEGREES
    assert oracle.run_point(tr, t, P(0, W.ST_HYBRID, dp=2, tp=2, pp=2, m=2, B=8), plan=[0, 9])["status"] == W.PT_BAD_PLAN
    assert oracle.run_point(tr, t, P(0, W.ST_HYBRID, dp=2, tp=2, pp=2, m=2, B=8))["status"] == 0
