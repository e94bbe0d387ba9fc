"""Oracle pins for the per-layer compute / communication breakdown ("the communication time and
computation time of each layer or stage"; Fig. 13; R22) by closed forms and invariants."""
import numpy as np
import pytest

import oracle
from paper_conf_isca_libwmvgjbj025_b200 import workloads as W
from tests.helpers import rel


def _layers_of(tr):
    return tr.ops["layer"].astype(np.int64)


@pytest.mark.parametrize("seed", range(6))
def test_compute_is_the_rank_program_split_by_layer(seed):
    """DP / DDP / TP: rank 0 runs every op, so the per-layer compute partitions compute_busy_max; with dyadic
    op times every partial fold is exact and the identity is bit-exact."""
    rng = np.random.Generator(np.random.PCG64(3100 + seed))
    tr = W.random_trace(rng, n_layers=int(rng.integers(2, 6)), max_ops_per_layer=3, dyadic=True)
    topo = W.ring(4, 2.0 ** 33, 2.0 ** -20)
    for pt in (W.make_point(0, W.ST_DDP, dp=4, B=4 * tr.trace_batch), W.make_point(0, W.ST_DP, dp=2, B=2),
               W.make_point(0, W.ST_TP, tp=4, B=tr.trace_batch, tp_mode=int(rng.integers(0, 2)))):
        r, comp, comm = oracle.run_point(tr, topo, pt, breakdown=True)
        assert r["status"] == 0
        assert comp.sum() == r["compute_busy_max_s"]
        t = tr.ops["time_s"]
        # the layer's own ops at the trace batch (dp = 4 at 4 x b0 per rank -> rho == 1 exactly for DDP)
        if pt["strategy"] == W.ST_DDP:
            for l in range(tr.n_layers):
                sel = t[_layers_of(tr) == l]
                acc = 0.0
                for v in sel:
                    acc = acc + float(v)
                assert comp[l] == acc


@pytest.mark.parametrize("p", [2, 4, 8])
def test_ddp_per_tensor_comm_is_sum_of_ring_allreduce_closed_forms(p):
    """DDP with one AllReduce per weight gradient on a uniform ring: the group is FIFO, so every collective
    runs alone from its start and takes 2(p-1)(a + S/(pB)) (CF5); a layer's communication time is the sum
    over the gradients whose producing op is in that layer."""
    rng = np.random.Generator(np.random.PCG64(3200 + p))
    tr = W.random_trace(rng, n_layers=4, max_ops_per_layer=3)
    B, a = 40e9, 3e-6
    pt = W.make_point(0, W.ST_DDP, dp=p, B=p * tr.trace_batch, bucket=0)
    r, comp, comm = oracle.run_point(tr, W.ring(p, bw=B, lat=a), pt, breakdown=True)
    assert r["status"] == 0
    exp = np.zeros(tr.n_layers)
    prod = {}
    for o, op in enumerate(tr.ops):
        for k in range(int(op["n_out"])):
            prod[int(tr.io[op["io_off"] + op["n_in"] + k])] = o
    for x, ts in enumerate(tr.tensors):
        if ts["category"] == W.CAT_WGRAD and x in prod and tr.ops[prod[x]]["phase"] != W.PH_OPT:
            exp[int(tr.ops[prod[x]]["layer"])] += 2 * (p - 1) * (a + float(ts["bytes_b0"]) / (p * B))
    assert np.all(np.abs(comm - exp) <= 1e-12 * np.maximum(exp, 1e-300))


def test_tp_blocking_comm_per_layer():
    """Megatron TP on a uniform ring: each layer's communication = its ROW-forward and COL-backward
    AllReduces, each 2(p-1)(a + S/(pB)) (the stream blocks on every collective, CF12)."""
    tr = W.transformer_trace("tiny", 2, 64, 4, 256, 16, 100, 2, 5)
    p, B, a = 4, 25e9, 1e-6
    pt = W.make_point(0, W.ST_TP, tp=p, B=2, tp_mode=W.TPM_MEGATRON)
    r, comp, comm = oracle.run_point(tr, W.ring(p, bw=B, lat=a), pt, breakdown=True)
    exp = np.zeros(tr.n_layers)
    for o, op in enumerate(tr.ops):
        role = int(op["tp_role"]) & 3
        for k in range(int(op["n_out"])):
            x = int(tr.io[op["io_off"] + op["n_in"] + k])
            cat = int(tr.tensors[x]["category"])
            if (role == 2 and op["phase"] == W.PH_FWD) or (role == 1 and op["phase"] == W.PH_BWD and cat == W.CAT_AGRAD):
                S = float(tr.tensors[x]["bytes_b0"]) * (1.0 if not tr.tensors[x]["batch_scaled"] else 2 / tr.trace_batch)
                exp[int(op["layer"])] += 2 * (p - 1) * (a + S / (p * B))
    assert exp.sum() > 0
    assert np.all(np.abs(comm - exp) <= 1e-12 * np.maximum(exp, 1e-300))
    assert rel(comp.sum(), r["compute_busy_max_s"]) < 1e-12


@pytest.mark.parametrize("S", [2, 3, 4])
def test_pp_stage_sums_and_p2p_closed_form(S):
    """GPipe: each layer's compute is on its stage's GPU (m instances of FWD/BWD ops, OPT once); the stage
    sums reproduce compute_busy_max as their max; every P2P send of a layer's output to a neighbouring
    stage over one uncontended link takes a + bytes/B."""
    rng = np.random.Generator(np.random.PCG64(3300 + S))
    tr = W.random_trace(rng, n_layers=6, max_ops_per_layer=2, roles=False)
    m, B, a = 3, 30e9, 2e-6
    pt = W.make_point(0, W.ST_PP, pp=S, m=m, B=m * tr.trace_batch)
    r, comp, comm = oracle.run_point(tr, W.ring(S, bw=B, lat=a), pt, breakdown=True)
    assert r["status"] == 0
    fl = oracle.partition(tr, S) + [tr.n_layers]
    stage_sum = [comp[fl[s]:fl[s + 1]].sum() for s in range(S)]
    assert rel(max(stage_sum), r["compute_busy_max_s"]) < 1e-12
    # P2P: a layer's output tensors read on another stage, once per micro-batch instance
    st = np.searchsorted(fl, np.arange(tr.n_layers), side="right") - 1
    readers = {}
    for o, op in enumerate(tr.ops):
        for k in range(int(op["n_in"])):
            readers.setdefault(int(tr.io[op["io_off"] + k]), set()).add(int(st[int(op["layer"])]))
    exp = np.zeros(tr.n_layers)
    for o, op in enumerate(tr.ops):
        l = int(op["layer"])
        n_inst = 1 if op["phase"] == W.PH_OPT else m
        for k in range(int(op["n_out"])):
            x = int(tr.io[op["io_off"] + op["n_in"] + k])
            for d in readers.get(x, ()):
                if d == st[l]:
                    continue
                hops = min((d - st[l]) % S, (st[l] - d) % S)
                if hops != 1:
                    pytest.skip("non-neighbour send (multi-hop route)")
                b = float(tr.tensors[x]["bytes_b0"]) * (1.0 if not tr.tensors[x]["batch_scaled"] else 1.0)
                exp[l] += n_inst * (a + b / B)
    assert np.all(np.abs(comm - exp) <= 1e-12 * np.maximum(exp, 1e-300))


@pytest.mark.parametrize("seed", range(4))
def test_hybrid_degenerate_degrees_reproduce_breakdowns(seed):
    """HYBRID with degenerate degrees is DDP / TP / PP bit for bit (R9) -- the breakdown too."""
    rng = np.random.Generator(np.random.PCG64(3400 + seed))
    tr = W.random_trace(rng, n_layers=4, max_ops_per_layer=3)
    topo = W.star(4, 50e9, 1e-6)
    P = W.make_point
    for a_, b_ in ((P(0, W.ST_DDP, dp=4, B=8, bucket=1 << 12), P(0, W.ST_HYBRID, dp=4, B=8, bucket=1 << 12)),
                   (P(0, W.ST_TP, tp=4, B=2), P(0, W.ST_HYBRID, tp=4, B=2)),
                   (P(0, W.ST_PP, pp=3, m=2, B=4), P(0, W.ST_HYBRID, pp=3, m=2, B=4))):
        ra, ca, ma = oracle.run_point(tr, topo, a_, breakdown=True)
        rb, cb, mb = oracle.run_point(tr, topo, b_, breakdown=True)
        assert ra["iter_time_s"] == rb["iter_time_s"]
        assert np.array_equal(ca, cb) and np.array_equal(ma, mb)


def test_breakdown_does_not_change_results():
    rng = np.random.Generator(np.random.PCG64(3500))
    tr = W.random_trace(rng, n_layers=4, max_ops_per_layer=3)
    pt = W.make_point(0, W.ST_HYBRID, dp=2, tp=2, pp=2, m=2, B=8)
    r0 = oracle.run_point(tr, W.mesh(2, 4, 30e9, 1e-6), pt)
    r1, _, _ = oracle.run_point(tr, W.mesh(2, 4, 30e9, 1e-6), pt, breakdown=True)
    assert r0.tobytes() == r1.tobytes()
