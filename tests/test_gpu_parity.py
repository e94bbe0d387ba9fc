"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle, element by element.

Small seeded cases are compared in full; the BASELINE.json configs are run at full size in
the launch configuration bench.py times and compared on seeded samples the oracle computes
one by one, plus properties that must hold for every point.
"""
import numpy as np
import pytest

import oracle
from paper_conf_isca_libwmvgjbj025_b200 import workloads as W
from tests import sweeps as S
from tests.parity import compare, expected_too_large

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ctx():
    import torch
    assert torch.cuda.is_available()
    from paper_conf_isca_libwmvgjbj025_b200 import triosim
    c = triosim.Context(0)
    yield c
    c.close()


def sample(n, k, seed):
    rng = np.random.Generator(np.random.PCG64(seed))
    return sorted(rng.choice(n, size=min(k, n), replace=False).tolist())


def check(got, sw, idx, allow_too_large=False):
    ref = oracle.run_sweep(sw, idx)
    bad, ulp = compare(got[idx], ref, idx, allow_too_large)
    assert not bad, "\n".join(bad[:20])
    return ulp


def test_c1_mlp_dp2_exact(ctx):
    sw = W.sweep_c1()
    got = ctx.run_sweep(sw)
    ref = oracle.run_sweep(sw)
    bad, ulp = compare(got, ref)
    assert not bad, bad
    assert ulp == 0
    assert (got["status"] == 0).all() and got["n_collectives"][0] == 8


@pytest.mark.parametrize("seed", range(4))
def test_random_small_all_strategies(ctx, seed):
    """Random traces x random topologies x every strategy / collective, several hundred points
    so each launch spans many warps, segments and a ragged tail."""
    sw = S.random_small(seed)
    got = ctx.run_sweep(sw)
    check(got, sw, list(range(len(sw.points))))
    assert (got["status"] == 0).sum() > 300


@pytest.mark.parametrize("seed", range(4))
def test_random_hybrid(ctx, seed):
    """HYBRID DP x TP x PP (R9) on random traces / topologies: every degree split, both TP modes,
    ring and tree, buckets, micro-batches; compared point by point with the oracle."""
    sw = S.random_hybrid(seed)
    got = ctx.run_sweep(sw)
    check(got, sw, list(range(len(sw.points))))
    assert (got["status"] == 0).sum() > 200


@pytest.mark.parametrize("seed", range(2))
def test_large_points_cta_kernel(ctx, seed):
    """More than 32 simulated GPUs (configs[4] scale): DDP / TP / PP points map to their exactly
    equivalent HYBRID form and run one point per CTA (64-256 ranks); compared with the oracle."""
    sw = S.large_points(seed)
    got = ctx.run_sweep(sw)
    assert (got["status"] == 0).all(), got["status"]
    check(got, sw, list(range(len(sw.points))))


def test_statuses_and_edge_cases(ctx):
    tr = W.mlp_trace()
    topos = [W.ring(4, 10e9, 1e-6), W.ring(32, 10e9, 1e-6), W.ring(40, 10e9, 1e-6), W.star(32, 10e9, 1e-6)]
    links = np.zeros(1, W.LINK_DTYPE)
    links[0] = (0, 1, 1e9, 0.0)
    topos.insert(3, W.Topology("oneway", 2, 2, links, np.arange(2, dtype=np.uint32)))
    P = W.make_point
    pts = W.points_array([
        P(0, W.ST_DP, dp=3, B=64),                       # bad batch
        P(0, W.ST_DP, dp=5, B=5),                        # too many GPUs
        P(0, W.ST_PP, pp=2, m=3, B=4),                   # bad batch (micro-batches)
        P(0, W.ST_PP, pp=2, m=1, B=4, plan=0),           # explicit plan ok
        P(0, W.ST_PP, pp=2, m=1, B=4, plan=1),           # bad plan
        P(0, W.ST_PP, pp=2, m=1, B=4, plan=7),           # plan index out of range
        P(9, W.ST_DP, dp=1, B=1),                        # topology out of range
        P(0, 7, dp=1, B=1),                              # unknown strategy
        P(0, W.ST_HYBRID, dp=2, tp=2, pp=1, m=1, B=4),   # hybrid DP x TP
        P(0, W.ST_DP, dp=1, B=64, bw=-1.0),              # bad scale
        P(3, W.ST_DDP, dp=2, B=128),                     # no route back
        P(1, W.ST_DDP, dp=32, B=32 * 64, bucket=1 << 20),  # 32 lanes: W = 32
        P(4, W.ST_DDP, dp=32, B=32 * 64, algo=W.ALG_TREE),  # tree over a 32-GPU switch
        P(0, W.ST_DP, dp=1, B=64),                       # single GPU: no communication
        P(0, W.ST_TP, tp=1, B=64),
        P(0, W.ST_PP, pp=1, m=2, B=128),
    ])
    sw = W.Sweep("edge", tr, topos, pts, plans=[[0, 2], [0, 0]])
    got = ctx.run_sweep(sw)
    check(got, sw, list(range(len(pts))))
    assert list(got["status"][:11]) == [1, 2, 1, 0, 6, 6, 7, 7, 0, 7, 3]
    # DataParallel (after-backward) with more than 32 GPUs runs in its HYBRID form; tree edges across a
    # 32-GPU ring span up to 16 hops -- past the 8 a flow caches in registers, read from the route table
    big = W.Sweep("big", tr, topos, W.points_array([P(2, W.ST_DP, dp=40, B=40 * 64),
                                                    P(1, W.ST_DDP, dp=32, B=32 * 64, algo=W.ALG_TREE)]))
    gb = ctx.run_sweep(big)
    assert list(gb["status"]) == [W.PT_OK, W.PT_OK]
    check(gb, big, [0, 1])
    # empty sweep
    empty = W.Sweep("empty", tr, topos, np.zeros(0, W.POINT_DTYPE))
    assert len(ctx.run_sweep(empty)) == 0


def test_partial_ranges_and_device_results(ctx):
    import torch
    rng = np.random.Generator(np.random.PCG64(3))
    tr = W.random_trace(rng, n_layers=4)
    topos = [W.ring(8, 20e9, 1e-6), W.mesh(2, 2, 20e9, 1e-6)]
    pts = W.points_array([W.make_point(i % 2, W.ST_DDP, dp=2 + (i % 3), B=12, bucket=(i % 4) * 500, bw=1 + i / 50)
                          for i in range(300)])
    sw = W.Sweep("ranges", tr, topos, pts)
    tid = ctx.triosim_load_trace(tr)
    sid = ctx.triosim_build_sweep(tid, topos, pts)
    ctx.triosim_simulate_batch(sid, 0, 300)
    full = ctx.triosim_results(sid, 0, 300)
    for first, count in ((0, 1), (17, 83), (299, 1), (100, 0)):
        ctx.triosim_simulate_batch(sid, first, count)
        part = ctx.triosim_results(sid, first, count)
        assert part.tobytes() == full[first:first + count].tobytes()
    buf = torch.zeros(300 * W.RESULT_DTYPE.itemsize, dtype=torch.uint8, device="cuda")
    s = torch.cuda.current_stream()
    ctx.triosim_simulate_batch(sid, 0, 300, stream=s.cuda_stream)
    ctx.triosim_results(sid, 0, 300, device_ptr=buf.data_ptr(), stream=s.cuda_stream)
    torch.cuda.synchronize()
    assert buf.cpu().numpy().tobytes() == full.tobytes()
    with pytest.raises(Exception):
        ctx.triosim_simulate_batch(sid, 250, 100)
    ctx.triosim_release(sid)
    ctx.triosim_release(tid)
    check(full, sw, sample(300, 60, 1))


def _properties_dp(got, sw):
    ok = got["status"] == 0
    assert ok.all()
    tr = sw.trace
    wsum = float(tr.tensors["bytes_b0"][tr.tensors["category"] == W.CAT_WGRAD].sum())
    p = sw.points["dp"].astype(np.int64)
    assert (got["coll_payload_bytes"] == wsum).all()
    assert (got["n_compute"] == p * len(tr.ops)).all()
    assert (got["n_flows"] == got["n_collectives"] * 2 * (p - 1) * p).all()
    assert (got["iter_time_s"] >= got["compute_busy_max_s"]).all()
    assert (got["exposed_comm_s"] == got["iter_time_s"] - got["compute_busy_max_s"]).all()


def test_c2_resnet50_dp_full_sweep(ctx):
    """configs[1] at full size (10,000 points, the bench workload): every point checked for
    the invariants, a stratified seeded sample against the oracle."""
    sw = W.sweep_c2()
    got = ctx.run_sweep(sw)
    _properties_dp(got, sw)
    # stratify: a few points of each (p, batch, bucket) class
    keys = {}
    for i, pt in enumerate(sw.points):
        keys.setdefault((int(pt["dp"]), int(pt["global_batch"]), int(pt["bucket_bytes"])), []).append(i)
    idx = sorted(set(i for v in keys.values() for i in v[:10]) | set(sample(len(sw.points), 600, 2)))
    check(got, sw, idx)


def test_c3_bert_large_tp_sampled(ctx):
    sw = W.sweep_c3()
    got = ctx.run_sweep(sw)
    assert (got["status"] == 0).all()
    check(got, sw, sample(len(sw.points), 1000, 3))


def test_c4_gpt2xl_pp_sampled(ctx):
    sw = W.sweep_c4()
    got = ctx.run_sweep(sw)
    assert (got["status"] == 0).all()
    assert (got["n_collectives"] == 0).all() and (got["n_p2p"] > 0).all()
    # cheap points plus a few of the largest (S=16, m=64)
    big = [i for i, pt in enumerate(sw.points) if pt["pp"] == 16 and pt["microbatches"] == 64][:3]
    check(got, sw, sorted(set(sample(len(sw.points), 300, 4) + big)))


def test_c5_gpt3_hybrid_sampled(ctx):
    """configs[4]'s structure at 8-32 GPUs (warp-segment hybrid kernel): a seeded subset of the lighter
    points (m = 8; the heaviest points have ~2M instants each) on the GPU, every point must simulate,
    16 of them against the oracle."""
    full = W.sweep_c5_small()
    light = [i for i, p in enumerate(full.points) if p["microbatches"] == 8 and p["tp"] <= 4]
    sub = [light[i] for i in sample(len(light), 120, 55)]
    sw = W.Sweep(full.name, full.trace, full.topos, full.points[sub])
    got = ctx.run_sweep(sw)
    assert (got["status"] == 0).all(), np.unique(got["status"], return_counts=True)
    check(got, sw, sample(len(sw.points), 16, 5))


def test_c5_full_scale_sampled(ctx):
    """configs[4] at full scale: the ~1M-point sweep over 64-1024 simulated GPUs (one point per CTA of up
    to 1024 threads).  A seeded sample of its lighter points at every N -- m = 8, dp <= 4, the symmetric
    hierarchical topologies above 64 GPUs (<= ~1.2e5 instants; the oracle finishes each in seconds.  The
    heaviest points, e.g. dp = 16 x tp = 8 at 128 GPUs or the perturbed topologies at 1024 GPUs, take
    1e6-1e7 instants and minutes of oracle time) -- in the sweep's launch configuration, all against the
    oracle."""
    full = W.sweep_c5()
    P = full.points
    N = P["dp"].astype(np.int64) * P["tp"] * P["pp"]
    sym = (P["topo"] % 2) == 0
    idx = []
    for n in (64, 128, 256, 512, 1024):
        cand = np.flatnonzero((N == n) & (P["microbatches"] == 8) & (P["dp"] <= 4) & (sym | (N == 64)))
        idx += [int(cand[i]) for i in sample(len(cand), 5, 600 + n)]
    sw = W.Sweep(full.name, full.trace, full.topos, P[sorted(set(idx))])
    got = ctx.run_sweep(sw)
    assert (got["status"] == 0).all(), np.unique(got["status"], return_counts=True)
    check(got, sw, list(range(len(sw.points))))


@pytest.mark.parametrize("seed", range(4))
def test_random_photonic(ctx, seed):
    """Photonic circuit-switched network (R20) on random traces: every strategy (all run in
    the hybrid kernel, whose lanes own their logical links), 1-4 ports (LRU teardown), 0-2 receive
    buffers, with and without setup latency; mixed in one sweep with flow-network points so warp
    segments of both models share a warp.  Compared point by point with the oracle."""
    sw = S.random_photonic(seed)
    got = ctx.run_sweep(sw)
    P = sw.points
    phot = np.array([sw.topos[int(p["topo"])].photonic is not None for p in P])
    # the one kernel limit (include/triosim.h): tree collectives over photonic links -- the broadcast flow's
    # sender is another lane -- for points that have a collective group
    coll = np.where(P["strategy"] == W.ST_TP, P["tp"] > 1,
                    np.where(P["strategy"] == W.ST_HYBRID, (P["dp"] > 1) | (P["tp"] > 1),
                             np.where(P["strategy"] == W.ST_PP, False, P["dp"] > 1)))
    expect = np.flatnonzero(phot & coll & (P["coll_algo"] == W.ALG_TREE))
    assert np.flatnonzero(got["status"] == W.PT_TOO_LARGE).tolist() == expect.tolist()
    check(got, sw, [i for i in range(len(P)) if i not in set(expect.tolist())])
    assert ((got["status"] == 0) & phot).sum() > 120


def test_wafer_passage_case_study(ctx):
    """NEXT 1 at full size: the 84-GPU wafer sweep (electrical mesh ring vs Passage photonic links, DDP
    ResNet-50), the bench workload of `bench.py --config wafer`; every point simulates, a seeded sample
    of both networks against the oracle, and the photonic ring pays one 20 ms link setup."""
    sw = W.sweep_wafer()
    got = ctx.run_sweep(sw)
    assert (got["status"] == 0).all()
    phot = sw.points["topo"] == 1
    assert (got["n_wf_calls"][phot] == 0).all() and (got["n_wf_calls"][~phot] > 0).all()
    assert (got["comm_busy_s"][phot] >= 20e-3 * sw.points["lat_scale"][phot]).all()
    idx = sample(len(sw.points), 24, 66)
    check(got, sw, idx)


def test_first_bucket_rule(ctx):
    """R24 (PyTorch DDP's first-bucket cap) for DP, DDP and HYBRID points, ring and tree, against the oracle;
    points differing only in the first cap fall in different structural classes."""
    rng = np.random.Generator(np.random.PCG64(2400))
    tr = W.resnet50_trace()
    topos = [W.ring(8, 100e9, 2e-6), W.star(8, 80e9, 1e-6)]
    pts = []
    for _ in range(160):
        st = int(rng.choice([W.ST_DP, W.ST_DDP, W.ST_HYBRID]))
        cap = int(rng.choice([0, 1 << 20, 25 << 20]))
        first = int(rng.choice([0, 1, 1 << 20, 4 << 20]))
        kw = dict(dp=int(rng.choice([2, 4, 8])), B=0) if st != W.ST_HYBRID else dict(dp=2, tp=2, pp=2, m=2, B=0)
        kw["B"] = kw["dp"] * int(kw.get("m", 1)) * 32
        pts.append(W.make_point(int(rng.integers(2)), st, bucket=cap, first_bucket=first, algo=int(rng.integers(2)),
                                bw=float(rng.uniform(0.2, 2)), lat=float(rng.uniform(0.5, 2)), **kw))
    sw = W.Sweep("first-bucket", tr, topos, W.points_array(pts))
    got = ctx.run_sweep(sw)
    assert (got["status"] == 0).all()
    check(got, sw, list(range(len(pts))))


@pytest.mark.parametrize("seed", range(2))
def test_chunked_ring(ctx, seed):
    """R25 pipelined rings (0-8 chunks per step) in every kernel that runs ring collectives -- warp
    segments with and without the uniform-ring fast-forward, the hybrid kernel, photonic flows and a
    64-rank CTA point -- against the oracle point by point."""
    sw = S.random_chunked(seed)
    got = ctx.run_sweep(sw)
    assert got["status"][-1] == W.PT_BAD_CONFIG
    # every point simulates (incl. HYBRID DP groups strided over the 64-ring, routes > 8 hops) but the
    # documented photonic-tree ones
    tl = expected_too_large(sw)
    assert np.flatnonzero(got["status"] == W.PT_TOO_LARGE).tolist() == tl
    assert ((got["status"] == 0).sum() + len(tl)) == len(sw.points) - 1
    check(got, sw, [i for i in range(len(sw.points)) if i not in set(tl)])


@pytest.mark.parametrize("seed", range(2))
def test_reduce_broadcast(ctx, seed):
    """R26 AllReduce as ring Reduce + ring Broadcast chains (0-6 chunks) in the warp, hybrid, photonic and
    64-rank CTA kernels, against the oracle point by point."""
    sw = S.random_redbcast(seed)
    got = ctx.run_sweep(sw)
    assert got["status"][-1] == W.PT_BAD_CONFIG
    assert (got["status"][:-1] == 0).all()
    check(got, sw, list(range(len(sw.points))))


def test_double_tree_small_and_long_routes(ctx):
    """R27 on the GPU for DDP and PAPER-mode TP on a ring, and the single tree / double tree over a 32-GPU
    ring where a child's route to its parent is up to 16 hops (past the 8 cached in registers)."""
    tr = W.mlp_trace()
    topos = [W.ring(8, 25e9, 1e-6), W.ring(32, 50e9, 1e-6)]
    pts = [W.make_point(0, W.ST_DDP, dp=8, B=64, algo=W.ALG_DBTREE),
           W.make_point(0, W.ST_DDP, dp=8, B=64, algo=W.ALG_TREE),
           W.make_point(0, W.ST_TP, tp=4, B=64, tp_mode=W.TPM_PAPER, algo=W.ALG_DBTREE),
           W.make_point(1, W.ST_DDP, dp=32, B=64, algo=W.ALG_TREE),
           W.make_point(1, W.ST_DDP, dp=32, B=64, algo=W.ALG_DBTREE),
           W.make_point(1, W.ST_TP, tp=32, B=64, algo=W.ALG_TREE, tp_mode=W.TPM_PAPER)]
    sw = W.Sweep("dbtree", tr, topos, W.points_array(pts))
    got = ctx.run_sweep(sw)
    assert (got["status"] == 0).all()
    check(got, sw, list(range(len(pts))))


@pytest.mark.parametrize("seed", range(3))
def test_reduce_scatter_all_gather(ctx, seed):
    """R29 AllReduce as ring ReduceScatter + ring AllGather (0-6 chunks) in the warp, hybrid, photonic and
    64-rank CTA kernels, against the oracle point by point."""
    sw = S.random_rsag(seed)
    got = ctx.run_sweep(sw)
    assert got["status"][-1] == W.PT_BAD_CONFIG
    assert (got["status"][:-1] == 0).all()
    check(got, sw, list(range(len(sw.points))))


@pytest.mark.parametrize("seed", range(3))
def test_double_binary_tree(ctx, seed):
    """R27 double binary tree AllReduce on the GPU (the hybrid kernel holds tree B on a spare flow slot):
    every point against the oracle.  The documented limits (include/triosim.h TRIOSIM_ALGO_DBTREE) are the
    only PT_TOO_LARGE points: HYBRID with both dp > 1 and tp > 1, and collectives over photonic links."""
    sw = S.random_dbtree(seed)
    got = ctx.run_sweep(sw)
    assert got["status"][-1] == W.PT_BAD_CONFIG
    P = sw.points[:-1]
    phot = np.array([getattr(sw.topos[int(p["topo"])], "photonic", None) is not None for p in P])
    both = (P["strategy"] == W.ST_HYBRID) & (P["dp"] > 1) & (P["tp"] > 1)
    coll = np.where(P["strategy"] == W.ST_TP, P["tp"] > 1,
                    np.where(P["strategy"] == W.ST_HYBRID, (P["dp"] > 1) | (P["tp"] > 1), P["dp"] > 1))
    expect = np.flatnonzero(both | (phot & coll))
    assert np.flatnonzero(got["status"][:-1] == W.PT_TOO_LARGE).tolist() == expect.tolist()
    ok = [i for i in range(len(P)) if i not in set(expect.tolist())]
    assert len(ok) > 100
    check(got, sw, ok)
