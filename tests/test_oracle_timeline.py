"""Oracle pins for the R23 timeline ("it shows the timeline of the communication process among GPUs
or the computation process on each GPU"; "a detailed timeline trace"): every compute task and every
flow with its times, checked against closed forms (single-GPU left fold, ring AllReduce steps, the GPipe
schedule of Fig. 4) and against the independently pinned result record (counts, makespan, busy times)."""
import numpy as np
import pytest

import oracle
from paper_conf_isca_libwmvgjbj025_b200 import workloads as W
from tests import sweeps as S
from tests.helpers import one_wgrad_trace, rel
from tests.test_oracle_closed_forms import gpipe_trace


@pytest.mark.parametrize("mk", [W.mlp_trace, W.resnet50_trace])
def test_single_gpu_tasks_are_the_left_fold_of_trace_times(mk):
    """DP on 1 GPU at b0 runs the trace itself: op k starts where op k-1 ends, ends start + t_k."""
    tr = mk()
    r, tasks, flows = oracle.run_point(tr, W.ring(2), W.make_point(0, W.ST_DDP, dp=1, B=tr.trace_batch),
                                       timeline=True)
    assert r["status"] == 0 and len(flows) == 0 and len(tasks) == len(tr.ops)
    assert (tasks["gpu"] == 0).all() and (tasks["prog"] == np.arange(len(tr.ops))).all()
    assert (tasks["op"] == np.arange(len(tr.ops))).all() and (tasks["mb"] == 0).all()
    t = 0.0
    for k, rec in enumerate(tasks):
        assert rec["start_s"] == t
        t = t + float(tr.ops["time_s"][k])
        assert rec["end_s"] == t
    assert tasks["end_s"][-1] == r["iter_time_s"]


@pytest.mark.parametrize("p", [2, 3, 4, 8])
def test_ring_allreduce_step_times(p):
    """Ring AllReduce on a uniform ring (CF5): step k of every member is released at
    t_fb + k(a + S/(pB)), activates a later (Q19) and is delivered S/(pB) after that."""
    Sz, B, a = 100e6, 50e9, 2e-6
    tr = one_wgrad_trace(int(Sz))
    r, tasks, flows = oracle.run_point(tr, W.ring(p, bw=B, lat=a), W.make_point(0, W.ST_DP, dp=p, B=p),
                                       timeline=True)
    assert r["status"] == 0 and len(flows) == 2 * (p - 1) * p == r["n_flows"]
    t_fb = 2.0 ** -10 + 2.0 ** -9
    step = (flows["code"] >> 16) & 0xFFFF
    member = flows["code"] & 0xFFFF
    for k in range(2 * (p - 1)):
        f = flows[step == k]
        assert len(f) == p and sorted(member[step == k]) == list(range(p))
        rel0 = t_fb + k * (a + Sz / (p * B))
        assert np.all(np.abs(f["release_s"] - rel0) <= 1e-12 * rel0)
        assert np.all(np.abs(f["start_s"] - (f["release_s"] + a)) <= 1e-12 * rel0)
        assert np.all(np.abs(f["delivered_s"] - (f["start_s"] + Sz / (p * B))) <= 1e-12 * rel0)
        assert (f["bytes"] == Sz / p).all()
        assert ((f["dst"].astype(np.int64) - f["src"].astype(np.int64)) % p == 1).all()   # m_i -> m_(i+1)


@pytest.mark.parametrize("p,m", [(2, 2), (4, 8), (3, 5)])
def test_gpipe_forward_schedule(p, m):
    """GPipe (Fig. 4) with uniform stages and c = a + A/B <= t_f: the forward of micro-batch j
    on stage s starts at j t_f + s (t_f + c); each activation send is released at the end of its forward
    and delivered c later."""
    t_f, t_b, t_opt = 2.0 ** -10, 2.0 ** -9, 2.0 ** -12
    A, B, a = 2 ** 20, 2.0 ** 32, 2.0 ** -16
    tr = gpipe_trace(p, t_f, t_b, t_opt, A)
    r, tasks, flows = oracle.run_point(tr, W.ring(p, bw=B, lat=a), W.make_point(0, W.ST_PP, pp=p, m=m, B=m),
                                       timeline=True)
    assert r["status"] == 0
    c = a + A / B
    fwd = tasks[tr.ops["phase"][tasks["op"]] == W.PH_FWD]
    assert len(fwd) == p * m
    for rec in fwd:
        s, j = int(rec["gpu"]), int(rec["mb"])
        exp = j * t_f + s * (t_f + c)
        assert rel(rec["start_s"], exp) < 1e-12 and rel(rec["end_s"], exp + t_f) < 1e-12
    act = flows[(flows["dst"] == flows["src"] + 1)]
    assert len(act) == (p - 1) * m and (act["code"] >> 59 == 1).all()
    for f in act:
        j = int((f["code"] >> 16) & 0xFFFF)
        s = int(f["src"])
        assert rel(f["release_s"], j * t_f + s * (t_f + c) + t_f) < 1e-12
        assert rel(f["delivered_s"], f["release_s"] + c) < 1e-12


def _union(iv):
    tot, cur_s, cur_e = 0.0, None, None
    for s, e in sorted(iv):
        if cur_e is None or s > cur_e:
            if cur_e is not None:
                tot += cur_e - cur_s
            cur_s, cur_e = s, e
        else:
            cur_e = max(cur_e, e)
    if cur_e is not None:
        tot += cur_e - cur_s
    return tot


@pytest.mark.parametrize("gen,seed", [(S.random_small, 0), (S.random_hybrid, 1), (S.random_photonic, 2)])
def test_timeline_agrees_with_the_result_record(gen, seed):
    """On random sweeps over every strategy, collective and both network models: record counts equal the
    result's counts; tasks of a GPU run in program order without overlap; every flow is released, then
    starts, then is delivered; the makespan is the last task end or delivery; comm_busy is the measure of
    the union of [release, delivery] (R18) and compute_busy_max the largest per-GPU task-time sum."""
    sw = gen(seed)
    checked = 0
    for i in range(0, len(sw.points), 7):
        pt = sw.points[i]
        r, tasks, flows = oracle.run_point(sw.trace, sw.topos[pt["topo"]], pt, timeline=True)
        if r["status"] != 0:
            assert len(tasks) == 0 and len(flows) == 0
            continue
        checked += 1
        assert len(tasks) == r["n_compute"] and len(flows) == r["n_flows"]
        assert int((flows["code"] >> 59 == 1).sum()) == r["n_p2p"]
        assert len(np.unique(flows["code"])) == len(flows)
        for g in np.unique(tasks["gpu"]):
            tg = tasks[tasks["gpu"] == g]
            assert (np.diff(tg["prog"].astype(np.int64)) > 0).all()
            assert (tg["start_s"][1:] >= tg["end_s"][:-1]).all()
        assert (tasks["end_s"] >= tasks["start_s"]).all()
        assert (flows["start_s"] >= flows["release_s"]).all() and (flows["delivered_s"] >= flows["start_s"]).all()
        assert (np.diff(flows["release_s"]) >= 0).all()
        last = max(tasks["end_s"].max(initial=0.0), flows["delivered_s"].max(initial=0.0))
        assert last == r["iter_time_s"]
        cb = _union(list(zip(flows["release_s"].tolist(), flows["delivered_s"].tolist())))
        assert abs(cb - r["comm_busy_s"]) <= 1e-12 * max(r["comm_busy_s"], 1e-30) + 1e-18
        # end - start = t' up to the rounding of the late time stamps (one ulp of the makespan per task)
        busy = max(float((tasks["end_s"] - tasks["start_s"])[tasks["gpu"] == g].sum()) for g in np.unique(tasks["gpu"]))
        tol = 2 * len(tasks) * float(np.spacing(r["iter_time_s"])) + 1e-12 * r["compute_busy_max_s"]
        assert abs(busy - r["compute_busy_max_s"]) <= tol
    assert checked > 20
