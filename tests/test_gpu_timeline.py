"""GPU parity of the R23 timeline (R23) against the oracle through the C ABI
(triosim_timeline): every task and flow record of sampled points of seeded random sweeps over every
strategy, collective algorithm, the one-point-per-CTA kernel and the photonic network, plus C1 and C2
points; and the recording kernel leaves the point's result record bit-identical."""
import numpy as np
import pytest

import oracle
from paper_conf_isca_libwmvgjbj025_b200 import workloads as W
from tests import sweeps as S

pytestmark = pytest.mark.gpu
RTOL = 1e-9


@pytest.fixture(scope="module")
def ctx():
    import torch
    assert torch.cuda.is_available()
    from paper_conf_isca_libwmvgjbj025_b200 import triosim
    c = triosim.Context(0)
    yield c
    c.close()


def _close(a, b):
    return np.all(np.abs(a - b) <= RTOL * np.abs(b))


def _check(ctx, sw, idx):
    tid = ctx.triosim_load_trace(sw.trace)
    sid = ctx.triosim_build_sweep(tid, sw.topos, sw.points, sw.plans or None)
    ctx.triosim_simulate_batch(sid, 0, len(sw.points))
    res = ctx.triosim_results(sid, 0, len(sw.points))
    bad, n_ok = [], 0
    for i in idx:
        tasks, flows = ctx.triosim_timeline(sid, i)
        pt = sw.points[i]
        plan = None
        if pt["stage_plan"] >= 0:
            plan = sw.plans[pt["stage_plan"]]
        r, rt, rf = oracle.run_point(sw.trace, sw.topos[pt["topo"]], pt, plan, timeline=True)
        if res[i]["status"] == W.PT_TOO_LARGE and r["status"] == 0:
            assert len(tasks) == 0 and len(flows) == 0
            continue   # a documented kernel limit (R3 / R20)
        if r["status"] != 0:
            assert len(tasks) == 0 and len(flows) == 0
            continue
        n_ok += 1
        if len(tasks) != len(rt) or len(flows) != len(rf):
            bad.append(f"point {i}: counts {len(tasks)}/{len(flows)} vs {len(rt)}/{len(rf)}")
            continue
        for f in ("gpu", "prog", "op", "mb"):
            if not np.array_equal(tasks[f], rt[f]):
                bad.append(f"point {i}: task field {f}")
        if not (_close(tasks["start_s"], rt["start_s"]) and _close(tasks["end_s"], rt["end_s"])):
            bad.append(f"point {i}: task times")
        g, o = np.sort(flows, order="code"), np.sort(rf, order="code")
        for f in ("code", "src", "dst"):
            if not np.array_equal(g[f], o[f]):
                bad.append(f"point {i}: flow field {f}")
        for f in ("bytes", "release_s", "start_s", "delivered_s"):
            if not _close(g[f], o[f]):
                bad.append(f"point {i}: flow field {f}")
        assert len(tasks) == res[i]["n_compute"] and len(flows) == res[i]["n_flows"]
    after = ctx.triosim_results(sid, 0, len(sw.points))
    assert after.tobytes() == res.tobytes()   # the recording run reproduces every result bit
    ctx.triosim_release(sid)
    ctx.triosim_release(tid)
    assert not bad, "\n".join(bad[:20])
    return n_ok


def _sample(n, k, seed):
    rng = np.random.Generator(np.random.PCG64(seed))
    return sorted(rng.choice(n, size=min(k, n), replace=False).tolist())


@pytest.mark.parametrize("gen,seed", [(S.random_small, 0), (S.random_small, 1), (S.random_hybrid, 0),
                                      (S.random_photonic, 0), (S.random_photonic, 1), (S.random_chunked, 0),
                                      (S.random_redbcast, 0)])
def test_timeline_random_sweeps(ctx, gen, seed):
    sw = gen(seed)
    assert _check(ctx, sw, _sample(len(sw.points), 40, 70 + seed)) > 15


def test_timeline_large_points_cta_kernel(ctx):
    sw = S.large_points(0)
    assert _check(ctx, sw, [0, 2, 4, 8]) == 4


def test_timeline_c1_and_c2(ctx):
    assert _check(ctx, W.sweep_c1(), [0, 1]) == 2
    sw = W.sweep_c2()
    assert _check(ctx, sw, _sample(len(sw.points), 6, 5)) == 6


def test_timeline_capacity_and_errors(ctx):
    sw = W.sweep_c1()
    tid = ctx.triosim_load_trace(sw.trace)
    sid = ctx.triosim_build_sweep(tid, sw.topos, sw.points)
    full_t, full_f = ctx.triosim_timeline(sid, 0)
    import ctypes as C
    nt, nf = C.c_uint64(), C.c_uint64()
    small = np.zeros(3, W.TASK_REC_DTYPE)
    st = ctx.L.triosim_timeline(ctx.h, sid, 0, small.ctypes.data_as(C.c_void_p), 3, None, 0, C.byref(nt), C.byref(nf))
    assert st == 0 and nt.value == len(full_t) and nf.value == len(full_f)
    with pytest.raises(Exception):
        ctx.triosim_timeline(sid, 99)
    ctx.triosim_release(sid)
    ctx.triosim_release(tid)
