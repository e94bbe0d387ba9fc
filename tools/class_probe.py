"""Latency vs throughput per point group: for a config, time each (strategy degree, topology) group as its
own sweep, and its single most expensive-looking point alone.  Usage: python tools/class_probe.py c3"""
import sys
from collections import defaultdict
sys.path.insert(0, ".")
import numpy as np
import torch
from paper_conf_isca_libwmvgjbj025_b200 import triosim, workloads as W

CFG = {"c2": W.sweep_c2, "c3": W.sweep_c3, "c4": W.sweep_c4}
sw = CFG[sys.argv[1]]()
ctx = triosim.Context(0)
tid = ctx.triosim_load_trace(sw.trace)


def timed(pts, reps=3):
    sid = ctx.triosim_build_sweep(tid, sw.topos, pts, sw.plans or None)
    ctx.triosim_simulate_batch(sid, 0, len(pts))
    torch.cuda.synchronize()
    ctx.timing(True)
    for _ in range(reps):
        ctx.triosim_simulate_batch(sid, 0, len(pts))
    _, k3 = ctx.timings()
    ctx.timing(False)
    r = ctx.triosim_results(sid, 0, len(pts))
    ctx.triosim_release(sid)
    return float(np.median(k3)), r


ms_all, r_all = timed(sw.points)
print(f"whole sweep: {len(sw.points)} points  k3 {ms_all:.3f} ms  instants/pt mean {r_all['n_instants'].mean():.0f} "
      f"max {r_all['n_instants'].max()}", flush=True)
groups = defaultdict(list)
for i, p in enumerate(sw.points):
    groups[(int(p["strategy"]), int(p["dp"]), int(p["tp"]), int(p["pp"]), int(p["microbatches"]), int(p["topo"]))].append(i)
rows = []
for k, idx in groups.items():
    ms, r = timed(sw.points[idx])
    j = idx[int(np.argmax(r["n_instants"]))]
    ms1, r1 = timed(sw.points[[j]])
    rows.append((ms, k, len(idx), ms1, int(r1["n_instants"][0]), float(r["n_wf_rounds"].sum() / max(r["n_wf_calls"].sum(), 1))))
rows.sort(reverse=True)
for ms, k, n, ms1, ni, rpc in rows[:25]:
    print(f"group {k} n={n:5d} k3={ms:8.3f} ms   heaviest alone {ms1:8.3f} ms  instants {ni:7d}  us/inst {1e3*ms1/ni:6.3f}  "
          f"rounds/call {rpc:5.2f}", flush=True)
