"""Run the configs[4] test subset point by point, report time / instants, to find pathological points."""
import sys
import time
import numpy as np
sys.path.insert(0, ".")
from paper_conf_isca_libwmvgjbj025_b200 import triosim, workloads as W

full = W.sweep_c5()
rng = np.random.Generator(np.random.PCG64(55))
sub = sorted(rng.choice(len(full.points), size=300, replace=False).tolist())
ctx = triosim.Context(0)
tid = ctx.triosim_load_trace(full.trace)
rows = []
t_all = time.time()
for k, i in enumerate(sub):
    pts = full.points[[i]]
    sid = ctx.triosim_build_sweep(tid, full.topos, pts)
    t0 = time.time()
    ctx.triosim_simulate_batch(sid, 0, 1)
    r = ctx.triosim_results(sid, 0, 1)
    dt = time.time() - t0
    p = pts[0]
    rows.append((dt, int(p['dp']), int(p['tp']), int(p['pp']), int(p['microbatches']), int(r['n_instants'][0]), int(r['status'][0])))
    ctx.triosim_release(sid)
    if time.time() - t_all > 200:
        print("stopping after", k + 1, "points")
        break
rows.sort(reverse=True)
print("total", sum(r[0] for r in rows), "s over", len(rows))
for r in rows[:10]:
    print(r)
