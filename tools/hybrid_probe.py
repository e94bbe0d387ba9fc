"""Per-instant latency of K3-hybrid on single configs[4] points (and small groups of them)."""
import sys
import time
import numpy as np
import torch
sys.path.insert(0, ".")
from paper_conf_isca_libwmvgjbj025_b200 import triosim, workloads as W

sw = W.sweep_c5()
ctx = triosim.Context(0)
tid = ctx.triosim_load_trace(sw.trace)
rng = np.random.Generator(np.random.PCG64(5))
for i in rng.choice(len(sw.points), int(sys.argv[1]) if len(sys.argv) > 1 else 6, replace=False):
    pts = sw.points[[i]]
    sid = ctx.triosim_build_sweep(tid, sw.topos, pts)
    t0 = time.time()
    ctx.triosim_simulate_batch(sid, 0, 1)
    r = ctx.triosim_results(sid, 0, 1)
    dt = time.time() - t0
    p = pts[0]
    print(f"dp={p['dp']} tp={p['tp']} pp={p['pp']} m={p['microbatches']} status={r['status'][0]} "
          f"instants={r['n_instants'][0]} wall={dt:.3f}s us/instant={1e6 * dt / max(r['n_instants'][0], 1):.2f}",
          flush=True)
    ctx.triosim_release(sid)
