"""K3 latency vs throughput per structural group of the C3 / C4 sweeps: for each degree, one point
alone (latency) and the whole group (throughput), with instants per point."""
import sys
import numpy as np
import torch
sys.path.insert(0, ".")
from paper_conf_isca_libwmvgjbj025_b200 import triosim, workloads as W

ctx = triosim.Context(0)
for cfg in sys.argv[1:] or ["c3", "c4"]:
    sw = {"c3": W.sweep_c3, "c4": W.sweep_c4}[cfg]()
    tid = ctx.triosim_load_trace(sw.trace)
    key = sw.points["tp"] if cfg == "c3" else sw.points["pp"]
    for k in np.unique(key):
        idx = np.nonzero(key == k)[0]
        for n in (1, len(idx)):
            pts = sw.points[idx[:n]]
            sid = ctx.triosim_build_sweep(tid, sw.topos, pts, sw.plans or None)
            for _ in range(2):
                ctx.triosim_simulate_batch(sid, 0, n)
            torch.cuda.synchronize()
            ctx.timing(True)
            for _ in range(3):
                ctx.triosim_simulate_batch(sid, 0, n)
            tot, k3 = ctx.timings()
            ctx.timing(False)
            r = ctx.triosim_results(sid, 0, n)
            inst = float(r["n_instants"].mean())
            print(f"{cfg} deg={k} n={n:5d} k3={np.mean(k3):8.3f} ms instants/pt={inst:8.0f} wf_rounds/pt={float(r['n_wf_rounds'].mean()):8.0f} "
                  f"us/instant={1e3 * np.mean(k3) / inst:6.3f} pts/s={n / np.mean(k3) * 1e3:10.0f}", flush=True)
            ctx.triosim_release(sid)
    ctx.triosim_release(tid)
