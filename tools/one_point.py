"""Time (and, under ncu, profile) ONE design point of a config alone: its K3 phase latency and per-instant /
per-round cost (probe).   python tools/one_point.py <c2|c3|c4|c5> <index|heaviest> [repeats]
c5 draws from the stratified bench subset (W.sweep_c5 with N in argv[4] if given)."""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
from paper_conf_isca_libwmvgjbj025_b200 import triosim, workloads as W  # noqa: E402

cfg, which = sys.argv[1], sys.argv[2]
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
if cfg == "c5":
    Ns = (int(sys.argv[4]),) if len(sys.argv) > 4 else (64,)
    full = W.sweep_c5(Ns=Ns, n_bw=2, n_lat=1)
else:
    full = {"c2": W.sweep_c2, "c3": W.sweep_c3, "c4": W.sweep_c4}[cfg]()
ctx = triosim.Context(0)
tid = ctx.triosim_load_trace(full.trace)
if which == "heaviest" and cfg != "c5":
    sid = ctx.triosim_build_sweep(tid, full.topos, full.points, full.plans or None)
    ctx.triosim_simulate_batch(sid, 0, len(full.points))
    r = ctx.triosim_results(sid, 0, len(full.points))
    i = int(np.argmax(r["n_instants"].astype(np.int64) * 4 + r["n_wf_rounds"].astype(np.int64)))
    ctx.triosim_release(sid)
else:
    i = int(which) if which != "heaviest" else 0
one = ctx.triosim_build_sweep(tid, full.topos, full.points[i:i + 1], full.plans or None)
ctx.triosim_simulate_batch(one, 0, 1)
torch.cuda.synchronize()
ctx.timing(True)
for _ in range(reps):
    ctx.triosim_simulate_batch(one, 0, 1)
tot, k3 = ctx.timings()
ctx.timing(False)
r = ctx.triosim_results(one, 0, 1)[0]
k3m = float(np.mean(k3))
print(f"{cfg} point {i} topo {full.topos[int(full.points[i]['topo'])].name} pt {full.points[i]} status {int(r['status'])} "
      f"instants {int(r['n_instants'])} wf_calls {int(r['n_wf_calls'])} rounds {int(r['n_wf_rounds'])} "
      f"flows {int(r['n_flows'])} tasks {int(r['n_compute'])} k3 {k3m:.3f} ms "
      f"ns/instant {1e6 * k3m / max(1, int(r['n_instants'])):.1f}", flush=True)
