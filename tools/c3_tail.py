"""C3 tail: the heaviest tp=8 points by instants / water-filling rounds, each timed alone (probe)."""
import sys
import numpy as np
import torch
sys.path.insert(0, ".")
from paper_conf_isca_libwmvgjbj025_b200 import triosim, workloads as W

ctx = triosim.Context(0)
sw = W.sweep_c3()
tid = ctx.triosim_load_trace(sw.trace)
sid = ctx.triosim_build_sweep(tid, sw.topos, sw.points)
ctx.triosim_simulate_batch(sid, 0, len(sw.points))
r = ctx.triosim_results(sid, 0, len(sw.points))
order = np.argsort(-r["n_wf_rounds"].astype(np.int64))
print("instants pctl", np.percentile(r["n_instants"], [50, 90, 99, 100]), "rounds pctl",
      np.percentile(r["n_wf_rounds"], [50, 90, 99, 100]))
for i in order[:8]:
    pt = sw.points[i]
    one = ctx.triosim_build_sweep(tid, sw.topos, sw.points[i:i + 1])
    ctx.triosim_simulate_batch(one, 0, 1)
    torch.cuda.synchronize()
    ctx.timing(True)
    for _ in range(3):
        ctx.triosim_simulate_batch(one, 0, 1)
    tot, k3 = ctx.timings()
    ctx.timing(False)
    print(int(i), "topo", sw.topos[int(pt["topo"])].name, "tp", int(pt["tp"]), "mode", int(pt["tp_mode"]),
          "algo", int(pt["coll_algo"]), "inst", int(r["n_instants"][i]), "rounds", int(r["n_wf_rounds"][i]),
          "maxact", int(r["max_active_flows"][i]), f"k3 {np.mean(k3):.3f} ms", flush=True)
    ctx.triosim_release(one)
