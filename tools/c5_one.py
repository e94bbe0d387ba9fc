"""Time single configs[4] points of a given simulated-GPU count N (probe)."""
import sys
import time

import numpy as np

sys.path.insert(0, ".")
from paper_conf_isca_libwmvgjbj025_b200 import triosim, workloads as W  # noqa: E402

Nw = int(sys.argv[1])
k = int(sys.argv[2]) if len(sys.argv) > 2 else 1
full = W.sweep_c5(Ns=(Nw,), n_bw=2, n_lat=1)
N = full.points["dp"].astype(int) * full.points["tp"] * full.points["pp"]
idx = np.flatnonzero((N == Nw) & (full.points["microbatches"] == 8))[:k]
sw = W.Sweep(full.name, full.trace, full.topos, full.points[idx])
ctx = triosim.Context(0)
tid = ctx.triosim_load_trace(sw.trace)
sid = ctx.triosim_build_sweep(tid, sw.topos, sw.points)
import torch  # noqa: E402
torch.cuda.synchronize()
t0 = time.time()
ctx.triosim_simulate_batch(sid, 0, len(idx))
got = ctx.triosim_results(sid, 0, len(idx))
dt = time.time() - t0
print(f"N={Nw}: {len(idx)} points in {dt:.3f} s", got[["status", "n_instants", "n_flows"]].tolist(),
      f"us/instant={dt / max(1, got['n_instants'].max()) * 1e6:.2f}", flush=True)
