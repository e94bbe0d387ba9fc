"""Where the end-to-end step's time goes: load_trace / build_sweep / simulate / results / release (probe)."""
import sys
import time
import numpy as np
import torch
sys.path.insert(0, ".")
from paper_conf_isca_libwmvgjbj025_b200 import triosim, workloads as W

ctx = triosim.Context(0)
sw = W.sweep_c2()
n = len(sw.points)
out = torch.empty(n * W.RESULT_DTYPE.itemsize, dtype=torch.uint8).pin_memory().numpy().view(W.RESULT_DTYPE)
rows = []
for i in range(6):
    torch.cuda.synchronize()
    t = [time.perf_counter()]
    tid = ctx.triosim_load_trace(sw.trace); t.append(time.perf_counter())
    sid = ctx.triosim_build_sweep(tid, sw.topos, sw.points); t.append(time.perf_counter())
    ctx.triosim_simulate_batch(sid, 0, n); t.append(time.perf_counter())
    ctx.triosim_results(sid, 0, n, out=out); t.append(time.perf_counter())
    ctx.triosim_release(sid); ctx.triosim_release(tid); t.append(time.perf_counter())
    rows.append(np.diff(t) * 1e3)
print("ms load / build / simulate(enqueue) / results(sync) / release:", np.round(np.median(rows[1:], axis=0), 3))
