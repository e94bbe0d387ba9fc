"""One C4 launch of the slowest PIPE class (pp = 16) for ncu source-level profiling."""
import sys
import numpy as np
import torch
sys.path.insert(0, ".")
from paper_conf_isca_libwmvgjbj025_b200 import triosim, workloads as W

deg = int(sys.argv[1]) if len(sys.argv) > 1 else 16
ctx = triosim.Context(0)
sw = W.sweep_c4()
tid = ctx.triosim_load_trace(sw.trace)
idx = np.nonzero(sw.points["pp"] == deg)[0][:600]
sid = ctx.triosim_build_sweep(tid, sw.topos, sw.points[idx], sw.plans or None)
ctx.triosim_simulate_batch(sid, 0, len(idx))
torch.cuda.synchronize()
print("ok", len(idx))
