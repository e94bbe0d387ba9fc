"""configs[4] at full scale (64-1024 simulated GPUs): time a seeded prefix of the sweep on the GPU and
compare a few points with the oracle (probe, not a test)."""
import sys
import time

import numpy as np

sys.path.insert(0, ".")
import oracle  # noqa: E402
from paper_conf_isca_libwmvgjbj025_b200 import triosim, workloads as W  # noqa: E402
from tests.parity import compare  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 300
full = W.sweep_c5()
sw = W.Sweep(full.name, full.trace, full.topos, full.points[:n])
ctx = triosim.Context(0)
tid = ctx.triosim_load_trace(sw.trace)
sid = ctx.triosim_build_sweep(tid, sw.topos, sw.points)
import torch  # noqa: E402
for rep in range(2):
    torch.cuda.synchronize()
    t0 = time.time()
    ctx.triosim_simulate_batch(sid, 0, n)
    got = ctx.triosim_results(sid, 0, n)
    print(f"rep {rep}: {n} points in {time.time() - t0:.2f} s", flush=True)
print("status", np.unique(got["status"], return_counts=True))
N = sw.points["dp"].astype(int) * sw.points["tp"] * sw.points["pp"]
for k in np.unique(N):
    s = N == k
    print(k, s.sum(), "instants mean", got["n_instants"][s].mean(), "max", got["n_instants"][s].max(), flush=True)
idx = [int(np.flatnonzero(N == k)[0]) for k in np.unique(N)]
t0 = time.time()
ref = oracle.run_sweep(sw, idx)
print("oracle", len(idx), "points", time.time() - t0, "s")
bad, ulp = compare(got[idx], ref, idx)
print("mismatches", len(bad), bad[:10], "ulp", ulp)
