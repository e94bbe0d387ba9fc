"""configs[4] stratified parity subset on the GPU, one N at a time: K3 phase time of the group (all its
points run concurrently, one CTA each) and each point's instants (probe).   python tools/c5_subset.py [N ...]"""
import sys
import time

import numpy as np
import torch

sys.path.insert(0, ".")
from paper_conf_isca_libwmvgjbj025_b200 import triosim, workloads as W  # noqa: E402

sw = W.sweep_c5_parity()
P = sw.points
N = P["dp"].astype(np.int64) * P["tp"] * P["pp"]
ctx = triosim.Context(0)
tid = ctx.triosim_load_trace(sw.trace)
for n in [int(x) for x in sys.argv[1:]] or sorted(set(N.tolist())):
    idx = np.flatnonzero(N == n)
    sid = ctx.triosim_build_sweep(tid, sw.topos, P[idx])
    torch.cuda.synchronize()
    ctx.timing(True)
    t0 = time.time()
    ctx.triosim_simulate_batch(sid, 0, len(idx))
    r = ctx.triosim_results(sid, 0, len(idx))
    wall = time.time() - t0
    tot, k3 = ctx.timings()
    ctx.timing(False)
    inst = r["n_instants"].astype(np.int64)
    print(f"N={n}: {len(idx)} points, K3 {float(np.mean(k3)):.1f} ms (wall {wall:.1f} s), status {np.unique(r['status'])}, "
          f"instants max {inst.max()} sum {inst.sum()}, us/instant of the longest {1e3 * float(np.mean(k3)) / max(1, inst.max()):.2f}",
          flush=True)
    np.save(f"gpurun_out/c5sub_N{n}.npy", r)
    ctx.triosim_release(sid)
