"""K3 latency vs load: sweeps made only of one C2 class (per-tensor DDP, p given), growing counts."""
import sys
import numpy as np
import torch
sys.path.insert(0, ".")
from paper_conf_isca_libwmvgjbj025_b200 import triosim, workloads as W

p = int(sys.argv[1]) if len(sys.argv) > 1 else 16
bucket = int(sys.argv[2]) if len(sys.argv) > 2 else 0
tr = W.resnet50_trace()
ctx = triosim.Context(0)
tid = ctx.triosim_load_trace(tr)
rng = np.random.Generator(np.random.PCG64(0))
for n in ([int(sys.argv[3])] if len(sys.argv) > 3 else (1, 2, 16, 148, 296, 592, 1250, 2500)):
    pts = W.points_array([W.make_point(0, W.ST_DDP, dp=p, B=p * 64, bucket=bucket, bw=float(rng.uniform(10e9, 900e9)),
                                       lat=float(rng.uniform(0.5e-6, 20e-6))) for _ in range(n)])
    sid = ctx.triosim_build_sweep(tid, [W.ring(p)], pts)
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
    print(f"p={p} n={n:5d} k3={np.mean(k3):8.3f} ms  instants/pt={inst:7.0f}  us/instant={1e3*np.mean(k3)/inst:6.3f}  "
          f"pts/s={n/np.mean(k3)*1e3:10.0f}", flush=True)
    ctx.triosim_release(sid)
