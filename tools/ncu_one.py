"""One simulate_batch over a config's sweep (bench.py's launch configuration, no warm-up), for ncu captures of
exactly one step's K1/K2/K3 launches.   python tools/ncu_one.py <cfg> [points]"""
import sys

import numpy as np

sys.path.insert(0, ".")
import bench  # noqa: E402
from paper_conf_isca_libwmvgjbj025_b200 import triosim  # noqa: E402

cfg = sys.argv[1]
sw = bench.make_sweep(cfg, 1, int(sys.argv[2]) if len(sys.argv) > 2 else 0)
ctx = triosim.Context(0)
tid = ctx.triosim_load_trace(sw.trace)
sid = ctx.triosim_build_sweep(tid, sw.topos, sw.points, sw.plans or None)
ctx.triosim_simulate_batch(sid, 0, len(sw.points))
r = ctx.triosim_results(sid, 0, len(sw.points))
print(cfg, len(r), np.bincount(r["status"]).tolist(), "instants", int(r["n_instants"].astype(np.int64).sum()))
ctx.close()
