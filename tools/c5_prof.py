"""Phase profile of the hybrid CTA kernel on configs[4] points (TS_PROF_H build: per point, thread 0 prints
cycles per phase of an instant; a point stops after TS_PROF_H instants).
    TRIOSIM_LIB=.../libtriosim_prof.so python tools/c5_prof.py [N ...]"""
import sys

import numpy as np

sys.path.insert(0, ".")
from paper_conf_isca_libwmvgjbj025_b200 import triosim, workloads as W  # noqa: E402

sw = W.sweep_c5_parity()
P = sw.points
N = P["dp"].astype(np.int64) * P["tp"] * P["pp"]
sel = []
for n in [int(x) for x in sys.argv[1:]] or sorted(set(N.tolist())):
    idx = np.flatnonzero(N == n)
    heavy = idx[np.argsort(-(P["dp"][idx].astype(np.int64) * P["tp"][idx]))][:3]
    sel += heavy.tolist() + idx[:2].tolist()
sel = sorted(set(sel))
for i in sel:
    print("point", i, "N", N[i], "dp", P["dp"][i], "tp", P["tp"][i], "pp", P["pp"][i], "m", P["microbatches"][i], "topo", P["topo"][i], flush=True)
ctx = triosim.Context(0)
tid = ctx.triosim_load_trace(sw.trace)
sid = ctx.triosim_build_sweep(tid, sw.topos, P[sel])
ctx.triosim_simulate_batch(sid, 0, len(sel))
r = ctx.triosim_results(sid, 0, len(sel))
print("done", r["n_instants"].tolist(), flush=True)
