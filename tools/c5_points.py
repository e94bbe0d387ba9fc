"""Run chosen configs[4] parity-sample points (indices into W.sweep_c5_parity) in one simulate_batch -- for ncu
captures of the CTA kernel with a TS_PROF_H build (each point stops after TS_PROF_H instants).
    TRIOSIM_LIB=... python tools/c5_points.py 28 [48 ...]"""
import sys

import numpy as np

sys.path.insert(0, ".")
from paper_conf_isca_libwmvgjbj025_b200 import triosim, workloads as W  # noqa: E402

sw = W.sweep_c5_parity()
sel = [int(x) for x in sys.argv[1:]]
ctx = triosim.Context(0)
tid = ctx.triosim_load_trace(sw.trace)
sid = ctx.triosim_build_sweep(tid, sw.topos, sw.points[sel])
ctx.triosim_simulate_batch(sid, 0, len(sel))
r = ctx.triosim_results(sid, 0, len(sel))
print("instants", r["n_instants"].tolist(), "rounds", r["n_wf_rounds"].tolist(), flush=True)
