"""One configs[4] point (index from argv) simulated alone, for ncu."""
import sys
sys.path.insert(0, ".")
from paper_conf_isca_libwmvgjbj025_b200 import triosim, workloads as W
sw = W.sweep_c5()
want = tuple(int(x) for x in sys.argv[1:5])  # dp tp pp m
idx = [i for i, p in enumerate(sw.points) if (p["dp"], p["tp"], p["pp"], p["microbatches"]) == want][0]
ctx = triosim.Context(0)
tid = ctx.triosim_load_trace(sw.trace)
sid = ctx.triosim_build_sweep(tid, sw.topos, sw.points[[idx]])
for _ in range(2):
    ctx.triosim_simulate_batch(sid, 0, 1)
print(ctx.triosim_results(sid, 0, 1)[["n_instants", "status"]])
