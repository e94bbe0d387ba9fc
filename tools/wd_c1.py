"""Debug: run C1 and a small random sweep through the library (set TRIOSIM_LIB to a watchdog build)."""
import sys
sys.path.insert(0, ".")
import numpy as np
import torch
from paper_conf_isca_libwmvgjbj025_b200 import triosim, workloads as W
from tests import sweeps as S
ctx = triosim.Context(0)
for sw in (W.sweep_c1(), S.random_small(0)):
    r = ctx.run_sweep(sw)
    torch.cuda.synchronize()
    print(sw.name, r["status"][:8], r["iter_time_s"][:4], flush=True)
