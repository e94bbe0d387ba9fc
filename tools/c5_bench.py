"""configs[4] bench line on the declared stratified subset (W.sweep_c5_parity: 100 GPT-3-class DP x TP x PP points,
20 per N in {64, 128, 256, 512, 1024} simulated GPUs, incl. the heaviest dp x tp = 64 classes on the perturbed
4:1 topologies).  One step = one simulate_batch over the 100 points (each runs on its own CTA, all concurrently,
so the step is the slowest point's latency); a step takes minutes, so this line times ONE step after no warm-up
(declared in the line) -- bench.py's W >= 3 protocol would take most of an hour.  Prints one JSON line with
points/s, the per-N instants and the per-instant latency of each N's slowest point, clocks, and the fp64
roofline of SURVEY 8(d) (2 ops per operator instance + 80 per water-filling call).

    python tools/c5_bench.py [--points K]      (K: a seeded subset of the 100, for quick checks)
"""
import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402
from paper_conf_isca_libwmvgjbj025_b200 import workloads as W  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--points", type=int, default=0)
    args = ap.parse_args()
    import torch
    from paper_conf_isca_libwmvgjbj025_b200 import triosim

    sw = W.sweep_c5_parity()
    if args.points:
        sel = np.sort(np.random.default_rng(5).choice(len(sw.points), args.points, replace=False))
        sw = W.Sweep(sw.name, sw.trace, sw.topos, sw.points[sel], sw.plans)
    P = sw.points
    n = len(P)
    N = P["dp"].astype(np.int64) * P["tp"] * P["pp"]
    ctx = triosim.Context(0)
    tid = ctx.triosim_load_trace(sw.trace)
    sid = ctx.triosim_build_sweep(tid, sw.topos, P, sw.plans or None)
    stream = torch.cuda.Stream()
    res_d = torch.zeros(n * W.RESULT_DTYPE.itemsize, dtype=torch.uint8, device="cuda")
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ctx.timing(True)
    t0 = time.time()
    with bench.Clocks(0) as clk:
        e0.record(stream)
        ctx.triosim_simulate_batch(sid, 0, n, stream.cuda_stream)
        ctx.triosim_results(sid, 0, n, device_ptr=res_d.data_ptr(), stream=stream.cuda_stream)
        e1.record(stream)
        torch.cuda.synchronize()
    wall = time.time() - t0
    ms = e0.elapsed_time(e1)
    _, k3 = ctx.timings()
    ctx.timing(False)
    r = res_d.cpu().numpy().view(W.RESULT_DTYPE)
    per_n = {}
    for v in sorted(set(N.tolist())):
        k = np.flatnonzero(N == v)
        inst = r["n_instants"][k].astype(np.int64)
        per_n[str(v)] = {"points": int(len(k)), "instants_max": int(inst.max()), "instants_sum": int(inst.sum()),
                         "rounds_sum": int(r["n_wf_rounds"][k].astype(np.int64).sum())}
    alg = bench.algorithmic_fp64(r)
    pk, src = bench.peaks()
    clock = float(pk.get("sm_max_mhz", 1965.0))
    peak = bench.N_SMS * bench.FP64_LANES_PER_SM * clock * 1e6
    k3_ms = float(np.mean(k3)) if len(k3) else ms
    out = {"metric": bench.METRIC, "value": round(n / (ms / 1e3), 4), "unit": bench.UNIT, "n_gpus": 1, "steps": 1,
           "warmup": 0, "ms_per_step": round(ms, 1), "higher_is_better": True, "vs_baseline": None, "dtype": "f64",
           "data": "synthetic", "scaling": "weak",
           "config": {"workload": bench.WORKLOAD["c5_subset"], "points": n, "points_ok": int((r["status"] == 0).sum()),
                      "timing": "one device-timed simulate_batch of the whole subset, no warm-up (a step is minutes)",
                      "per_N": per_n},
           "slowest_point_us_per_instant": round(1e3 * ms / max(1, int(r["n_instants"].max())), 3),
           "roofline": {"bound": "alu", "achieved": round(alg / (k3_ms / 1e3) / 1e12, 6), "peak": round(peak / 1e12, 3),
                        "unit": "TFLOP/s (fp64, non-tensor)", "frac": round(alg / (k3_ms / 1e3) / peak, 7),
                        "alg_fp64_ops": int(alg), "k3_ms": round(k3_ms, 1),
                        "alg_derivation": "SURVEY 8(d).2: 2 x n_compute + 80 x n_wf_calls over the subset / K3 time"},
           "clocks": clk.summary(), "wall_s": round(wall, 1), "status_counts": np.bincount(r["status"]).tolist()}
    print(json.dumps(out), flush=True)
    np.save(os.path.join(ROOT, "gpurun_out", "c5_bench_records.npy"), r)
    ctx.close()


if __name__ == "__main__":
    main()
