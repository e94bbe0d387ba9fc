#!/usr/bin/env python
"""Benchmark: simulated design points / s on B200 (BASELINE.json metric), configs[1] workload
(ResNet-50 DP/DDP sweep, 10,000 points, 2-16 simulated GPUs on an NVLink-style ring).

One step = one pass of the whole hot path over the sweep: K1b operator rescale + K2 task-graph
expansion for every structural class + K3 timeline for every point, results written to device
memory (and all-gathered over NCCL when N > 1).  Inputs are resident in HBM (built once).

    python bench.py [--gpus N --steps K --warmup W] [--impl reference]

Under torchrun each rank simulates its own full sweep (weak scaling) and the per-point records are
gathered with one NCCL all_gather per step.  Rank 0 prints one JSON line.
"""
from __future__ import annotations

import argparse
import json
import multiprocessing as mp
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

from paper_conf_isca_libwmvgjbj025_b200 import workloads as W  # noqa: E402

METRIC = "simulated design points/sec"
UNIT = "points/s"
CONFIGS = {"c2": W.sweep_c2, "c3": W.sweep_c3, "c4": W.sweep_c4, "c1": W.sweep_c1, "c5": W.sweep_c5,
           "wafer": W.sweep_wafer}
DEFAULT_POINTS = {"c5": 296}   # configs[4]'s 966k-point sweep: a seeded prefix (two waves of 1024-thread CTAs)
WORKLOAD = {"c2": "configs[1]: ResNet-50 DP/DDP, 2-16 simulated GPUs on an NVLink-style ring, 10k-point "
                  "bandwidth x latency x batch x bucket sweep",
            "c3": "configs[2]: BERT-large Megatron/paper TP 2/4/8, ring/star/mesh/cube-mesh/ring-graph/"
                  "double-ring topologies incl. asymmetric",
            "c4": "configs[3]: GPT-2 XL GPipe 4-16 stages x 8-64 micro-batches on 2D meshes",
            "c1": "configs[0]: 4-layer MLP DDP on 2 GPUs, one uniform link",
            "c5": "configs[4]: GPT-3-class DP x TP x PP on 64-1024 simulated GPUs, hierarchical 1:1 / 2:1 / 4:1 "
                  "topology incl. a seeded slow-link subset (966k-point sweep, seeded prefix)",
            "wafer": "NEXT 1: 84-GPU 12x7 wafer, DDP ResNet-50, ring over the electrical mesh vs Passage photonic "
                     "logical links (P:330-342)"}
FP64_LANES_PER_SM = 64     # B200 FP64 pipe: 64 DFMA/DADD/DMUL lanes per SM per clock
N_SMS = 148


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f), "measured"
    except Exception:
        return {"hbm_gbs": 6650.0, "sm_max_mhz": 1965.0}, "fallback"


class Clocks:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md clocks line)."""

    def __init__(self, gpu):
        self.gpu = gpu
        self.rows = []
        self.proc = None

    def __enter__(self):
        q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
             "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--id={self.gpu}", f"--query-gpu={q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def summary(self):
        sm = [float(r[1]) for r in self.rows if len(r) >= 9 and r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in self.rows if len(r) >= 9 and r[2].replace(".", "").isdigit()]
        reasons = set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in self.rows:
            if len(r) >= 9:
                for n, v in zip(names, r[5:9]):
                    if v.strip().lower() == "active":
                        reasons.add(n)
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm)}


# ------------------------------------------------------------------------------------------
# CPU oracle legs (cpu_baseline and --impl reference): test infrastructure, run as it stands
# ------------------------------------------------------------------------------------------
def _oracle_chunk(args):
    cfg, idx = args
    import oracle
    sw = CONFIGS[cfg]()
    t0 = time.perf_counter()
    oracle.run_sweep(sw, idx)
    return time.perf_counter() - t0


def oracle_rate(cfg, seconds=12.0, procs=None):
    """Oracle points/s on the host: first single-process calibration, then `procs` processes on
    disjoint chunks of the seeded sweep order (about `seconds` of wall time)."""
    import oracle
    oracle.build()
    sw = CONFIGS[cfg]()
    n = len(sw.points)
    t0 = time.perf_counter()
    k = 0
    while time.perf_counter() - t0 < min(2.0, seconds / 4) and k < n:
        oracle.run_sweep(sw, [k])
        k += 1
    one = k / (time.perf_counter() - t0)
    procs = procs or os.cpu_count() or 1
    per = max(1, int(one * seconds * 0.6))
    chunks = [(cfg, [(k + i * per + j) % n for j in range(per)]) for i in range(procs)]
    t0 = time.perf_counter()
    with mp.get_context("spawn").Pool(procs) as pool:
        pool.map(_oracle_chunk, chunks)
    wall = time.perf_counter() - t0
    return {"value": round(procs * per / wall, 3), "unit": UNIT, "cores": procs, "kind": "oracle",
            "single_core_value": round(one, 3),
            "sample": f"{procs} processes x {per} points of the seeded {cfg} sweep order "
                      f"(oracle/triosim_oracle.c, gcc -O2 -ffp-contract=off, 1 thread each); "
                      f"CPU {cpu_model()}"}


def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return "unknown"


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import oracle
    oracle.build()
    sw = CONFIGS[args.config]()
    n = len(sw.points)
    per_step = args.ref_points
    times = []
    for s in range(args.warmup + args.steps):
        idx = [(s * per_step + j) % n for j in range(per_step)]
        t0 = time.perf_counter()
        oracle.run_sweep(sw, idx)
        dt = time.perf_counter() - t0
        if s >= args.warmup:
            times.append(dt)
    ms = 1e3 * float(np.mean(times))
    value = per_step / (ms / 1e3)
    out = {"metric": METRIC, "value": round(value, 3), "unit": UNIT, "impl": "reference", "n_gpus": args.gpus,
           "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms, 3), "higher_is_better": True,
           "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
           "config": {"workload": WORKLOAD[args.config], "points_per_step": per_step},
           "cpu_baseline": {"value": round(value, 3), "unit": UNIT, "cores": 1, "kind": "oracle",
                            "sample": f"{per_step} consecutive points of the seeded {args.config} sweep per step, "
                                      f"single-threaded oracle; CPU {cpu_model()}"},
           "e2e": {"value": round(value, 3), "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)


# ------------------------------------------------------------------------------------------
# our arm
# ------------------------------------------------------------------------------------------
def algorithmic_bytes(sw):
    """Bytes the method must read / write per sweep: the trace tables once
    per class, per point its descriptor (56 B), its topology's used links and routes, its
    result record (112 B)."""
    tr = sw.trace
    trace_b = tr.ops.nbytes + tr.tensors.nbytes + tr.io.nbytes
    ncls = len({(int(p["strategy"]), int(p["dp"]), int(p["tp"]), int(p["pp"]), int(p["global_batch"]),
                 int(p["bucket_bytes"]), int(p["microbatches"]), int(p["tp_mode"]), int(p["coll_algo"]))
                for p in sw.points})
    per_pt = W.POINT_DTYPE.itemsize + W.RESULT_DTYPE.itemsize
    topo_b = sum(sw.topos[int(p["topo"])].links.nbytes for p in sw.points)
    return ncls * trace_b + len(sw.points) * per_pt + topo_b


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="c2", choices=sorted(CONFIGS))
    ap.add_argument("--ref-points", type=int, default=300)
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=10)
    ap.add_argument("--points", type=int, default=0,
                    help="simulate a seeded prefix of this many points of the sweep (0 = config default)")
    ap.add_argument("--shard", action="store_true",
                    help="strong scaling: deal one sweep to the ranks by cost instead of a full sweep per rank")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    if args.impl == "reference":
        return run_reference(args)

    import torch
    import torch.distributed as dist
    from paper_conf_isca_libwmvgjbj025_b200 import dist as D, triosim

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))

    sw = CONFIGS[args.config]()
    npts = args.points or DEFAULT_POINTS.get(args.config, 0)
    if npts and npts < len(sw.points):
        sw = W.Sweep(sw.name, sw.trace, sw.topos, sw.points[:npts], sw.plans)
    n_sweep = len(sw.points)
    if args.shard and world > 1:
        tr = sw.trace
        wg = tr.tensors[tr.tensors["category"] == W.CAT_WGRAD]
        costs = D.point_cost(sw.points, len(tr.ops), len(wg), int(wg["bytes_b0"].sum()))
        maxc = max(D.shard_sizes(n_sweep, world, costs))
        sw = W.Sweep(sw.name, sw.trace, sw.topos, sw.points[D.shard_points(costs, world, rank)], sw.plans)
    n = len(sw.points)
    maxc = maxc if (args.shard and world > 1) else n
    ctx = triosim.Context(local)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    tid = ctx.triosim_load_trace(sw.trace)
    t1 = time.perf_counter()
    sid = ctx.triosim_build_sweep(tid, sw.topos, sw.points, sw.plans or None)
    t2 = time.perf_counter()
    setup_ms = {"load_trace": round((t1 - t0) * 1e3, 3), "build_sweep": round((t2 - t1) * 1e3, 3)}
    stream = torch.cuda.Stream()
    rec = W.RESULT_DTYPE.itemsize
    res_local = torch.zeros(n * rec, dtype=torch.uint8, device="cuda")
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")   # > 126 MB L2

    def step():
        ctx.triosim_simulate_batch(sid, 0, n, stream.cuda_stream)
        ctx.triosim_results(sid, 0, n, device_ptr=res_local.data_ptr(), stream=stream.cuda_stream)
        if world > 1:
            with torch.cuda.stream(stream):
                D.gather_records(res_local, world, maxc)   # one NCCL all-gather of the records

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    k0 = ctx.launch_counts()
    ctx.timing(True)
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    with Clocks(local) as clk:
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        for i in range(args.steps):
            with torch.cuda.stream(stream):
                flush.zero_()                       # L2 flush between steps, outside the events
                evs[i][0].record(stream)
            step()
            evs[i][1].record(stream)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
    k1 = ctx.launch_counts()
    step_ms = [a.elapsed_time(b) for a, b in evs]
    tot_ms, k3_ms = ctx.timings()
    ctx.timing(False)
    alg_ops = ctx.work_counters(sid)
    ms = float(np.mean(step_ms))
    if world > 1:
        t = torch.tensor([ms], device="cuda", dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    total_points = n_sweep if (args.shard and world > 1) else n * world
    value = total_points / (ms / 1e3)
    gpu_launches = sum(k1) - sum(k0)
    res = ctx.triosim_results(sid, 0, n)
    n_ok = int((res["status"] == 0).sum())

    # end to end through the public API with host buffers: H2D of the trace / topologies / points
    # from pinned host memory, the full path, D2H of the results, every step
    pin = {k: torch.from_numpy(v.view(np.uint8)).pin_memory().numpy().view(v.dtype) for k, v in
           (("ops", sw.trace.ops), ("ts", sw.trace.tensors), ("io", sw.trace.io), ("pts", sw.points))}
    tr_pinned = W.Trace(sw.trace.name, pin["ops"], pin["ts"], pin["io"], sw.trace.trace_batch, sw.trace.n_layers)
    e2e_t = []
    out_host = torch.empty(n * rec, dtype=torch.uint8).pin_memory().numpy().view(W.RESULT_DTYPE)
    for i in range(args.e2e_steps + 1):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        t2 = ctx.triosim_load_trace(tr_pinned)
        s2 = ctx.triosim_build_sweep(t2, sw.topos, pin["pts"], sw.plans or None)
        ctx.triosim_simulate_batch(s2, 0, n, stream.cuda_stream)
        ctx.triosim_results(s2, 0, n, out=out_host, stream=stream.cuda_stream)
        ctx.triosim_release(s2)
        ctx.triosim_release(t2)
        dt = time.perf_counter() - t0
        if i > 0:
            e2e_t.append(dt)
    assert out_host.tobytes() == res.tobytes()
    h2d = (sw.trace.ops.nbytes + sw.trace.tensors.nbytes + sw.trace.io.nbytes + sw.points.nbytes +
           sum(t.links.nbytes + t.ring_order.nbytes for t in sw.topos))
    # mean over consecutive steps (what a user calling the API in a loop sees), then max over ranks
    e2e_ms = float(np.mean(e2e_t)) * 1e3 if e2e_t else float("nan")
    e2e_points = total_points
    if world > 1:
        t = torch.tensor([e2e_ms], device="cuda", dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        e2e_ms = float(t.item())

    # the p = 8 slice of C2 timed on its own, per-tensor and 25 MiB buckets
    slices = {}
    if args.config == "c2" and rank == 0 and not args.shard:
        for name, bucket in (("p8_per_tensor", 0), ("p8_bucket_25MiB", 25 << 20)):
            sel = (sw.points["dp"] == 8) & (sw.points["bucket_bytes"] == bucket)
            if not sel.any():
                continue
            t3 = ctx.triosim_load_trace(sw.trace)
            s3 = ctx.triosim_build_sweep(t3, sw.topos, sw.points[sel], sw.plans or None)
            k = int(sel.sum())
            times = []
            for r in range(6):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                with torch.cuda.stream(stream):
                    flush.zero_()
                    e0.record(stream)
                ctx.triosim_simulate_batch(s3, 0, k, stream.cuda_stream)
                e1.record(stream)
                torch.cuda.synchronize()
                if r > 0:
                    times.append(e0.elapsed_time(e1))
            ctx.triosim_release(s3)
            ctx.triosim_release(t3)
            med = float(np.median(times))
            slices[name] = {"points": k, "value": round(k / (med / 1e3), 1), "unit": UNIT, "ms": round(med, 4),
                            "timing": "median of 5 device-timed simulate_batch calls, L2 flushed before each"}

    if rank == 0:
        pk, src = peaks()
        k3 = float(np.mean(k3_ms)) if len(k3_ms) else float("nan")
        clock_mhz = float(pk.get("sm_max_mhz", 1965.0))
        peak_ops = N_SMS * FP64_LANES_PER_SM * clock_mhz * 1e6
        achieved = alg_ops / (k3 / 1e3)
        traffic = None
        try:
            with open(os.path.join(ROOT, "profiles", "k3_ncu_summary.json")) as f:
                traffic = json.load(f).get(f"dram_bytes_per_launch_{args.config}")
        except Exception:
            pass
        alg_b = algorithmic_bytes(sw)
        out = {
            "metric": METRIC, "value": round(value, 1), "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": round(ms, 4), "higher_is_better": True,
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "scaling": "strong" if (args.shard and world > 1) else "weak",
            "config": {"workload": WORKLOAD[args.config], "points": n, "points_ok": n_ok,
                       "sweep_points": len(CONFIGS[args.config]().points) if npts else n_sweep,
                       "trace": sw.trace.name, "ops": int(len(sw.trace.ops)),
                       "parallelism": (f"one sweep dealt to {world} ranks by cost; records all-gathered over NCCL"
                                       if (args.shard and world > 1) else
                                       f"each of {world} rank(s) simulates a full sweep (weak scaling); "
                                       "records all-gathered over NCCL"),
                       "l2": "flushed (256 MB write) before every timed step"},
            "roofline": {"bound": "alu", "kernel": "k3_timeline", "achieved": round(achieved / 1e12, 6),
                         "peak": round(peak_ops / 1e12, 3), "unit": "TFLOP/s (fp64, non-tensor)",
                         "frac": round(achieved / peak_ops, 6), "traffic": traffic,
                         "k3_ms": round(k3, 4), "alg_fp64_ops_per_launch": int(alg_ops),
                         "peak_source": f"{N_SMS} SMs x {FP64_LANES_PER_SM} fp64 lanes x {clock_mhz} MHz "
                                        f"(sm_max_mhz {src})"},
            "hbm_roofline": {"bound": "hbm", "achieved": round(alg_b / (k3 / 1e3) / 1e9, 3),
                             "peak": pk.get("hbm_gbs"), "unit": "GB/s",
                             "frac": round(alg_b / (k3 / 1e3) / 1e9 / float(pk.get("hbm_gbs", 6650.0)), 7),
                             "algorithmic_bytes_per_launch": int(alg_b), "peak_source": src},
            "e2e": {"value": round(e2e_points / (e2e_ms / 1e3), 1), "unit": UNIT, "h2d_bytes_per_step": int(h2d),
                    "d2h_bytes_per_step": int(n * rec), "ms_per_step": round(e2e_ms, 3),
                    "steps": len(e2e_t), "timing": "wall clock, mean of consecutive API calls, max over ranks"},
            "gpu_launches": int(gpu_launches),
            "setup_ms": setup_ms,
            "clocks": clk.summary(),
            "paper_context": "TrioSim (Go/Akita, 1 CPU process): 'within seconds' per simulation, host not "
                             "stated (P:29, P:306)",
        }
        if slices:
            out["slices"] = slices
        if not args.no_cpu_baseline and world == 1:
            cb = oracle_rate(args.config, seconds=args.cpu_seconds)
            out["cpu_baseline"] = cb
            out["speedup_vs_oracle"] = {"one_core": round(value / cb["single_core_value"], 1),
                                        f"{cb['cores']}_cores": round(value / cb["value"], 1)}
        print(json.dumps(out), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    ctx.close()


if __name__ == "__main__":
    main()
