#!/usr/bin/env python
"""Benchmark: simulated design points / s on B200 (BASELINE.json metric), configs[1] workload
(ResNet-50 DDP sweep, 10,000 points, 2-16 simulated GPUs on an NVLink-style ring).

One step = one pass of the whole hot path over the sweep: K1b operator rescale + K2 task-graph
expansion for every structural class + K3 timeline for every point, results written to device
memory, then (N > 1) one NCCL all-gather of the 112-B records and their scatter into sweep order.
Inputs are resident in HBM (built once).

    python bench.py [--gpus N --steps K --warmup W] [--impl reference] [--config c2|c3|c4|c5|...]

--gpus N > 1 without torchrun re-launches itself under torch.distributed.run (one process per GPU).
Multi-GPU: the sweep at N GPUs is configs[1]'s family at N x 10,000 distinct
points (its bandwidth axis refined N-fold; N = 1 is configs[1] itself), dealt to the ranks by estimated
cost in snake order -- every point simulated exactly once, per-GPU work fixed (weak scaling).
--scaling strong instead deals the fixed 10,000-point sweep.  Rank 0 prints one JSON line.
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
           "c5_subset": W.sweep_c5_parity, "wafer": W.sweep_wafer, "hop": W.sweep_hop}
DEFAULT_POINTS = {"c5": 296}   # configs[4]'s 966k-point sweep: a seeded prefix (two waves of 1024-thread CTAs)
WORKLOAD = {"c2": "configs[1]: ResNet-50 DDP (data parallel), 2-16 simulated GPUs on an NVLink-style ring, 10k-point "
                  "bandwidth x latency x batch x bucket sweep",
            "c3": "configs[2]: BERT-large Megatron/paper TP 2/4/8, ring/star/mesh/cube-mesh/ring-graph/"
                  "double-ring topologies incl. asymmetric",
            "c4": "configs[3]: GPT-2 XL GPipe 4-16 stages x 8-64 micro-batches on 2D meshes",
            "c1": "configs[0]: 4-layer MLP DDP on 2 GPUs, one uniform link",
            "c5": "configs[4]: GPT-3-class DP x TP x PP on 64-1024 simulated GPUs, hierarchical 1:1 / 2:1 / 4:1 "
                  "topology incl. a seeded slow-link subset (966k-point sweep, seeded prefix)",
            "c5_subset": "configs[4] stratified subset: 100 GPT-3-class DP x TP x PP points, 20 per N in {64..1024} "
                         "simulated GPUs incl. the dp x tp = 64 heavy class on the perturbed 4:1 topologies (the C5 "
                         "parity sample, W.sweep_c5_parity)",
            "hop": "NEXT 4: Hop decentralized training (P:348-364, Fig. 16), VGG-11 bs128 on 8 workers, ring-based / "
                   "double-ring graphs, 8 random 1-10x slowdown groups, 0 / 1 backup worker, staleness + token gap",
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
    """SM clock and throttle-reason sampling during the timed region (B200_PROFILING.md clocks line): NVML
    polled every ~2 ms from a thread (a C2 timed region is ~40 ms, shorter than nvidia-smi's 100 ms loop),
    with nvidia-smi as the fallback when NVML is unavailable."""

    REASONS = (("hw_slowdown", "nvmlClocksEventReasonHwSlowdown"),
               ("hw_thermal_slowdown", "nvmlClocksEventReasonHwThermalSlowdown"),
               ("sw_thermal_slowdown", "nvmlClocksEventReasonSwThermalSlowdown"),
               ("sw_power_cap", "nvmlClocksEventReasonSwPowerCap"))

    def __init__(self, gpu):
        self.gpu = gpu
        self.rows = []
        self.proc = None
        self.nv = None
        self.stop = threading.Event()

    def __enter__(self):
        try:
            import pynvml as nv
            nv.nvmlInit()
            self.h = nv.nvmlDeviceGetHandleByIndex(self.gpu)
            self.mx = float(nv.nvmlDeviceGetMaxClockInfo(self.h, nv.NVML_CLOCK_SM))
            self.nv = nv
            self.t = threading.Thread(target=self._poll, daemon=True)
            self.t.start()
            return self
        except Exception:
            self.nv = None
        return self._enter_smi()

    def _poll(self):
        nv = self.nv
        while not self.stop.is_set():
            try:
                sm = float(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
                rs = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                self.rows.append([str(self.gpu), str(sm), str(self.mx), "", ""] +
                                 ["Active" if rs & getattr(nv, c) else "Not Active" for _, c in self.REASONS])
            except Exception:
                pass
            self.stop.wait(0.002)

    def _enter_smi(self):
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
        if self.nv is not None:
            self.stop.set()
            self.t.join(timeout=2)
            try:
                self.nv.nvmlShutdown()
            except Exception:
                pass
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
                "reasons": sorted(reasons), "samples": len(sm), "source": "nvml" if self.nv is not None else "nvidia-smi"}


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
OPS_PER_TASK = 2      # algorithmic fp64 ops per operator instance (rescale + fold)
OPS_PER_WF_CALL = 80  # algorithmic fp64 ops per water-filling call (|A| <= 16)
DEFAULT_NBW = {"c2": 25, "c3": 8, "c4": 25, "c5": 25, "wafer": 10, "hop": 5}


def make_sweep(cfg, scale=1, npts=0):
    """The config's sweep; scale > 1 refines its bandwidth axis scale-fold (distinct points, same mix)."""
    f = CONFIGS[cfg]
    sw = f(n_bw=DEFAULT_NBW[cfg] * scale) if (scale > 1 and cfg in DEFAULT_NBW) else f()
    if npts and npts < len(sw.points):
        sw = W.Sweep(sw.name, sw.trace, sw.topos, sw.points[:npts], sw.plans)
    return sw


def algorithmic_fp64(res):
    """SURVEY 8(d).2's algorithmic fp64 count of the simulated points: 2 per operator instance plus
    80 per water-filling call (counts from the result records, which the oracle pins)."""
    ok = res["status"] == 0
    return int(OPS_PER_TASK * res["n_compute"][ok].astype(np.int64).sum()
               + OPS_PER_WF_CALL * res["n_wf_calls"][ok].astype(np.int64).sum())


def algorithmic_bytes(sw):
    """SURVEY 8(d).2's algorithmic bytes: per point the trace SoA read once (16 B per operator: time f64,
    packed flags, layer), the weight-gradient sizes (8 B each), its topology's links (24 B each) and route
    table (5 B per GPU pair), its descriptor (56 B) and its result record (112 B)."""
    tr = sw.trace
    n_wg = int((tr.tensors["category"] == W.CAT_WGRAD).sum())
    per_trace = 16 * len(tr.ops) + 8 * n_wg
    topo_b = np.asarray([t.links.nbytes + 5 * t.n_gpus * t.n_gpus for t in sw.topos])
    return int(len(sw.points) * (per_trace + W.POINT_DTYPE.itemsize + W.RESULT_DTYPE.itemsize)
               + topo_b[sw.points["topo"].astype(np.int64)].sum())


def issue_evidence(cfg):
    """Warp-instruction counts of the K3 launches of one step from a committed ncu capture."""
    try:
        with open(os.path.join(ROOT, "profiles", f"ncu_issue_{cfg}.json")) as f:
            return json.load(f)
    except Exception:
        return None


def relaunch(n):
    import socket
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


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
    ap.add_argument("--scaling", default="weak", choices=["weak", "strong"],
                    help="weak: N x the sweep (distinct points) over N GPUs; strong: one sweep dealt to N GPUs")
    ap.add_argument("--sweep-scale", type=int, default=0,
                    help="bandwidth-axis refinement of the sweep (0 = N for weak scaling, 1 for strong)")
    ap.add_argument("--dump-records", default="", help="rank 0 writes the sweep-ordered records here")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    if args.impl == "reference":
        return run_reference(args)
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        sys.exit(relaunch(args.gpus))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if world != args.gpus:
        print(json.dumps({"error": f"--gpus {args.gpus} but WORLD_SIZE {world}"}), flush=True)
        sys.exit(2)

    import torch
    import torch.distributed as dist
    from paper_conf_isca_libwmvgjbj025_b200 import dist as D, triosim

    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    dev_idx = 0 if os.environ.get("TS_SHARE_GPU") == "1" else local   # TS_SHARE_GPU: test-only, ranks share GPU 0
    torch.cuda.set_device(dev_idx)
    backend = os.environ.get("TS_DIST_BACKEND", "nccl")
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", dev_idx))
        else:
            dist.init_process_group(backend)

    scale = args.sweep_scale or (world if args.scaling == "weak" else 1)
    sw = make_sweep(args.config, scale, args.points or DEFAULT_POINTS.get(args.config, 0))
    n_sweep = len(sw.points)
    plan = D.ShardPlan(D.sweep_cost(sw), world, rank)
    sub = plan.sub_sweep(sw)
    n = len(sub.points)
    ctx = triosim.Context(dev_idx)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    tid = ctx.triosim_load_trace(sub.trace)
    t1 = time.perf_counter()
    sid = ctx.triosim_build_sweep(tid, sub.topos, sub.points, sub.plans or None)
    t2 = time.perf_counter()
    setup_ms = {"load_trace": round((t1 - t0) * 1e3, 3), "build_sweep": round((t2 - t1) * 1e3, 3)}
    stream = torch.cuda.Stream()
    rec = W.RESULT_DTYPE.itemsize
    res_local = torch.zeros(max(n, 1) * rec, dtype=torch.uint8, device="cuda")
    res_all = torch.zeros(n_sweep * rec, dtype=torch.uint8, device="cuda")
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")   # > 126 MB L2

    def step():
        if n:
            ctx.triosim_simulate_batch(sid, 0, n, stream.cuda_stream)
            ctx.triosim_results(sid, 0, n, device_ptr=res_local.data_ptr(), stream=stream.cuda_stream)
        with torch.cuda.stream(stream):
            plan.gather(res_local[: n * rec], out=res_all)   # one all-gather + scatter into sweep order

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    k0 = ctx.launch_counts()
    ctx.timing(True)
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    with Clocks(dev_idx) as clk:
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
    kernel_ops = ctx.work_counters(sid)
    ms = float(np.mean(step_ms))
    k3 = float(np.mean(k3_ms)) if len(k3_ms) else float("nan")
    if world > 1:
        t = torch.tensor([ms, k3], device="cuda", dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms, k3 = float(t[0].item()), float(t[1].item())
    value = n_sweep / (ms / 1e3)
    gpu_launches = sum(k1) - sum(k0)
    if world > 1:
        t = torch.tensor([gpu_launches], device="cuda", dtype=torch.int64)
        dist.all_reduce(t)
        gpu_launches = int(t.item())
    res = res_all.cpu().numpy().view(W.RESULT_DTYPE).copy()
    n_ok = int((res["status"] == 0).sum())
    if args.dump_records and rank == 0:
        res.tofile(args.dump_records)

    # end to end through the public API with host buffers, every step: H2D of this rank's trace / topologies
    # / points from pinned host memory (load_trace, build_sweep), simulate, results, the all-gather into
    # sweep order and the D2H of the sweep's records on rank 0 (D.simulate_sharded)
    pin = {k: torch.from_numpy(v.view(np.uint8)).pin_memory().numpy().view(v.dtype) for k, v in
           (("ops", sub.trace.ops), ("ts", sub.trace.tensors), ("io", sub.trace.io), ("pts", sub.points))}
    sub_pinned = W.Sweep(sub.name, W.Trace(sub.trace.name, pin["ops"], pin["ts"], pin["io"], sub.trace.trace_batch,
                                           sub.trace.n_layers), sub.topos, pin["pts"], sub.plans)
    e2e_t = []
    for i in range(args.e2e_steps + 1):
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        t0 = time.perf_counter()
        with torch.cuda.stream(stream):
            host = D.simulate_sharded(ctx, sw, plan, sub=sub_pinned, host_on_rank0=True)
        dt = time.perf_counter() - t0
        if i > 0:
            e2e_t.append(dt)
        if rank == 0:
            assert host.tobytes() == res.tobytes(), "e2e records differ from the device-timed step"
    h2d = int(sum((sub.trace.ops.nbytes + sub.trace.tensors.nbytes + sub.trace.io.nbytes + len(plan.shards[r]) *
                   W.POINT_DTYPE.itemsize + sum(t.links.nbytes + t.ring_order.nbytes for t in sw.topos))
                  for r in range(world)))
    e2e_ms = float(np.mean(e2e_t)) * 1e3 if e2e_t else float("nan")
    if world > 1:
        t = torch.tensor([e2e_ms], device="cuda", dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        e2e_ms = float(t.item())

    # the p = 8 slice of C2 timed on its own, per-tensor and 25 MiB buckets
    slices = {}
    if args.config == "c2" and world == 1:
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
        clock_mhz = float(pk.get("sm_max_mhz", 1965.0))
        peak_ops = N_SMS * FP64_LANES_PER_SM * clock_mhz * 1e6
        alg_ops = algorithmic_fp64(res) / world          # per rank (one K3 phase), whole sweep / N
        achieved = alg_ops / (k3 / 1e3)
        alg_b = algorithmic_bytes(sw) / world
        iss = issue_evidence(args.config)
        roof = {"bound": "alu", "kernel": "k3_timeline (K3 phase: every K3 launch of the step)",
                "achieved": round(achieved / 1e12, 6), "peak": round(peak_ops / 1e12, 3),
                "unit": "TFLOP/s (fp64, non-tensor)", "frac": round(achieved / peak_ops, 6),
                "traffic": None if iss is None else iss.get("dram_bytes_per_step"),
                "traffic_source": None if iss is None else f"profiles/ncu_issue_{args.config}.json ({iss.get('run')})",
                "k3_ms": round(k3, 4), "alg_fp64_ops_per_launch": int(alg_ops),
                "alg_derivation": f"SURVEY 8(d).2: {OPS_PER_TASK} x n_compute + {OPS_PER_WF_CALL} x n_wf_calls summed "
                                  "over the step's points (counts from the result records), / K3 phase time",
                "kernel_executed_fp64_ops_per_launch": int(kernel_ops),
                "peak_source": f"{N_SMS} SMs x {FP64_LANES_PER_SM} fp64 lanes x {clock_mhz} MHz (sm_max_mhz {src}; "
                               "derived, MEASURED_PEAKS.json has no fp64 entry)"}
        if iss is not None and iss.get("warp_inst_per_step"):
            ipeak = N_SMS * 4 * clock_mhz * 1e6
            roof["issue"] = {"warp_inst_per_step": iss["warp_inst_per_step"], "peak_warp_inst_per_s": ipeak,
                             "frac": round(iss["warp_inst_per_step"] / (k3 / 1e3) / ipeak, 4),
                             "warps_active_pct": iss.get("warps_active_pct"),
                             "lane_efficiency": iss.get("lane_efficiency"),
                             "source": f"profiles/ncu_issue_{args.config}.json ({iss.get('run')}): ncu "
                                       "smsp__inst_executed.sum over the step's K3 launches / (148 SMs x 4 "
                                       "schedulers x sm_max_mhz) / measured K3 phase time"}
        out = {
            "metric": METRIC, "value": round(value, 1), "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": round(ms, 4), "higher_is_better": True,
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "scaling": args.scaling,
            "config": {"workload": WORKLOAD[args.config], "points": n_sweep, "points_ok": n_ok,
                       "points_per_rank": [len(s) for s in plan.shards], "sweep_scale": scale,
                       "trace": sw.trace.name, "ops": int(len(sw.trace.ops)),
                       "parallelism": (f"{n_sweep} distinct points dealt to {world} rank(s) by estimated cost (snake "
                                       "order), each simulated once; records all-gathered over "
                                       f"{backend if world > 1 else 'NCCL'} and scattered into sweep order"),
                       "l2": "flushed (256 MB write) before every timed step"},
            "roofline": roof,
            "hbm_roofline": {"bound": "hbm", "achieved": round(alg_b / (k3 / 1e3) / 1e9, 3),
                             "peak": pk.get("hbm_gbs"), "unit": "GB/s",
                             "frac": round(alg_b / (k3 / 1e3) / 1e9 / float(pk.get("hbm_gbs", 6650.0)), 7),
                             "algorithmic_bytes_per_launch": int(alg_b), "peak_source": src},
            "e2e": {"value": round(n_sweep / (e2e_ms / 1e3), 1), "unit": UNIT, "h2d_bytes_per_step": h2d,
                    "d2h_bytes_per_step": int(n_sweep * rec), "ms_per_step": round(e2e_ms, 3),
                    "steps": len(e2e_t), "timing": "wall clock, mean of consecutive public-API calls "
                                                   "(dist.simulate_sharded), max over ranks"},
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
