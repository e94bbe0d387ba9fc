"""Summarise an `ncu -i <rep> --page raw --csv` export of K3 launches into a small committed JSON (run here,
no GPU needed): per launch the time, grid, registers, occupancy limit, warps active, issue active, executed
warp instructions, lane efficiency, DRAM bytes, fp64 pipe activity and the stall reasons per issue.

    python profiles/raw_summary.py <raw.csv> <out.json> <run id> [note] [--issue <cfg>]

--issue <cfg> also writes profiles/ncu_issue_<cfg>.json, the issue evidence bench.py prints next to its
roofline (warp instructions of one step's K3 launches, lane efficiency, time-weighted warps active, DRAM
bytes per step).
"""
import csv
import json
import os
import sys

KEYS = {
    "time_ms": "gpu__time_duration.sum", "grid": "launch__grid_size", "block": "launch__block_size",
    "registers": "launch__registers_per_thread", "occupancy_limit_registers": "launch__occupancy_limit_registers",
    "warps_active_pct": "sm__warps_active.avg.pct_of_peak_sustained_active",
    "issue_active_pct": "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "warp_inst": "smsp__inst_executed.sum",
    "threads_per_inst": "smsp__thread_inst_executed_per_inst_executed.ratio",
    "dram_read_bytes": "dram__bytes_read.sum", "dram_write_bytes": "dram__bytes_write.sum",
    "fp64_pipe_pct": "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
    "l1_hit_pct": "l1tex__t_sector_hit_rate.pct", "l2_hit_pct": "lts__t_sector_hit_rate.pct",
}
STALL = "smsp__average_warps_issue_stalled_%s_per_issue_active.ratio"
STALLS = ["wait", "long_scoreboard", "short_scoreboard", "barrier", "branch_resolving", "no_instruction",
          "math_pipe_throttle", "mio_throttle", "lg_throttle", "membar", "dispatch_stall", "not_selected", "selected"]


def num(x):
    try:
        return float(x.replace(",", ""))
    except Exception:
        return None


def main(path, out, run, note="", issue_cfg=None):
    rows = list(csv.reader(open(path)))
    h = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
    hdr = rows[h]
    units = rows[h + 1]
    launches = []
    for r in rows[h + 2:]:
        if len(r) < len(hdr):
            continue
        d = {"kernel": r[hdr.index("Kernel Name")]}
        for k, m in KEYS.items():
            if m in hdr:
                v = num(r[hdr.index(m)])
                u = units[hdr.index(m)]
                if k == "time_ms" and v is not None:
                    v = v * {"ns": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0, "nsecond": 1e-6}.get(u, 1.0)
                if k.startswith("dram") and v is not None:
                    v = v * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1.0)
                d[k] = v
        d["stalls_per_issue"] = {s: num(r[hdr.index(STALL % s)]) for s in STALLS if STALL % s in hdr}
        launches.append(d)
    tot_t = sum(l.get("time_ms") or 0 for l in launches)
    tot_i = sum(l.get("warp_inst") or 0 for l in launches)
    res = {"run": run, "source": path, "note": note, "launches": launches,
           "total_time_ms_serialised": round(tot_t, 4), "total_warp_inst": tot_i}
    with open(out, "w") as f:
        json.dump(res, f, indent=1)
    if issue_cfg:
        thr = sum((l.get("warp_inst") or 0) * (l.get("threads_per_inst") or 0) for l in launches)
        dur = sum(l.get("time_ms") or 0 for l in launches)
        warps = sum((l.get("warps_active_pct") or 0) * (l.get("time_ms") or 0) for l in launches) / max(dur, 1e-30)
        iss = {"run": run, "config": issue_cfg, "launches": len(launches), "warp_inst_per_step": tot_i,
               "lane_efficiency": round(thr / max(tot_i, 1.0) / 32.0, 4), "warps_active_pct": round(warps, 3),
               "dram_bytes_per_step": sum((l.get("dram_read_bytes") or 0) + (l.get("dram_write_bytes") or 0)
                                          for l in launches),
               "serialised_k3_ns": round(dur * 1e6), "source": path}
        with open(os.path.join(os.path.dirname(os.path.abspath(__file__)), f"ncu_issue_{issue_cfg}.json"), "w") as f:
            json.dump(iss, f, indent=1)
    for l in launches:
        print(l["kernel"][:40], l.get("time_ms"), l.get("registers"), l.get("warps_active_pct"), l.get("issue_active_pct"),
              {k: v for k, v in l["stalls_per_issue"].items() if v and v > 0.3})


if __name__ == "__main__":
    argv = sys.argv[1:]
    cfg = None
    if "--issue" in argv:
        k = argv.index("--issue")
        cfg = argv[k + 1]
        del argv[k:k + 2]
    main(*argv, issue_cfg=cfg)
