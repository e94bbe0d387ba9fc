"""Summarise ncu captures into small committed files (run here, no GPU needed).

    python profiles/summarize.py launches <launches.csv> <out.json>
    python profiles/summarize.py full <capture.ncu-rep> <out.json>
"""
import collections
import csv
import io
import json
import subprocess
import sys

FULL_METRICS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "launch__grid_size",
    "launch__block_size", "launch__registers_per_thread", "launch__occupancy_limit_registers",
    "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "smsp__inst_executed.sum", "smsp__thread_inst_executed_per_inst_executed.ratio",
    "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active", "l1tex__t_sector_hit_rate.pct",
    "lts__t_sector_hit_rate.pct", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed",
]


def launches(path):
    rows = list(csv.reader(open(path)))
    h = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
    hdr = rows[h]
    ki, vi = hdr.index("Kernel Name"), hdr.index("Metric Value")
    agg = collections.OrderedDict()
    for r in rows[h + 1:]:
        if len(r) > vi:
            agg.setdefault(r[ki], []).append(float(r[vi].replace(",", "")))
    tot = sum(sum(v) for v in agg.values())
    return {"note": "ncu --metrics gpu__time_duration.sum --clock-control none (serialised, cold cache: "
                    "compare shares, not absolutes)",
            "kernels": [{"kernel": k, "launches": len(v), "avg_us": round(sum(v) / len(v) / 1e3, 3),
                         "total_ms": round(sum(v) / 1e6, 4), "share": round(sum(v) / tot, 4)}
                        for k, v in agg.items()]}


def full(path):
    raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units = rows[0], rows[1]
    out = []
    for r in rows[2:]:
        d = {"kernel": r[hdr.index("Kernel Name")]}
        for m in FULL_METRICS:
            if m in hdr:
                d[m] = f"{r[hdr.index(m)]} {units[hdr.index(m)]}".strip()
        stalls = []
        for i, n in enumerate(hdr):
            if n.startswith("smsp__average_warps_issue_stalled_") and n.endswith("_per_issue_active.ratio"):
                try:
                    stalls.append((float(r[i]), n.split("stalled_")[1].split("_per_issue")[0]))
                except ValueError:
                    pass
        d["top_stalls_per_issue"] = {k: round(v, 3) for v, k in sorted(stalls, reverse=True)[:8]}
        out.append(d)
    return {"note": "ncu --set full --clock-control none --import-source on -k regex:k3_timeline", "launches": out}


if __name__ == "__main__":
    mode, src, dst = sys.argv[1:4]
    res = launches(src) if mode == "launches" else full(src)
    json.dump(res, open(dst, "w"), indent=1)
    print(json.dumps(res, indent=1)[:3000])
