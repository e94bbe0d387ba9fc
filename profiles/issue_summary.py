"""Summarise an ncu --metrics CSV of ONE bench step's K3 launches into profiles/ncu_issue_<cfg>.json, the
issue evidence bench.py prints next to the roofline (run here, no GPU needed).

    python profiles/issue_summary.py <ncu.csv> <cfg> <run id>
"""
import csv
import json
import os
import sys


def main(path, cfg, run):
    rows = list(csv.reader(open(path)))
    h = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
    hdr = rows[h]
    ki, mi, vi = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value")
    per = {}
    for r in rows[h + 1:]:
        if len(r) <= vi or "k3_" not in r[ki]:
            continue
        per.setdefault(r[0], {"kernel": r[ki]})[r[mi]] = float(r[vi].replace(",", ""))
    launches = list(per.values())
    tot = lambda k: sum(l.get(k, 0.0) for l in launches)
    inst = tot("smsp__inst_executed.sum")
    thr = tot("smsp__thread_inst_executed.sum")
    dur = tot("gpu__time_duration.sum")
    warps = sum(l.get("sm__warps_active.avg.pct_of_peak_sustained_active", 0.0) * l.get("gpu__time_duration.sum", 0.0)
                for l in launches) / max(dur, 1e-30)
    out = {"run": run, "config": cfg, "launches": len(launches),
           "warp_inst_per_step": inst, "lane_efficiency": round(thr / max(inst, 1.0) / 32.0, 4),
           "warps_active_pct": round(warps, 3),
           "dram_bytes_per_step": tot("dram__bytes_read.sum") + tot("dram__bytes_write.sum"),
           "serialised_k3_ns": dur,
           "kernels": [{k: v for k, v in l.items()} for l in launches]}
    dst = os.path.join(os.path.dirname(os.path.abspath(__file__)), f"ncu_issue_{cfg}.json")
    json.dump(out, open(dst, "w"), indent=1)
    print(json.dumps({k: v for k, v in out.items() if k != "kernels"}))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2], sys.argv[3])
