"""Per-source-line instruction / stall-sample attribution of an ncu capture (run here, no GPU).

    python profiles/sass_lines.py <capture.ncu-rep | source-page.csv[.gz]> <libtriosim.so> <mangled kernel> [top] [section]

Joins ncu's SASS source page (per-instruction counts, by address order) with nvdisasm -g line
info of the same cubin, and prints the hottest source lines.
"""
import collections
import csv
import io
import os
import re
import subprocess
import sys
import tempfile


def main(rep, so, fn, top=40, section=None):
    if rep.endswith(".csv.gz") or rep.endswith(".csv"):   # a source page exported on the GPU box
        import gzip
        sass = (gzip.open(rep, "rt") if rep.endswith(".gz") else open(rep)).read()
    else:
        sass = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                              capture_output=True, text=True).stdout
    allrows = list(csv.reader(io.StringIO(sass)))
    starts = [i for i, r in enumerate(allrows) if r and r[0] == "Kernel Name"] + [len(allrows)]
    rows = None
    for a, b in zip(starts, starts[1:]):
        if section is None or section in allrows[a][1]:
            rows = allrows[a:b]
            break
    hdr = rows[1]
    ie, ss = hdr.index("Instructions Executed"), hdr.index("Warp Stall Sampling (All Samples)")
    counts = [(int(r[ie] or 0), int(r[ss] or 0)) for r in rows[2:] if len(r) > ie]
    with tempfile.TemporaryDirectory() as d:
        subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath(so)], cwd=d, capture_output=True)
        lines = []
        for f in sorted(os.listdir(d)):
            out = subprocess.run(["nvdisasm", "-g", "-c", os.path.join(d, f)], capture_output=True,
                                 text=True).stdout
            start = out.find(f".text.{fn}:")
            if start >= 0:
                body = out[start:]
                nxt = body.find("//---------------------", 10)
                body = body if nxt < 0 else body[:nxt]
                cur = None
                for ln in body.splitlines():
                    m = re.search(r'//## File "([^"]+)", line (\d+)', ln)
                    if m:
                        cur = f"{os.path.basename(m.group(1))}:{m.group(2)}"
                    elif re.search(r"/\*[0-9a-f]{4,}\*/", ln):
                        lines.append(cur)
                break
    agg = collections.defaultdict(lambda: [0, 0])
    for (n, s), l in zip(counts, lines):
        agg[l][0] += n
        agg[l][1] += s
    tot_i = sum(v[0] for v in agg.values()) or 1
    tot_s = sum(v[1] for v in agg.values()) or 1
    print(f"instructions {tot_i}, stall samples {tot_s}, sass {len(counts)} vs lines {len(lines)}")
    for l, (n, s) in sorted(agg.items(), key=lambda kv: -kv[1][1])[:top]:
        print(f"{l:24s} inst {100 * n / tot_i:6.2f}%  samples {100 * s / tot_s:6.2f}%")


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2], sys.argv[3], int(sys.argv[4]) if len(sys.argv) > 4 else 40,
         sys.argv[5] if len(sys.argv) > 5 else None)
