"""Per-source-line share of executed instructions and stall samples of one kernel in an
ncu report (development aid).   python tools/ncu_lines.py report.ncu-rep [top]"""
import collections
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
cur_file, hdr, agg, ti, ts = None, None, collections.defaultdict(lambda: [0.0, 0.0]), 0.0, 0.0
num = lambda x: float(x) if x and x.replace(".", "", 1).isdigit() else 0.0  # noqa: E731
for r in rows:
    if not r:
        continue
    if r[0] == "File Path":
        cur_file = r[1].split("/")[-1]
        continue
    if r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or not r[0] or r[0] == "Function Name":
        continue
    d = dict(zip(hdr, r))
    ie, ss = num(d.get("Instructions Executed", "")), num(d.get("Warp Stall Sampling (All Samples)", ""))
    agg[(cur_file, r[0], r[1].strip()[:72])][0] += ie
    agg[(cur_file, r[0], r[1].strip()[:72])][1] += ss
    ti, ts = ti + ie, ts + ss
print(f"instructions {ti:.4g}  stall samples {ts:.0f}")
for k, v in sorted(agg.items(), key=lambda kv: -kv[1][1])[:top]:
    print(f"{v[0] / ti * 100:5.1f}% inst {v[1] / ts * 100:5.1f}% samp  {k[0]}:{k[1]} {k[2]}")
