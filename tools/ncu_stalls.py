"""Summarise the last kernel of an ncu report: key metrics + stall sampling per SASS instruction.
    python tools/ncu_stalls.py report.ncu-rep [top_n] [launch_skip]"""
import csv, io, subprocess, sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 30
skip = sys.argv[3] if len(sys.argv) > 3 else "1"
M = ("gpu__time_duration.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,"
     "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active,"
     "smsp__inst_executed.sum,sm__warps_active.avg.per_cycle_active,launch__grid_size,launch__block_size,"
     "sm__cycles_active.avg,sm__cycles_active.max,sm__cycles_active.min,sm__cycles_elapsed.max,"
     "dram__bytes_read.sum,dram__bytes_write.sum")
out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv", "--metrics", M], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
h = rows[0]
for r in rows[2:]:
    print(r[h.index("Kernel Name")][:70])
    for i, k in enumerate(h):
        if "__" in k:
            print(f"   {k:60s} {r[i]}")
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass", "--launch-skip", skip,
                      "--launch-count", "1"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(src)))
his = [i for i, r in enumerate(rows) if r and r[0] == "Address"]
if not his:
    sys.exit(0)
hdr = rows[his[-1]]
data = [dict(zip(hdr, r)) for r in rows[his[-1] + 1:] if len(r) == len(hdr)]
f = lambda x: float(x) if x and x.replace(".", "", 1).isdigit() else 0.0
S = "Warp Stall Sampling (All Samples)"
reasons = [k for k in hdr if k.startswith("stall_") and "Not Issued" not in k]
tot = sum(f(d[S]) for d in data) or 1.0
print("stall samples", tot)
for r, v in sorted(((r, sum(f(d[r]) for d in data)) for r in reasons), key=lambda kv: -kv[1])[:8]:
    print(f"  {r:28s} {v / tot * 100:6.2f}%")
for d in sorted(data, key=lambda d: -f(d[S]))[:top]:
    t3 = sorted(((f(d[r]), r) for r in reasons), reverse=True)[:3]
    print(f"{f(d[S]) / tot * 100:5.2f}% {d['Address'][-5:]} exec={d['Instructions Executed']:>10} {d['Source'][:58]:58s} "
          + " ".join(f"{r[6:]}={v / tot * 100:.2f}" for v, r in t3 if v))
