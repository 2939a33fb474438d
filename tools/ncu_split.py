"""Split an ncu source-page capture of one kernel at a marker instruction and
summarise each part (instructions executed, stall reasons, top instructions).
    python tools/ncu_split.py report.ncu-rep MARKER [top]   (development aid)"""
import csv, subprocess, sys, io, collections

rep, marker = sys.argv[1], sys.argv[2]
top = int(sys.argv[3]) if len(sys.argv) > 3 else 10
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True,
                     text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hi = [i for i, r in enumerate(rows) if r and r[0] == "Address"][-1]
h = rows[hi]
data = [dict(zip(h, r)) for r in rows[hi + 1:] if len(r) == len(h)]
f = lambda x: float(x) if x and x.replace('.', '', 1).isdigit() else 0.0
S = "Warp Stall Sampling (All Samples)"
reasons = [k for k in h if k.startswith("stall_") and "Not Issued" not in k]
b = [i for i, d in enumerate(data) if marker in d['Source']][0]
for name, part in (("before", data[:b]), ("after", data[b:])):
    tot = sum(f(d[S]) for d in part)
    ins = sum(f(d['Instructions Executed']) for d in part)
    print(f"{name}: instructions {ins:.3e}, stall samples {tot:.0f}")
    for r, v in sorted(((r, sum(f(d[r]) for d in part)) for r in reasons), key=lambda kv: -kv[1])[:6]:
        print(f"    {r:24s} {v:6.0f}")
    for d in sorted(part, key=lambda d: -f(d[S]))[:top]:
        t3 = sorted(((f(d[r]), r) for r in reasons), reverse=True)[:2]
        print(f"   {f(d[S]):6.0f} {d['Address'][-5:]} ex={d['Instructions Executed']:>7} {d['Source'][:55]:55s}",
              " ".join(f"{r[6:]}={v:.0f}" for v, r in t3))
