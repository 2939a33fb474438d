"""Summarise an ncu --page source --csv dump: stall reasons per instruction (development aid)."""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hi = [i for i, r in enumerate(rows) if r and r[0] == 'Address'][0]
hdr = rows[hi]
data = [dict(zip(hdr, r)) for r in rows[hi + 1:] if len(r) == len(hdr)]
reasons = [h for h in hdr if h.startswith('stall_') and 'Not Issued' not in h]
f = lambda x: float(x or 0)
tot = sum(f(d['Warp Stall Sampling (All Samples)']) for d in data)
agg = {r: sum(f(d[r]) for d in data) for r in reasons}
print("total samples", tot)
for r, v in sorted(agg.items(), key=lambda kv: -kv[1]):
    if v: print(f"  {r:28s} {v / tot * 100:6.2f}%")
n = int(sys.argv[2]) if len(sys.argv) > 2 else 30
print("top instructions:")
for d in sorted(data, key=lambda d: -f(d['Warp Stall Sampling (All Samples)']))[:n]:
    top = sorted(((f(d[r]), r) for r in reasons), reverse=True)[:3]
    print(f"{f(d['Warp Stall Sampling (All Samples)']) / tot * 100:5.2f}% exec={d['Instructions Executed']:>10} "
          f"{d['Source'][:55]:55s} " + " ".join(f"{r[6:]}={v / tot * 100:.2f}" for v, r in top if v))
