"""Summarise ncu captures of a measurement pass into profiles/<tag>/ (tracked).

python tools/summarize_ncu.py gpurun_out/r1b profiles/r1
Writes: <w>_full.txt (key metrics + stall breakdown of the dominant kernel),
<w>_launches.csv (copied launch list) + <w>_launch_share.txt, and updates
profiles/ncu_summary.json (dram bytes per launch, read by bench.py as `traffic`)."""
import csv
import io
import json
import os
import shutil
import subprocess
import sys

src, dst = sys.argv[1], sys.argv[2]
os.makedirs(dst, exist_ok=True)
root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
summ_path = os.path.join(root, "profiles", "ncu_summary.json")
summary = json.load(open(summ_path)) if os.path.exists(summ_path) else {}
KEYS = ["gpu__time_duration.sum", "sm__cycles_elapsed.avg.per_second", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
        "sm__warps_active.avg.per_cycle_active", "launch__registers_per_thread", "launch__grid_size",
        "launch__block_size", "smsp__inst_executed.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "lts__t_bytes.sum", "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
        "sm__sass_thread_inst_executed_op_fadd_pred_on.sum", "sm__sass_thread_inst_executed_op_fmul_pred_on.sum",
        "sm__sass_thread_inst_executed_op_ffma_pred_on.sum"]
UNIT_SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
for f in sorted(os.listdir(src)):
    if not f.endswith(".ncu-rep"):
        continue
    w = f.split("_")[0]  # the workload (c3, c5think10, ...)
    rep = os.path.join(src, f)
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units = rows[0], rows[1]
    out = []
    for row in rows[2:]:
        d = dict(zip(hdr, row))
        u = dict(zip(hdr, units))
        out.append(f"kernel: {d.get('Kernel Name')}")
        for k in KEYS:
            if k in d:
                out.append(f"  {k:70s} {d[k]} {u.get(k, '')}")
        def val(k):
            try:
                return float(d[k]) * UNIT_SCALE.get(u.get(k, "byte"), 1)
            except Exception:
                return None
        rd, wr = val("dram__bytes_read.sum"), val("dram__bytes_write.sum")
        if rd is not None and wr is not None:
            summary.setdefault(w, {})["dram_bytes_per_launch"] = rd + wr
            summary[w]["kernel"] = d.get("Kernel Name")
            summary[w]["source"] = os.path.relpath(os.path.join(dst, f"{w}_full.txt"), root)
    srcpage = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv"], capture_output=True, text=True).stdout
    tmp = os.path.join(dst, f"_{w}_src.csv")
    open(tmp, "w").write(srcpage)
    stalls = subprocess.run([sys.executable, os.path.join(root, "tools", "ncu_src.py"), tmp, "25"],
                            capture_output=True, text=True).stdout
    os.remove(tmp)
    open(os.path.join(dst, f"{w}_full.txt"), "w").write("\n".join(out) + "\n\nstall sampling (source page):\n" + stalls)
for f in sorted(os.listdir(src)):
    if f.startswith("launches_") and f.endswith(".csv"):
        w = f[len("launches_"):-4]
        shutil.copy(os.path.join(src, f), os.path.join(dst, f"{w}_launches.csv"))
        lines = open(os.path.join(src, f)).read().splitlines()
        hi = [i for i, l in enumerate(lines) if l.startswith('"ID"')]
        if not hi:
            continue
        rr = list(csv.DictReader(lines[hi[0]:]))
        tot, per = 0.0, {}
        for r in rr:
            if r.get("Metric Name") != "gpu__time_duration.sum":
                continue
            v = float(r["Metric Value"].replace(",", ""))
            if r.get("Metric Unit") in ("usecond", "us"):
                v *= 1e3
            elif r.get("Metric Unit") in ("msecond", "ms"):
                v *= 1e6
            name = r["Kernel Name"].split("(")[0]
            per[name] = per.get(name, 0.0) + v
            tot += v
        txt = [f"{k:60s} {v / 1e3:12.1f} us  {v / tot * 100:5.1f}%" for k, v in sorted(per.items(), key=lambda kv: -kv[1])]
        open(os.path.join(dst, f"{w}_launch_share.txt"), "w").write(
            "ncu --metrics gpu__time_duration.sum --clock-control none (cold-cache, serialised launches)\n"
            + "\n".join(txt) + "\n")
json.dump(summary, open(summ_path, "w"), indent=1)
print(json.dumps(summary, indent=1))
