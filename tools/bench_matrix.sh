#!/bin/bash
# Bench lines over workloads x option sets (development aid; run under gpurun).
# usage: OUT=gpurun_out/x WL="c1 c2" OPTS="--graph=0 --graph=1+--kernel-timing=pass" bash tools/bench_matrix.sh
# (an option set joins options with '+', an option and its value with '=')
OUT=${OUT:-gpurun_out/bm}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { echo BUILD FAILED; tail $OUT/build.log; exit 1; }
for w in ${WL:-c1 c2 c3 c4}; do
  for o in ${OPTS:---graph=1}; do
    tag=$(echo "$w$o" | tr -c 'a-zA-Z0-9_\n' '_')
    timeout 600 python bench.py --workload $w --no-cpu-baseline ${NOE2E---no-e2e} $(echo $o | tr '+=' '  ') > $OUT/bench_$tag.json 2> $OUT/bench_$tag.err
    python - "$OUT/bench_$tag.json" "$w $o" <<'PY'
import json, sys
try:
    d = json.load(open(sys.argv[1]))
except Exception as e:
    print(sys.argv[2], "FAILED", e); sys.exit()
r = d["roofline"]
e = d.get("e2e") or {}
print(sys.argv[2], "%.4g" % d["value"], "ms/step %.4f" % d["ms_per_step"], "frac %.3f" % r["frac"],
      "kern %.4f" % r["kernel_ms_per_launch"], "e2e %.3g" % e.get("value", 0), "launches", d["gpu_launches"])
PY
    [ -s $OUT/bench_$tag.json ] || tail -3 $OUT/bench_$tag.err
  done
done
