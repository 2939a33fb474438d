#!/bin/bash
# compute-sanitizer pass over every kernel path (run under gpurun): writes $OUT/*.txt
OUT=${OUT:-gpurun_out/san}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in racecheck synccheck memcheck initcheck; do
  for p in ${PATHS:-sym scan small fused grid route gridbig scanbig symshard spatial}; do
    timeout 900 $CS --tool $tool --print-limit 20 python tools/racecheck_paths.py $p > $OUT/${tool}_$p.txt 2>&1
    echo "$tool $p rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|Error|ok ' $OUT/${tool}_$p.txt | tail -2 | tr '\n' ' ')"
  done
done
