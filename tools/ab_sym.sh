#!/bin/bash
# A/B of k_sym variants on the GPU box (development aid): parity subset, then bench lines.
# usage: OUT=gpurun_out/x VARS="BOIDS_SYM_HALVES=1 BOIDS_SYM_HALVES=2" WL="c3 c4" bash tools/ab_sym.sh
OUT=${OUT:-gpurun_out/ab}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { echo BUILD FAILED; tail $OUT/build.log; exit 1; }
for v in ${VARS:-X=0}; do
  env $v timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "${TK:-trajectory or c3 or c4 or large}" > $OUT/pytest_$v.log 2>&1
  echo "$v $(tail -1 $OUT/pytest_$v.log)"
  for w in ${WL:-c3 c4}; do
    for rep in 1 2; do
      env $v python bench.py --workload $w --no-cpu-baseline --no-e2e > $OUT/bench_${w}_${v}_$rep.json 2>/dev/null
      python -c "
import json; d=json.load(open('$OUT/bench_${w}_${v}_$rep.json')); r=d['roofline']
print('$w $v rep$rep', '%.4g'%d['value'], 'ms/step %.4f'%d['ms_per_step'], 'frac %.3f'%r['frac'], 'kern %.4f'%r['kernel_ms_per_launch'], d['kernel_profile_ms'])"
    done
  done
done
