#!/bin/bash
# One measurement pass on the GPU box (run under gpurun).  Writes gpurun_out/$TAG/*.
TAG=${TAG:-r1}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { echo BUILD FAILED; exit 1; }
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv > $OUT/smi_before.csv
timeout 600 python -m pytest tests -m gpu -x -q > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1
for w in ${WORKLOADS:-c4 c3 c2 c1 c5}; do
  timeout 600 python bench.py --workload $w > $OUT/bench_$w.json 2> $OUT/bench_$w.err
done
for w in c3 c4 c5; do
  timeout 600 python bench.py --workload $w --think 10 --no-cpu-baseline > $OUT/bench_${w}_think10.json 2> $OUT/bench_${w}_think10.err
done
timeout 300 python bench.py --impl reference > $OUT/bench_reference.json 2>&1
if [ -z "$NO_NCU" ]; then
for w in ${NCU_WORKLOADS:-c4 c3 c5}; do
  K=k_sym; [ $w = c5 ] && K=k_grid; [ $w = c1 ] && K=k_scan
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_$w.csv \
     python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/ncu_launch_$w.log 2>&1
  timeout 1200 ncu --set full --clock-control none --import-source on -k $K -s 2 -c 1 -o $OUT/prof_$w \
     python bench.py --workload $w --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/ncu_full_$w.log 2>&1
done
timeout 900 ncu --set full --clock-control none -k regex:k_apply -s 2 -c 1 -o $OUT/prof_c5think10apply \
   python bench.py --workload c5 --think 10 --steps 1 --warmup 11 --no-cpu-baseline --no-e2e > $OUT/ncu_apply.log 2>&1
fi
ls -la $OUT
