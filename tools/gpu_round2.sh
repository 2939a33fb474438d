#!/bin/bash
# Round-2 measurement pass on the GPU box (run under gpurun).  Writes gpurun_out/$TAG/*.
TAG=${TAG:-r2}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { echo BUILD FAILED; exit 1; }
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv > $OUT/smi_before.csv
if [ -z "$NO_TESTS" ]; then
  timeout 900 python -m pytest tests -m gpu -x -q > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1
fi
for w in ${WORKLOADS:-c4 c5 c3 c2 c1}; do
  KT=live; case $w in c1|c2|c3) KT=pass;; esac
  timeout 600 python bench.py --workload $w --kernel-timing $KT > $OUT/bench_$w.json 2> $OUT/bench_$w.err
done
for w in ${THINK_WL:-c3 c4 c5}; do
  timeout 600 python bench.py --workload $w --think 10 --no-cpu-baseline > $OUT/bench_${w}_think10.json 2> $OUT/bench_${w}_think10.err
done
timeout 300 python bench.py --impl reference > $OUT/bench_reference.json 2>$OUT/bench_reference.err
for w in c4 c5; do
  timeout 600 python bench.py --workload $w --force-shard --no-cpu-baseline > $OUT/bench_${w}_force_shard.json 2> $OUT/bench_${w}_force_shard.err
  timeout 900 python tools/rank_emulation.py --workload $w --ranks 1 2 4 8 > $OUT/ranks_$w.json 2> $OUT/ranks_$w.err
done
if [ -z "$NO_NCU" ]; then
for w in ${NCU_WORKLOADS:-c2 c3 c4 c5}; do
  K=k_sym; [ $w = c5 ] && K=k_grid; case $w in c1|c2) K=k_small;; esac
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_$w.csv \
     python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/ncu_launch_$w.log 2>&1
  timeout 1200 ncu --set full --clock-control none --import-source on -k $K -s 3 -c 1 -o $OUT/${w}_$K \
     python bench.py --workload $w --steps 1 --warmup 4 --no-cpu-baseline --no-e2e > $OUT/ncu_full_$w.log 2>&1
done
timeout 900 ncu --set full --clock-control none -k regex:k_apply -s 2 -c 1 -o $OUT/c5think10_k_apply \
   python bench.py --workload c5 --think 10 --steps 1 --warmup 11 --no-cpu-baseline --no-e2e > $OUT/ncu_apply.log 2>&1
timeout 900 ncu --set full --clock-control none -k regex:k_bin -s 6 -c 4 -o $OUT/c5_k_bin \
   python bench.py --workload c5 --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/ncu_bin.log 2>&1
fi
ls -la $OUT
