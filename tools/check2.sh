python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pt.txt 2>&1
python tools/diag_stats.py c4 > gpurun_out/diag.txt 2>&1
for w in c5; do timeout 300 python bench.py --workload $w --no-cpu-baseline --no-e2e > gpurun_out/bench_$w.json 2>gpurun_out/bench_$w.err; done
timeout 300 python bench.py --workload c5 --think 10 --no-cpu-baseline --no-e2e > gpurun_out/bench_c5_think.json 2>/dev/null
