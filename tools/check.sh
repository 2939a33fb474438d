# quick GPU check (run under gpurun): build, gpu tests, c3/c4 bench both search variants
O=gpurun_out/${TAG:-chk}; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q ${PYTEST_K:+-k "$PYTEST_K"} > $O/pytest.log 2>&1; echo rc=$? >> $O/pytest.log
for w in ${WORKLOADS:-c3 c4}; do
  timeout 300 python bench.py --workload $w --no-e2e --no-cpu-baseline > $O/bench_$w.json 2>$O/bench_$w.err
  [ -n "$NOSYM" ] && timeout 300 python bench.py --workload $w --no-e2e --no-cpu-baseline --no-sym > $O/bench_${w}_nosym.json 2>$O/bench_${w}_nosym.err
done
true
