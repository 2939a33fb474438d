python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
python -m pytest tests/test_gpu_parity.py -q -x -k "trajectory or c4_warm" > gpurun_out/pt.txt 2>&1
for nt in 512 128; do for wd in 4 6 8; do
  for w in c3 c4; do echo "nt=$nt wd4=$wd $w $(BOIDS_SYM_NT=$nt BOIDS_SYM_WD4=$wd python bench.py --workload $w --no-cpu-baseline --no-e2e 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print(d['ms_per_step'], d['kernel_profile_ms'])")"; done
done; done
