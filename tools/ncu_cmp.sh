python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
mkdir -p gpurun_out/cmp
python tools/diag_stats.py c3 c4 > gpurun_out/cmp/diag.txt 2>&1
BOIDS_SYM_NT=128 python tools/diag_stats.py c3 > gpurun_out/cmp/diag_c3_128.txt 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_sym -s 2 -c 2 -o gpurun_out/cmp/sym_c4 python bench.py --workload c4 --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/cmp/sym4.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_sym -s 2 -c 2 -o gpurun_out/cmp/sym_c3 python bench.py --workload c3 --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/cmp/sym3.log 2>&1
ls -la gpurun_out/cmp
