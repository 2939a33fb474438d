python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
mkdir -p gpurun_out/cmp
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_grid -s 2 -c 1 -o gpurun_out/cmp/grid_c5 python bench.py --workload c5 --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/cmp/grid.log 2>&1
