python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
mkdir -p gpurun_out/cmp; python tools/diag_stats.py c4 > gpurun_out/diag.txt 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_route -s 2 -c 1 -o gpurun_out/cmp/route_c4 python bench.py --workload c4 --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/cmp/route.log 2>&1
