python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
timeout 600 python -m pytest tests -m gpu -q -x > gpurun_out/pt.txt 2>&1
for rf in 1 0; do BOIDS_ROUTE_FUSED=$rf python tools/diag_stats.py c3 c4 > gpurun_out/diag_rf$rf.txt 2>&1; done
BOIDS_ROUTE_FUSED=0 timeout 600 python -m pytest tests -m gpu -q -x -k "wrap or c4_warm or trajectory" > gpurun_out/pt0.txt 2>&1
