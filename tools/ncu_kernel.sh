#!/bin/bash
# One `ncu --set full` capture of a kernel of a bench workload (development aid).
# usage: bash tools/ncu_kernel.sh <workload> <kernel regex> <out name> [skip]
python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
mkdir -p gpurun_out/cmp
timeout 900 ncu --set full --clock-control none --import-source on -k regex:$2 -s ${4:-3} -c 1 -o gpurun_out/cmp/$3 \
  python bench.py --workload $1 --steps 1 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/cmp/$3.log 2>&1
