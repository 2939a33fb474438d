#!/bin/bash
# Development pass on the GPU box: build, quick timings (A/B by env), optional GPU tests.
# TAG=... QT="c3 c4" AB="BOIDS_SELECT_P=1" TESTS="-k parity" bash tools/gpu_quick.sh
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1 || { echo BUILD FAIL; exit 1; }
mkdir -p gpurun_out/$TAG
python tools/quick_time.py ${QT:-c3 c4} > gpurun_out/$TAG/qt.txt 2>&1
for ab in $AB; do echo "== $ab" >> gpurun_out/$TAG/qt.txt; env $ab python tools/quick_time.py ${QT:-c3 c4} >> gpurun_out/$TAG/qt.txt 2>&1; done
if [ -n "$TESTS" ]; then timeout 900 python -m pytest tests -m gpu -x -q $TESTS > gpurun_out/$TAG/pytest.txt 2>&1; echo rc=$? >> gpurun_out/$TAG/pytest.txt; fi
