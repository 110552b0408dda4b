#!/bin/bash
# Round 2 check: unfiltered ncu launch list of smoke() (as the driver runs it) + the GPU test suite.
mkdir -p gpurun_out
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 1000 --csv \
   --log-file gpurun_out/launches_smoke.csv python -c 'import __graft_entry__ as g; g.smoke()' > gpurun_out/ncu_smoke.log 2>&1
echo "ncu_smoke rc=$?"
timeout 1500 python -m pytest tests -m gpu -x -q ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1
echo "pytest rc=$?"; tail -n 5 gpurun_out/pytest_gpu.log
