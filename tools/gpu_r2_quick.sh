#!/bin/bash
# Round 2 quick check: smoke + decode parity tests (bounded by timeouts).
mkdir -p gpurun_out
timeout 120 python -c 'import __graft_entry__ as g; g.smoke()' > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -n 3 gpurun_out/smoke.log
timeout 1200 python -m pytest tests -m gpu -x -q ${PYTEST_ARGS:-tests/test_gpu_parity.py} > gpurun_out/pytest_quick.log 2>&1
echo "pytest rc=$?"; tail -n 30 gpurun_out/pytest_quick.log
