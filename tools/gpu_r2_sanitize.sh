#!/bin/bash
# compute-sanitizer (memcheck / racecheck / synccheck) on small decode and MPNN parity runs
# (incl. the distributed K segments + key-block split attention case).
mkdir -p gpurun_out
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in memcheck racecheck synccheck; do
  timeout 900 $CS --tool $tool --print-limit 20 --error-exitcode 17 \
    python -m pytest -q -x tests/test_gpu_parity.py -k "c1_tiny or mpnn_parity or tensor_core_batches or chained_vs_distributed_small" \
    > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$? $(grep -E 'ERROR SUMMARY|passed|failed' gpurun_out/sanitize_$tool.log | tail -n 2 | tr '\n' ' ')"
done
