#!/bin/bash
# A/B of the decode kernel on one box: MX_LIB=ab/libmx_base.so (the baseline)
# vs the in-tree libmx.so, interleaved, single-instance task times.
mkdir -p gpurun_out
if [ -n "$TESTS" ]; then
  timeout 1200 python -m pytest $TESTS -m gpu -x -q > gpurun_out/pytest_ab.log 2>&1
  echo "pytest rc=$?"; tail -n 3 gpurun_out/pytest_ab.log
fi
IFS=";" read -ra PL <<< "${PERF_SPECS:-gpt2s 4 1;gpt2s 148 1;llama7b 148 1;llama7b 148 8;llama7b 36 1}"
for rep in 1 2; do
  for spec in "${PL[@]}"; do
    set -- $spec
    for lib in ab/libmx_base.so paper_conf_sc_dhakalrwercfm23_b200/libmx.so; do
      r=$(MX_LIB=$lib timeout 300 python tools/prof_decode.py --cfg $1 --sms $2 --batch $3 --tasks 3 2>&1 | tail -n 1)
      echo "$spec $(basename $lib): $r"
    done
  done
done
if [ -n "$SPECS" ]; then bash tools/gpu_r2_buckets.sh; fi
