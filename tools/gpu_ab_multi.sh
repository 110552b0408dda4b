#!/bin/bash
# A/B/C... of decode builds on one box: LIBS (space-separated .so paths), PERF_SPECS as gpu_ab_decode.sh.
mkdir -p gpurun_out
IFS=";" read -ra PL <<< "${PERF_SPECS:-gpt2s 4 1;llama7b 148 1;llama7b 148 8;llama7b 36 1}"
for rep in 1 2; do
  for spec in "${PL[@]}"; do
    set -- $spec
    for lib in $LIBS; do
      r=$(MX_LIB=$lib timeout 300 python tools/prof_decode.py --cfg $1 --sms $2 --batch $3 --tasks 3 2>&1 | tail -n 1)
      echo "$spec $(basename $lib): $r"
    done
  done
done
