#!/bin/bash
# Timelines (profiling builds) of the baseline and the candidate on one box.
mkdir -p gpurun_out
IFS=";" read -ra PL <<< "${SPECS:-gpt2s 148 1;gpt2s 4 1;llama7b 148 1}"
for spec in "${PL[@]}"; do
  set -- $spec
  for lib in ab/libmx_base_prof.so ab/libmx_prof.so; do
    echo "== $spec $(basename $lib)"
    MX_TL_OUT=gpurun_out/tl_$(basename $lib .so)_${1}_${2}_${3}.npy MX_LIB=$lib MX_DECODE_PROF=1 timeout 300 python tools/prof_decode.py --cfg $1 --sms $2 --batch $3 --tasks 2 2>&1 | tail -n 20
  done
done
