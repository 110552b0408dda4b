#!/bin/bash
# Cycle buckets of the decode kernel (profiling build in abx/, MX_PROF_BUCKETS).
mkdir -p gpurun_out abx
MX_DEFS=-DMX_PROF_BUCKETS python -m paper_conf_sc_dhakalrwercfm23_b200.build --out abx/libmx_prof.so --build-dir abx/build_prof > /dev/null
IFS=";" read -ra SPECLIST <<< "${SPECS:-gpt2s 4 1;gpt2s 148 1;llama7b 148 1}"
for spec in "${SPECLIST[@]}"; do
  set -- $spec
  MX_LIB=abx/libmx_prof.so MX_DECODE_PROF=1 timeout 300 python tools/prof_decode.py --cfg $1 --sms $2 --batch $3 --tasks 2 > gpurun_out/buckets_${1}_${2}sm_b${3}.txt 2>&1
  echo "== $spec"; tail -n 10 gpurun_out/buckets_${1}_${2}sm_b${3}.txt
done
