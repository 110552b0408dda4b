#!/bin/bash
# Round 2 perf snapshot: default bench line + single-instance decode timings.
mkdir -p gpurun_out
timeout 900 python bench.py ${BENCH_ARGS} > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
for spec in "gpt2s 4 1" "gpt2s 148 1" "llama7b 148 1" "llama7b 148 8" "llama7b 36 1" "llama7b 36 8"; do
  set -- $spec
  timeout 300 python tools/prof_decode.py --cfg $1 --sms $2 --batch $3 --tasks 3 > gpurun_out/prof_${1}_${2}sm_b${3}.txt 2>&1
  echo "$spec: $(tail -n 1 gpurun_out/prof_${1}_${2}sm_b${3}.txt)"
done
