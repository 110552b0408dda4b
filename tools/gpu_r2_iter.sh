#!/bin/bash
# Round 2 kernel iteration: parity subset, cycle buckets, single-instance timings, bench.
mkdir -p gpurun_out
if [ -z "$NO_TESTS" ]; then
  timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_iter.log 2>&1
  echo "pytest rc=$?"; tail -n 3 gpurun_out/pytest_iter.log
fi
SPECS="${SPECS:-gpt2s 4 1;gpt2s 148 1;llama7b 148 1}" bash tools/gpu_r2_buckets.sh
IFS=";" read -ra PL <<< "${PERF_SPECS:-gpt2s 4 1;gpt2s 148 1;llama7b 148 1;llama7b 148 8;llama7b 36 8}"
for spec in "${PL[@]}"; do
  set -- $spec
  timeout 300 python tools/prof_decode.py --cfg $1 --sms $2 --batch $3 --tasks 3 > gpurun_out/prof_${1}_${2}sm_b${3}.txt 2>&1
  echo "$spec: $(tail -n 1 gpurun_out/prof_${1}_${2}sm_b${3}.txt)"
done
if [ -n "$BENCH" ]; then
  timeout 900 python bench.py $BENCH > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
  python -c "import json; d=json.load(open('gpurun_out/bench.json')); print(d['value'], d['roofline']['frac'], d['clocks']); [print(s['partitions'], round(s['tasks_per_s'],1), round(s['hbm_frac'],3)) for s in d['partitions_sweep']]"
fi
