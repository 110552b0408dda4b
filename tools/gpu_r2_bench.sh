#!/bin/bash
# Round 2: the default bench line (as the driver runs it) + nvidia-smi clocks.
mkdir -p gpurun_out
timeout 900 python bench.py ${BENCH_ARGS} > gpurun_out/bench.json 2> gpurun_out/bench.err
echo "bench rc=$?"; tail -c 600 gpurun_out/bench.json
