#!/bin/bash
# Round 2: the measurement suite on the current build.
mkdir -p gpurun_out
for c in smsweep "c3 --tasks 24" c4 c5 modes n3; do
  name=$(echo $c | cut -d' ' -f1)
  timeout 1200 python tools/suite.py $c > gpurun_out/suite_$name.json 2> gpurun_out/suite_$name.err
  echo "$name rc=$? $(head -c 300 gpurun_out/suite_$name.json)"
done
