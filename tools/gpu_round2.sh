set -x
timeout 900 python tools/suite.py c3 --tasks 24 > gpurun_out/c3.json 2> gpurun_out/c3.err
export MX_DECODE_PROF=1
for spec in "llama7b 148 1" "llama7b 36 8" "llama7b 36 4"; do set -- $spec; timeout 300 python tools/prof_decode.py --cfg $1 --sms $2 --batch $3 --tasks 2 > gpurun_out/prof_${1}_${2}sm_b${3}.txt 2>&1; done
unset MX_DECODE_PROF
MX_TRACE_RESIZE=1 timeout 600 python tools/suite.py c5 > gpurun_out/c5.json 2> gpurun_out/c5.err
timeout 600 python bench.py > gpurun_out/bench.log 2>&1
tail -n 2 gpurun_out/*.err
