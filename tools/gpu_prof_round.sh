set -x
export MX_DECODE_PROF=1
for spec in "llama7b 148 1" "llama7b 36 1" "llama7b 36 8" "gpt2s 4 1"; do set -- $spec; timeout 300 python tools/prof_decode.py --cfg $1 --sms $2 --batch $3 --tasks 2 > gpurun_out/prof_${1}_${2}sm_b${3}.txt 2>&1; done
unset MX_DECODE_PROF
MX_TRACE_RESIZE=1 timeout 600 python tools/suite.py c5 > gpurun_out/c5.json 2> gpurun_out/c5.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:decode_kernel -c 120 --csv --log-file gpurun_out/launches.csv python bench.py --steps 1 --warmup 0 --sweep "" --layout 37 --no-cpu-baseline > gpurun_out/ncu_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:decode_kernel -s 2 -c 1 -o gpurun_out/decode_gpt2s_4sm python tools/prof_decode.py --sms 4 --tasks 3 > gpurun_out/ncu_full.log 2>&1
ls -la gpurun_out
