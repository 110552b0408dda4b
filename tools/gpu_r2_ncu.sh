#!/bin/bash
# ncu evidence for the decode kernel: one full capture (GPT-2s task, 4-SM partition) -> traffic
# json stamped with the kernel source hash; the bench's launch list (37 x 4-SM partitions).
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:decode_kernel -s 2 -c 1 \
  -o gpurun_out/decode_gpt2s_4sm -f python tools/prof_decode.py --sms 4 --tasks 3 > gpurun_out/ncu_full.log 2>&1
echo "ncu full rc=$?"
python tools/capture_traffic.py gpurun_out/decode_gpt2s_4sm.ncu-rep > gpurun_out/traffic.log 2>&1; echo "traffic rc=$?"; cat gpurun_out/traffic.log | tail -2
ncu -i gpurun_out/decode_gpt2s_4sm.ncu-rep --page details --csv > gpurun_out/decode_gpt2s_4sm_details.csv 2>/dev/null
ncu -i gpurun_out/decode_gpt2s_4sm.ncu-rep --page raw --csv > gpurun_out/decode_gpt2s_4sm_raw.csv 2>/dev/null
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:decode_kernel -c 120 --csv \
  --log-file gpurun_out/launches_bench37.csv python bench.py --steps 1 --warmup 0 --sweep "" --layout 37 --no-cpu-baseline --no-n3 > gpurun_out/ncu_bench.log 2>&1
echo "ncu launches rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:mpnn_kernel -s 2 -c 1 \
  -o gpurun_out/mpnn_148sm -f python tools/prof_mpnn.py --sms 148 --tasks 3 > gpurun_out/ncu_mpnn.log 2>&1
echo "ncu mpnn rc=$?"
python tools/prof_mpnn.py --sms 148 --tasks 8 > gpurun_out/prof_mpnn_148.txt 2>&1; tail -n 3 gpurun_out/prof_mpnn_148.txt
