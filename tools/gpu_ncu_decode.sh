timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:decode_kernel -c 120 --csv --log-file gpurun_out/launches.csv python bench.py --steps 1 --warmup 0 --sweep "" --layout 37 --no-cpu-baseline --no-n3 > gpurun_out/ncu_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:decode_kernel -s 2 -c 1 -o gpurun_out/decode_gpt2s_4sm_cw11 python tools/prof_decode.py --sms 4 --tasks 3 > gpurun_out/ncu_full.log 2>&1
tail -n 3 gpurun_out/ncu_full.log; ls -la gpurun_out/*.ncu-rep
