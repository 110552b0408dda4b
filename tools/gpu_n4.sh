timeout 900 python -m pytest tests/test_gpu_mpnn_train.py -x -q > gpurun_out/pytest_n4.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_n4.log
tail -n 30 gpurun_out/pytest_n4.log
for s in 4 20 148; do timeout 300 python tools/prof_mpnn_train.py --sms $s --tasks 3; done > gpurun_out/n4_timing.txt 2>&1
cat gpurun_out/n4_timing.txt
