timeout 600 python -m pytest tests -m gpu -x -q -k "mpnn or mixed" > gpurun_out/pytest_mpnn2.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_mpnn2.log
tail -n 3 gpurun_out/pytest_mpnn2.log
for s in 4 20 148; do timeout 120 python tools/prof_mpnn.py --sms $s --tasks 4 | tail -n 1; done > gpurun_out/mpnn_tc2.txt 2>&1
cat gpurun_out/mpnn_tc2.txt
