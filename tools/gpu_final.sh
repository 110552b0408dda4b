set -x
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_final.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_final.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_final.log 2>&1
timeout 600 python bench.py > gpurun_out/bench_final.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:mpnn_kernel -s 2 -c 1 -o gpurun_out/mpnn_tc_20sm python tools/prof_mpnn.py --sms 20 --tasks 3 > gpurun_out/ncu_mpnn.log 2>&1
timeout 300 python tools/suite.py c4 > gpurun_out/c4.json 2> gpurun_out/c4.err
for f in gpurun_out/pytest_final.log gpurun_out/smoke_final.log gpurun_out/bench_final.log gpurun_out/ncu_mpnn.log; do tail -n 3 $f; done
