set -x
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_final5.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_final5.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_final5.log 2>&1
timeout 600 python bench.py > gpurun_out/bench_final5.log 2>&1
timeout 600 python tools/suite.py smsweep > gpurun_out/smsweep.json 2> gpurun_out/smsweep.err
for f in gpurun_out/pytest_final5.log gpurun_out/smoke_final5.log gpurun_out/bench_final5.log; do tail -n 2 $f | cut -c1-300; done
