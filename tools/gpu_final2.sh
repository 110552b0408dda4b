set -x
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_final2.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_final2.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_final2.log 2>&1
timeout 600 python bench.py > gpurun_out/bench_final2.log 2>&1
timeout 600 python tools/suite.py c5 > gpurun_out/c5.json 2> gpurun_out/c5.err
timeout 300 python tools/suite.py c4 > gpurun_out/c4.json 2> gpurun_out/c4.err
for f in gpurun_out/pytest_final2.log gpurun_out/smoke_final2.log gpurun_out/bench_final2.log gpurun_out/c5.err; do tail -n 2 $f | cut -c1-400; done
