set -x
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_final4.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_final4.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_final4.log 2>&1
timeout 600 python bench.py > gpurun_out/bench_final4.log 2>&1
timeout 600 python bench.py --cpu-suite > gpurun_out/d6.json 2> gpurun_out/d6.err
timeout 600 python tools/suite.py n3 > gpurun_out/n3.json 2> gpurun_out/n3.err
for f in gpurun_out/pytest_final4.log gpurun_out/smoke_final4.log gpurun_out/d6.err gpurun_out/n3.err; do tail -n 2 $f | cut -c1-300; done
