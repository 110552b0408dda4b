timeout 600 python -m pytest tests -m gpu -x -q -k "mpnn or mixed" > gpurun_out/pytest_mpnn3.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_mpnn3.log
tail -n 2 gpurun_out/pytest_mpnn3.log
for s in 4 20 148; do timeout 120 python tools/prof_mpnn.py --sms $s --tasks 3 2>&1 | tail -n 1; done
for s in 4 148; do MX_LIB=ab/libmx_mprof.so timeout 120 python tools/prof_mpnn.py --sms $s --tasks 2 2>&1 | tail -n 1; done
