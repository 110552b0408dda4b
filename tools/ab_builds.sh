# A/B of the MPNN neighbour-sum gathers interleaved over a thread's 4 items
timeout 600 python -m pytest tests -m gpu -x -q -k "mpnn or mixed or train" > gpurun_out/pytest_builds.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_setup.log
tail -n 2 gpurun_out/pytest_builds.log
for s in 4 20 148; do for v in r2 new r2 new; do
  MX_LIB=abx/libmx_$v.so timeout 120 python tools/prof_mpnn.py --sms $s --tasks 5 2>&1 | tail -n 1 | sed "s/^/sm$s $v: /"
done; done
for s in 4 148; do for v in r2 new; do
  MX_LIB=abx/libmx_${v}_prof.so timeout 120 python tools/prof_mpnn.py --sms $s --tasks 2 2>&1 | tail -n 1 | sed "s/^/sm$s $v prof: /"
done; done
