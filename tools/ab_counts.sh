# A/B of the per-atom bond-type counts from smem atomics in the remap (r4 = per-atom scan)
timeout 600 python -m pytest tests -m gpu -x -q -k "mpnn or mixed" > gpurun_out/pytest_counts.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_counts.log
tail -n 2 gpurun_out/pytest_counts.log
for s in 4 20 148; do for v in r4 new r4 new; do
  MX_LIB=abx/libmx_$v.so timeout 120 python tools/prof_mpnn.py --sms $s --tasks 5 2>&1 | tail -n 1 | sed "s/^/sm$s $v: /"
done; done
for s in 4 148; do MX_LIB=abx/libmx_new_prof.so timeout 120 python tools/prof_mpnn.py --sms $s --tasks 2 2>&1 | tail -n 1 | sed "s/^/sm$s new prof: /"; done
