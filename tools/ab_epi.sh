# A/B of the epilogue skipped by all-padding warps (r6 = every warp)
timeout 600 python -m pytest tests -m gpu -x -q -k "mpnn or mixed or smoke" > gpurun_out/pytest_epi.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_epi.log
tail -n 2 gpurun_out/pytest_epi.log
for s in 4 20 148; do for v in r6 new r6 new; do
  MX_LIB=abx/libmx_$v.so timeout 120 python tools/prof_mpnn.py --sms $s --tasks 5 2>&1 | tail -n 1 | sed "s/^/sm$s $v: /"
done; done
