# A/B of the MPNN tile set-up change (h0 gather issued with the first loads,
# one edge pass for degrees + per-type counts, bond-type mask in one OR pass)
timeout 600 python -m pytest tests -m gpu -x -q -k "mpnn or mixed" > gpurun_out/pytest_setup.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_setup.log
tail -n 2 gpurun_out/pytest_setup.log
for s in 4 20 148; do for v in r1 new r1 new; do
  MX_LIB=abx/libmx_$v.so timeout 120 python tools/prof_mpnn.py --sms $s --tasks 5 2>&1 | tail -n 1 | sed "s/^/sm$s $v: /"
done; done
for s in 4 148; do for v in r1 new; do
  MX_LIB=abx/libmx_${v}_prof.so timeout 120 python tools/prof_mpnn.py --sms $s --tasks 2 2>&1 | tail -n 1 | sed "s/^/sm$s $v prof: /"
done; done
