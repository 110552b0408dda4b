# A/B of the balanced tile packing for MPNN inference (r5 = 128-atom greedy only)
timeout 600 python -m pytest tests -m gpu -x -q -k "mpnn or mixed or smoke" > gpurun_out/pytest_pack.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_pack.log
tail -n 2 gpurun_out/pytest_pack.log
for s in 4 20 148; do for v in r5 new r5 new; do
  MX_LIB=abx/libmx_$v.so timeout 120 python tools/prof_mpnn.py --sms $s --tasks 5 2>&1 | tail -n 1 | sed "s/^/sm$s $v: /"
done; done
