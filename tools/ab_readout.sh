# A/B of the MPNN readout change (8-molecule batch, no per-molecule system fence,
# vectorised r reads): kernel time per 1024-molecule task, then cycle buckets.
timeout 600 python -m pytest tests -m gpu -x -q -k "mpnn or mixed" > gpurun_out/pytest_readout.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_readout.log
tail -n 2 gpurun_out/pytest_readout.log
for s in 4 20 148; do for v in base new base new; do
  MX_LIB=abx/libmx_$v.so timeout 120 python tools/prof_mpnn.py --sms $s --tasks 5 2>&1 | tail -n 1 | sed "s/^/sm$s $v: /"
done; done
for s in 4 148; do for v in base new; do
  MX_LIB=abx/libmx_${v}_prof.so timeout 120 python tools/prof_mpnn.py --sms $s --tasks 2 2>&1 | tail -n 1 | sed "s/^/sm$s $v prof: /"
done; done
