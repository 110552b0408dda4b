# A/B: fused attention on every grid (cur) vs only on grids <= 32 / 64 CTAs
for spec in "gpt2s 148 1" "gpt2s 76 1" "gpt2s 40 1" "gpt2s 24 1"; do
  set -- $spec
  for v in cur fuse32 fuse64; do
    if [ $v = cur ]; then L=""; else L=ab/libmx_$v.so; fi
    MX_LIB=$L timeout 300 python tools/prof_decode.py --cfg $1 --sms $2 --batch $3 --tasks 3 2>&1 | tail -1 | sed "s/^/$1 sm$2 b$3 $v: /"
  done
done > gpurun_out/ab_fuse.txt
MX_LIB=ab/libmx_fuse32.so timeout 600 python -m pytest tests -m gpu -x -q -k "identical or c1_tiny or ragged or gpt2s_one" > gpurun_out/pytest_fuse.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_fuse.log
cat gpurun_out/ab_fuse.txt; tail -n 2 gpurun_out/pytest_fuse.log
