# tensor-core path with 11 consumer warps: split 3 / 4 / 5 vs the current 12-warp split-4 build
for spec in "llama7b 148 8" "llama7b 36 8" "llama7b 148 4" "llama7b 36 4"; do
  set -- $spec
  for v in cur cw11s3 cw11s4 cw11s5; do
    if [ $v = cur ]; then L=""; else L=ab/libmx_$v.so; fi
    MX_LIB=$L timeout 300 python tools/prof_decode.py --cfg $1 --sms $2 --batch $3 --tasks 2 2>&1 | tail -1 | sed "s/^/$1 sm$2 b$3 $v: /"
  done
done > gpurun_out/ab_cw_tc.txt
cat gpurun_out/ab_cw_tc.txt
