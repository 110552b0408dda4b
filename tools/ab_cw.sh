# A/B: consumer warps per CTA (12 = 128-register cap with spills; 11 -> 168 regs; 7 -> 255 regs)
for spec in "gpt2s 4 1" "gpt2s 12 1" "gpt2s 148 1" "llama7b 148 1" "llama7b 36 1" "gpt2s 4 2"; do
  set -- $spec
  for v in cur cw11 cw7; do
    if [ $v = cur ]; then L=""; else L=ab/libmx_$v.so; fi
    MX_LIB=$L timeout 300 python tools/prof_decode.py --cfg $1 --sms $2 --batch $3 --tasks 2 2>&1 | tail -1 | sed "s/^/$1 sm$2 b$3 $v: /"
  done
done > gpurun_out/ab_cw.txt
cat gpurun_out/ab_cw.txt
