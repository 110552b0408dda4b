for spec in "llama7b 148 1" "llama7b 36 1" "gpt2s 4 1" "gpt2s 148 1" "llama7b 148 2"; do
  set -- $spec
  for v in cur rv12; do
    if [ $v = cur ]; then L=""; else L=ab/libmx_$v.so; fi
    MX_LIB=$L timeout 300 python tools/prof_decode.py --cfg $1 --sms $2 --batch $3 --tasks 2 2>&1 | tail -1 | sed "s/^/$1 sm$2 b$3 $v: /"
  done
done > gpurun_out/ab_regvals.txt
cat gpurun_out/ab_regvals.txt
