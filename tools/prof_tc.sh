export MX_DECODE_PROF=1
for spec in "gpt2s 4 8 prof" "gpt2s 4 1 prof" "gpt2s 4 1 proftcb1" "llama7b 36 8 prof" "gpt2s 4 4 prof"; do
  set -- $spec
  echo "== $1 sm$2 b$3 $4"
  MX_LIB=ab/libmx_$4.so timeout 300 python tools/prof_decode.py --cfg $1 --sms $2 --batch $3 --tasks 2 2>&1 | tail -n 9
done > gpurun_out/prof_tc.txt
cat gpurun_out/prof_tc.txt
