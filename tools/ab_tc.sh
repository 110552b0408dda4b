# A/B of the tensor-core GEMV split (MX_TC_SPLIT) and of the tensor-core path at B=1 (MX_TC_MIN_BATCH=1)
run() { # cfg sms batch variant
  if [ $4 = cur ]; then L=""; else L=ab/libmx_$4.so; fi
  MX_LIB=$L timeout 300 python tools/prof_decode.py --cfg $1 --sms $2 --batch $3 --tasks 2 2>&1 | tail -1 | sed "s/^/$1 sm$2 b$3 $4: /"
}
for spec in "llama7b 148 8" "llama7b 36 8" "llama7b 148 4" "gpt2s 4 8"; do
  set -- $spec; for v in cur tcs1 tcs2 tcs12; do run $1 $2 $3 $v; done
done > gpurun_out/ab_tc.txt
for spec in "llama7b 148 1" "llama7b 36 1" "gpt2s 4 1" "gpt2s 148 1" "llama7b 148 2"; do
  set -- $spec; for v in cur tcb1 tcb1s12; do run $1 $2 $3 $v; done
done >> gpurun_out/ab_tc.txt
cat gpurun_out/ab_tc.txt
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_tc.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_tc.log
MX_LIB=ab/libmx_tcb1.so timeout 900 python -m pytest tests -m gpu -x -q -k "decode or parity" > gpurun_out/pytest_tcb1.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_tcb1.log
tail -3 gpurun_out/pytest_tc.log gpurun_out/pytest_tcb1.log
