for spec in "llama7b 148 8" "llama7b 36 8" "llama7b 148 4" "llama7b 36 4" "llama7b 148 1"; do
  set -- $spec
  for v in head cur; do
    if [ $v = cur ]; then L=""; else L=ab/libmx_$v.so; fi
    MX_LIB=$L timeout 300 python tools/prof_decode.py --cfg $1 --sms $2 --batch $3 --tasks 2 2>&1 | tail -1 | sed "s/^/$1 sm$2 b$3 $v: /"
  done
done > gpurun_out/ab_stagevec.txt
timeout 600 python -m pytest tests -m gpu -x -q -k "tensor_core or batch8 or split_k or identical" > gpurun_out/pytest_sv.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_sv.log
cat gpurun_out/ab_stagevec.txt; tail -n 2 gpurun_out/pytest_sv.log
