for spec in "gpt2s 4 1" "gpt2s 12 1" "gpt2s 148 1" "llama7b 36 1" "gpt2s 4 1" "gpt2s 148 1" "gpt2s 4 2"; do
  set -- $spec
  for v in head cur; do
    if [ $v = cur ]; then L=""; else L=ab/libmx_$v.so; fi
    MX_LIB=$L timeout 300 python tools/prof_decode.py --cfg $1 --sms $2 --batch $3 --tasks 3 2>&1 | tail -1 | sed "s/^/$1 sm$2 b$3 $v: /"
  done
done > gpurun_out/ab_attpf.txt
timeout 600 python -m pytest tests -m gpu -x -q -k "c1_tiny or identical or gpt2s_one or ragged or llama7b or single_token" > gpurun_out/pytest_attpf.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_attpf.log
cat gpurun_out/ab_attpf.txt; tail -n 2 gpurun_out/pytest_attpf.log
