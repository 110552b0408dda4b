# A/B on one box: HEAD (ab/a0) vs the current build vs the MX_V4=8 variant
for spec in "gpt2s 4 1" "gpt2s 148 1" "llama7b 148 1" "llama7b 36 1" "llama7b 148 8" "llama7b 36 4"; do
  set -- $spec
  for v in a0 cur v8; do
    case $v in
      a0) (cd ab/a0 && timeout 300 python tools/prof_decode.py --cfg $1 --sms $2 --batch $3 --tasks 2) ;;
      cur) timeout 300 python tools/prof_decode.py --cfg $1 --sms $2 --batch $3 --tasks 2 ;;
      v8) MX_LIB=ab/libmx_v8.so timeout 300 python tools/prof_decode.py --cfg $1 --sms $2 --batch $3 --tasks 2 ;;
    esac 2>&1 | tail -1 | sed "s/^/$1 sm$2 b$3 $v: /"
  done
done > gpurun_out/ab_stage.txt
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu2.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu2.log
cat gpurun_out/ab_stage.txt; tail -3 gpurun_out/pytest_gpu2.log
