#!/bin/bash
# A/B of decode variant builds (VARIANTS: space-separated, each a comma-joined MX_DEFS list)
# on a parity selection + single-instance timings.
mkdir -p gpurun_out abx
i=0
for v in ${VARIANTS}; do
  i=$((i+1)); defs=$(echo $v | tr ',' ' '); lib=abx/libmx_v$i.so
  MX_DEFS="$defs" python -m paper_conf_sc_dhakalrwercfm23_b200.build --out $lib --build-dir abx/build_v$i > gpurun_out/ab_build_v$i.log 2>&1 || echo "build $v failed"
  MX_LIB=$lib timeout 600 python -m pytest tests -m gpu -x -q ${PYTEST_SEL:-tests/test_gpu_parity.py} > gpurun_out/ab_pytest_v$i.log 2>&1
  echo "== v$i [$defs]: pytest rc=$? $(tail -n 1 gpurun_out/ab_pytest_v$i.log)"
  IFS=";" read -ra PL <<< "${PERF_SPECS:-gpt2s 4 1}"
  for spec in "${PL[@]}"; do set -- $spec
    MX_LIB=$lib timeout 300 python tools/prof_decode.py --cfg $1 --sms $2 --batch $3 --tasks 3 2>&1 | tail -n 1 | sed "s/^/   $spec: /"
  done
done
