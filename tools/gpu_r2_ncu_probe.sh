#!/bin/bash
# Round 2: why does an unfiltered ncu launch list stop at the first green-context kernel?
mkdir -p gpurun_out; rm -f gpurun_out/ncu_probe_*
S='import __graft_entry__ as g; g.smoke()'
run() { v=$1; shift; extra=$1; shift
  timeout 300 env "$@" ncu --metrics gpu__time_duration.sum --clock-control none -c 1000 --csv $extra \
     --log-file gpurun_out/ncu_probe_$v.csv python -c "$S" > gpurun_out/ncu_probe_$v.log 2>&1
  echo "$v rc=$? rows=$(grep -c '^"[0-9]' gpurun_out/ncu_probe_$v.csv)" | tee -a gpurun_out/ncu_probe_summary.txt
}
env MX_LAUNCH_PER_CTX=1 python -c "$S" > gpurun_out/ncu_probe_noprof_perctx1.log 2>&1; echo "noprof perctx1 rc=$?" >> gpurun_out/ncu_probe_summary.txt
run perctx1 "" MX_LAUNCH_PER_CTX=1
run perctx2 "" MX_LAUNCH_PER_CTX=2
run fillprim "" MX_FILL_PRIMARY=1
run fillprim_perctx1 "" MX_FILL_PRIMARY=1 MX_LAUNCH_PER_CTX=1
run kfill "-k regex:fill" X=1
run appreplay "--replay-mode application" X=1
run cachenone "--cache-control none" X=1
