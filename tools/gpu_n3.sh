timeout 600 python -m pytest tests/test_gpu_shared_weights.py -x -q > gpurun_out/pytest_n3.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_n3.log
tail -n 15 gpurun_out/pytest_n3.log
timeout 1200 python tools/suite.py n3 > gpurun_out/n3.json 2> gpurun_out/n3.err
tail -n 3 gpurun_out/n3.err
python -c "
import json; d=json.load(open('gpurun_out/n3.json'))
for r in d['rows']: print({k: r.get(k) for k in ('model','partitions','mode','tasks_per_s','hbm_frac_algorithmic','load_s','hbm_held_gib','p50_ms','skipped')})"
