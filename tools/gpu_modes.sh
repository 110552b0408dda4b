timeout 900 python tools/suite.py modes > gpurun_out/modes.json 2> gpurun_out/modes.err; tail -n 2 gpurun_out/modes.err
