# A/B on one box: the current build vs ab/a0 (commit a0d214b), GPT-2s decode on 4 SMs
(cd ab/a0 && python tools/prof_decode.py --sms 4 --tasks 3) > gpurun_out/ab_a0_prof.txt 2>&1
python tools/prof_decode.py --sms 4 --tasks 3 > gpurun_out/ab_cur_prof.txt 2>&1
(cd ab/a0 && python tools/prof_decode.py --sms 4 --tasks 3) >> gpurun_out/ab_a0_prof.txt 2>&1
python tools/prof_decode.py --sms 4 --tasks 3 >> gpurun_out/ab_cur_prof.txt 2>&1
tail -n 3 gpurun_out/ab_*prof.txt
