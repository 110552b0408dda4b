# MPNN set-up split: global-load round trips vs remap + neighbour-list build
for s in 4 20 148; do MX_LIB=abx/libmx_new_prof.so timeout 120 python tools/prof_mpnn.py --sms $s --tasks 2 2>&1 | tail -n 1 | sed "s/^/sm$s: /"; done
