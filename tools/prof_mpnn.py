"""Run IP-emulator (MPNN) tasks of 1024 molecules on one partition (profiling driver)."""
import argparse
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_dhakalrwercfm23_b200 import mx  # noqa: E402
from workloads.configs import MPNN  # noqa: E402
from workloads.inputs import molecules  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--sms", type=int, default=12)
ap.add_argument("--tasks", type=int, default=3)
ap.add_argument("--mols", type=int, default=1024)
a = ap.parse_args()
mx.mx_init([0])
p = mx.part_create(0, a.sms, 1 << 30)
fn = mx.fn_register(mx.mpnn_desc(MPNN, a.mols, a.mols * 32, a.mols * 64))
mx.fn_load(fn, p)
mols = [molecules(k + 1, a.mols) for k in range(a.tasks)]
for k in range(a.tasks):
    t = mx.mpnn_task(fn, mols[k])
    h0 = time.perf_counter()
    mx.fn_submit(p, t)
    h1 = time.perf_counter()
    r = mx.fn_wait(t)
    h2 = time.perf_counter()
    print(f"mpnn task {k}: status {r['status']} kernel {r['kernel_ns'] / 1e6:.3f} ms "
          f"wall {(h2 - h0) * 1e3:.3f} ms (fn_submit {(h1 - h0) * 1e3:.3f} ms, "
          f"submit->kernel start {(r['t_start_ns'] - r['t_submit_ns']) / 1e6:.3f} ms) "
          f"-> {5.307e9 / (r['kernel_ns'] * 1e-9) / 1e12:.2f} TFLOP/s algorithmic")
mx.part_destroy(p)
mx.mx_shutdown()
