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
    r = mx.fn_wait(t)
    print(f"mpnn task {k}: status {r['status']} kernel {r['kernel_ns'] / 1e6:.3f} ms "
          f"wall {(time.perf_counter() - h0) * 1e3:.1f} ms  -> {5.307e9 / (r['kernel_ns'] * 1e-9) / 1e12:.2f} TFLOP/s algorithmic")
mx.part_destroy(p)
mx.mx_shutdown()
