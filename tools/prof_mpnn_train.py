"""Time IP-emulator training steps (N4) of M molecules on one partition."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_dhakalrwercfm23_b200 import mx  # noqa: E402
from paper_conf_sc_dhakalrwercfm23_b200.metrics import mpnn_task_flops  # noqa: E402
from workloads.configs import MPNN  # noqa: E402
from workloads.inputs import molecules, ip_targets  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--sms", type=int, default=20)
ap.add_argument("--tasks", type=int, default=4)
ap.add_argument("--mols", type=int, default=256)
ap.add_argument("--lr", type=float, default=0.5)
a = ap.parse_args()
mx.mx_init([0])
p = mx.part_create(0, a.sms, 4 << 30)
fn = mx.fn_register(mx.mpnn_train_desc(MPNN, a.mols, a.mols * 32, a.mols * 64))
mx.fn_load(fn, p)
for k in range(a.tasks):
    mol = molecules(100 + k, a.mols)
    t = mx.mpnn_train_task(fn, mol, ip_targets(100 + k, a.mols), a.lr)
    mx.fn_submit(p, t)
    r = mx.fn_wait(t)
    fl = 3 * mpnn_task_flops(mol, MPNN.hidden, MPNN.steps)
    print(f"train step {k}: status {r['status']} loss {t.loss[0]:.5f} kernel {r['kernel_ns'] / 1e6:.3f} ms "
          f"-> {fl / (r['kernel_ns'] * 1e-9) / 1e12:.2f} TFLOP/s (3x forward flops)")
mx.part_destroy(p)
mx.mx_shutdown()
