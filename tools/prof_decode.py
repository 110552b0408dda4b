"""Profiling driver: run GPT-2s (or another config) decode tasks on one partition.

    python tools/prof_decode.py --sms 12 --tasks 2 [--cfg gpt2s] [--layers N]

Used under ncu (`-k regex:decode_kernel -s 1 -c 1`) to capture one warm launch.
"""
import argparse
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_dhakalrwercfm23_b200 import mx  # noqa: E402
from workloads.configs import DECODE_CFGS  # noqa: E402
from workloads.inputs import prompt_tokens  # noqa: E402
from paper_conf_sc_dhakalrwercfm23_b200.metrics import decode_task_bytes  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--sms", type=int, default=12)
ap.add_argument("--tasks", type=int, default=2)
ap.add_argument("--cfg", default="gpt2s")
ap.add_argument("--layers", type=int, default=0)
ap.add_argument("--batch", type=int, default=1)
ap.add_argument("--P", type=int, default=16)
ap.add_argument("--G", type=int, default=32)
ap.add_argument("--vocab", type=int, default=0)
ap.add_argument("--dff", type=int, default=0)
a = ap.parse_args()
cfg = DECODE_CFGS[a.cfg]
if a.layers:
    cfg = cfg.with_layers(a.layers)
from dataclasses import replace  # noqa: E402
if a.vocab:
    cfg = replace(cfg, vocab=a.vocab)
if a.dff:
    cfg = replace(cfg, d_ff=a.dff)
mx.mx_init([0])
p = mx.part_create(0, a.sms, 24 << 30)
fn = mx.fn_register(mx.decode_desc(cfg, max_batch=a.batch))
mx.fn_load(fn, p)
for k in range(a.tasks):
    t = mx.decode_task(fn, prompt_tokens(k + 1, a.batch, a.P, cfg.vocab), a.G)
    h0 = time.perf_counter()
    mx.fn_submit(p, t)
    r = mx.fn_wait(t)
    gbs = decode_task_bytes(cfg, a.batch, a.P, a.G) / r['kernel_ns']
    print(f"task {k}: status {r['status']} kernel {r['kernel_ns'] / 1e6:.3f} ms  {gbs:.1f} GB/s "
          f"({gbs / mx.part_query(p)['n_ctas']:.1f} GB/s/SM) "
          f"wall {(time.perf_counter() - h0) * 1e3:.1f} ms")
if os.environ.get("MX_DECODE_PROF") == "1":
    n = mx.part_query(p)["n_ctas"]
    pr = mx.decode_profile(p, 2 * n).astype(float).reshape(n, 16)
    names = {0: "total", 1: "grid_barrier", 2: "stage_input", 3: "mma_wait_full", 4: "gemv(mma+epi)",
             5: "attention", 6: "producer_wait", 7: "mma_wait_acc", 8: "epi_wait_tfull",
             9: "mma_wait_operand"}
    tot = pr[:, 0].mean()
    for i, nm in names.items():
        print(f"  {nm:16s} mean {pr[:, i].mean() / 1e6:9.2f} Mcyc  ({pr[:, i].mean() / tot * 100:5.1f}%)"
              f"  min {pr[:, i].min() / 1e6:8.2f} max {pr[:, i].max() / 1e6:8.2f}")
    # timeline of layer L/2 at step S/2 (globaltimer ns, words 2560.. of the buffer)
    import numpy as np
    full = mx.decode_profile(p, 1024).reshape(-1).astype(np.int64)
    tl = full[2560:2560 + n * 5 * 6].reshape(n, 5, 6)
    base = tl[:, 0, 0][tl[:, 0, 0] > 0].min() if (tl[:, 0, 0] > 0).any() else 0
    print("timeline (us from the first phase start; median/max over CTAs)")
    print("  ph  start(min..max)   ready-start  mma_end(med/max)  epi_end(med/max)  arrive(min..max)"
          "  exit(min..max)  exit-lastarrive")
    for ph in range(5):
        t = tl[:, ph, :].astype(float)
        if not (t[:, 0] > 0).any():
            continue
        r = (t - base) / 1e3
        arr, ex = r[:, 4], r[:, 5]
        print(f"  {ph}  {r[:, 0].min():7.2f}..{r[:, 0].max():7.2f}  {np.median(r[:, 1] - r[:, 0]):6.2f}"
              f"  {np.median(r[:, 2]):7.2f}/{r[:, 2].max():7.2f}  {np.median(r[:, 3]):7.2f}/{r[:, 3].max():7.2f}"
              f"  {arr.min():7.2f}..{arr.max():7.2f}  {ex.min():7.2f}..{ex.max():7.2f}  {ex.min() - arr.max():6.2f}")
    os.makedirs("gpurun_out", exist_ok=True)
    np.save(os.environ.get("MX_TL_OUT", f"gpurun_out/tl_{a.cfg}_{a.sms}sm_b{a.batch}.npy"), tl)
mx.part_destroy(p)
mx.mx_shutdown()
