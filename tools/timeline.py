#!/usr/bin/env python3
"""Per-partition timeline of one closed batch of GPT-2s decode tasks: where the
device span goes between kernels (launch gaps, tails, stream serialisation).

    python tools/timeline.py --layout 37 --tasks 700 [--batches 2]
"""
import argparse
import os
import sys
import time

os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

from workloads.configs import GPT2S, LAYOUTS_FILL  # noqa: E402
from workloads.inputs import prompt_tokens  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--layout", type=int, default=37)
    ap.add_argument("--tasks", type=int, default=700)
    ap.add_argument("--batches", type=int, default=2)
    ap.add_argument("--gen", type=int, default=32)
    a = ap.parse_args()
    from paper_conf_sc_dhakalrwercfm23_b200 import mx
    mx.mx_init([0])
    fn = mx.fn_register(mx.decode_desc(GPT2S))
    sizes = LAYOUTS_FILL[a.layout]
    parts = [mx.part_create(0, s, 512 << 20) for s in sizes]
    for p in parts:
        mx.fn_load(fn, p)
    prompts = [prompt_tokens(k, 1, 16, GPT2S.vocab) for k in range(1, a.tasks + 1)]
    eq = len(set(sizes)) == 1
    for b in range(a.batches):
        h0 = time.perf_counter()
        ts = []
        for k in range(1, a.tasks + 1):
            t = mx.decode_task(fn, prompts[k - 1], a.gen)
            mx.fn_submit(parts[(k - 1) % len(parts)] if eq else mx.MX_PART_ANY, t)
            ts.append(t)
        h1 = time.perf_counter()
        res = [mx.fn_wait(t) for t in ts]
        h2 = time.perf_counter()
        t0 = min(r["t_start_ns"] for r in res)
        t1 = max(r["t_end_ns"] for r in res)
        span = (t1 - t0) / 1e6
        by = {}
        for r in res:
            by.setdefault(r["part"], []).append(r)
        busy_tot = 0.0
        lines = []
        for p, rs in sorted(by.items()):
            rs.sort(key=lambda r: r["t_start_ns"])
            busy = sum(r["t_end_ns"] - r["t_start_ns"] for r in rs) / 1e6
            gaps = [(rs[i + 1]["t_start_ns"] - rs[i]["t_end_ns"]) / 1e6 for i in range(len(rs) - 1)]
            busy_tot += busy
            lines.append(f"  part {p:3d}: n={len(rs):3d} first={(rs[0]['t_start_ns'] - t0) / 1e6:8.2f} "
                         f"last_end={(rs[-1]['t_end_ns'] - t0) / 1e6:8.2f} busy={busy:8.2f} "
                         f"gap_mean={np.mean(gaps) if gaps else 0:6.3f} gap_max={max(gaps) if gaps else 0:6.3f} "
                         f"serv={np.mean([(r['t_end_ns'] - r['t_start_ns']) / 1e6 for r in rs]):7.2f} "
                         f"kern={np.mean([r['kernel_ns'] / 1e6 for r in rs]):7.2f}")
        print(f"batch {b}: layout {a.layout} tasks {a.tasks}: submit {1e3 * (h1 - h0):.1f} ms, "
              f"wait {1e3 * (h2 - h1):.1f} ms, device span {span:.1f} ms, "
              f"busy fraction {busy_tot / (len(by) * span):.3f}")
        if b == a.batches - 1:
            print("\n".join(lines))
    mx.mx_shutdown()


if __name__ == "__main__":
    main()
