#!/usr/bin/env python3
"""Measurement suite for the SURVEY.md §8(d) rows beyond the headline bench
(bench.py = D2, configs[1]). Each subcommand prints ONE JSON line.

    python tools/suite.py smsweep   # D2b: single-instance SM sweep (Fig. 2 analog)
    python tools/suite.py c3        # D3:  7B-Llama-shaped decode, B 1/2/4/8, 1/2/4 partitions, 14 GiB quotas
    python tools/suite.py c4        # D4:  decode + MPNN co-located on 7 partitions vs 1 (WLAW)
    python tools/suite.py c5        # D5:  10k-task farm, 50/50 mix, part_resize every 1000 submissions
    python tools/suite.py modes     # N1:  partitioned vs unpartitioned-concurrent vs time-shared
    python tools/suite.py n3        # N3:  private vs shared read-only weights (GPT-2s C2, 7B C3)

All inputs are seeded and synthetic (workloads/); weights are generated on the
device from seeds. Times are device %globaltimer stamps (t_start/t_end of each
task); HBM fractions use algorithmic bytes (metrics.decode_task_bytes) over the
device span against MEASURED_PEAKS.json. Output parity of these workloads is
covered by tests/ (-m gpu; the D5 farm's checks in tests/test_gpu_farm_d5.py);
this tool only measures.
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))

import numpy as np  # noqa: E402

from paper_conf_sc_dhakalrwercfm23_b200.metrics import (decode_task_bytes,  # noqa: E402
                                                        mpnn_task_flops, percentiles)
from workloads.configs import GPT2S, LLAMA7B, MPNN, LAYOUTS_FILL  # noqa: E402
from workloads.inputs import molecules, prompt_tokens, shuffle  # noqa: E402

P_LEN, G_LEN = 16, 32
MOLS = 1024


def peak_gbs():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return float(json.load(f)["hbm_gbs"])
    except Exception:
        return 6650.0


def peak_bf16_tflops():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        for k in ("bf16_tflops", "bf16_dense_tflops", "tc_bf16_tflops"):
            if k in d:
                return float(d[k])
    except Exception:
        pass
    return 2250.0


def closed_batch(mx, items):
    """items: list of (part_or_ANY, Task). Submit all at t0, wait all.
    Returns (results, host wall seconds)."""
    h0 = time.perf_counter()
    for part, t in items:
        mx.fn_submit(part, t)
    res = [mx.fn_wait(t) for _, t in items]
    wall = time.perf_counter() - h0
    bad = [r for r in res if r["status"] != 0]
    if bad:
        raise RuntimeError(f"{len(bad)} task(s) failed, first {bad[0]}")
    return res, wall


def span_s(res):
    return (max(r["t_end_ns"] for r in res) - min(r["t_start_ns"] for r in res)) / 1e9


def lat(res):
    comp = [(r["t_end_ns"] - r["t_submit_ns"]) / 1e6 for r in res]
    serv = [(r["t_end_ns"] - r["t_start_ns"]) / 1e6 for r in res]
    c, s = percentiles(comp), percentiles(serv)
    return {"p50_ms": round(c["p50"], 3), "p99_ms": round(c["p99"], 3),
            "service_p50_ms": round(s["p50"], 3), "service_p99_ms": round(s["p99"], 3)}


# ---------------------------------------------------------------------------
# D2b: single instance, SM sweep
# ---------------------------------------------------------------------------

def cmd_smsweep(a, mx):
    cfg = GPT2S
    fn = mx.fn_register(mx.decode_desc(cfg))
    bytes_task = decode_task_bytes(cfg, 1, P_LEN, G_LEN)
    steps = P_LEN + G_LEN - 1
    rows = []
    for sm in [int(x) for x in a.sms.split(",")]:
        p = mx.part_create(0, sm, 512 << 20)
        got = mx.part_query(p)["sm_count"]
        mx.fn_load(fn, p)
        warm = mx.decode_task(fn, prompt_tokens(1, 1, P_LEN, cfg.vocab), G_LEN)
        closed_batch(mx, [(p, warm)])
        items = [(p, mx.decode_task(fn, prompt_tokens(k, 1, P_LEN, cfg.vocab), G_LEN))
                 for k in range(1, a.tasks + 1)]
        res, _ = closed_batch(mx, items)
        kern = float(np.median([r["kernel_ns"] for r in res])) / 1e9
        rows.append({"sm": got, "task_ms": round(kern * 1e3, 3),
                     "step_us": round(kern / steps * 1e6, 2),
                     "gbs": round(bytes_task / kern / 1e9, 1),
                     "gbs_per_sm": round(bytes_task / kern / 1e9 / got, 2),
                     "hbm_frac": round(bytes_task / kern / 1e9 / peak_gbs(), 4)})
        mx.part_destroy(p)
    return {"suite": "D2b smsweep", "workload": "configs[1] GPT-2s decode B=1 P=16 G=32, one "
            "instance alone on a partition of `sm` SMs", "tasks_per_point": a.tasks,
            "peak_gbs": peak_gbs(), "points": rows}


# ---------------------------------------------------------------------------
# D3: 7B-shaped decode, quotas
# ---------------------------------------------------------------------------

def cmd_c3(a, mx):
    cfg = LLAMA7B
    quota = 14 << 30
    fn = mx.fn_register(mx.decode_desc(cfg, max_batch=8))
    # negative: a 12 GiB quota cannot hold 12.55 GiB of weights (D3)
    pn = mx.part_create(0, 8, 12 << 30)
    try:
        mx.fn_load(fn, pn)
        enomem = "loaded (unexpected)"
    except mx.MxError as e:
        enomem = "MX_ENOMEM" if e.code == mx.MX_ENOMEM else f"error {e.code}"
    mx.part_destroy(pn)
    out_rows = []
    batches = [int(x) for x in a.batches.split(",")]
    for n in [int(x) for x in a.layouts.split(",")]:
        sizes = LAYOUTS_FILL[n]
        parts = [mx.part_create(0, s, quota) for s in sizes]
        t0 = time.perf_counter()
        for p in parts:
            mx.fn_load(fn, p)
        load_s = time.perf_counter() - t0
        info = [mx.part_query(p) for p in parts]
        for B in batches:
            warm = [(p, mx.decode_task(fn, prompt_tokens(9000 + i, B, P_LEN, cfg.vocab), 2))
                    for i, p in enumerate(parts)]
            closed_batch(mx, warm)
            items = []
            for k in range(1, a.tasks + 1):
                part = parts[(k - 1) % len(parts)]   # STATIC (k-1) mod P
                items.append((part, mx.decode_task(fn, prompt_tokens(k, B, P_LEN, cfg.vocab),
                                                   G_LEN)))
            res, wall = closed_batch(mx, items)
            sp = span_s(res)
            tb = decode_task_bytes(cfg, B, P_LEN, G_LEN)
            gbs = a.tasks * tb / sp / 1e9
            out_rows.append({"partitions": n, "sms": sizes, "batch": B, "tasks": a.tasks,
                             "tasks_per_s": round(a.tasks / sp, 4),
                             "gen_tok_per_s": round(a.tasks * B * G_LEN / sp, 1),
                             "hbm_gbs": round(gbs, 1), "hbm_frac": round(gbs / peak_gbs(), 4),
                             **lat(res)})
        out_rows[-1]["load_s_all_partitions"] = round(load_s, 3)
        out_rows[-1]["hbm_peak_bytes"] = [i["hbm_peak"] for i in info]
        for p in parts:
            mx.part_destroy(p)
    for r in out_rows:
        base = [x for x in out_rows if x["partitions"] == 1 and x["batch"] == r["batch"]]
        if base:
            r["ratio_vs_1_partition"] = round(r["tasks_per_s"] / base[0]["tasks_per_s"], 3)
    return {"suite": "D3 c3", "workload": "configs[2] 7B-Llama-shaped decode (L32 d4096 "
            "d_ff11008 V32000), P=16 G=32, STATIC placement, quota 14 GiB per partition",
            "quota_12GiB_fn_load": enomem, "peak_gbs": peak_gbs(), "rows": out_rows}


# ---------------------------------------------------------------------------
# D4 / D5: mixed decode + MPNN
# ---------------------------------------------------------------------------

def mixed_items(mx, fd, fm, n_dec, n_mpnn, mol_cache):
    kinds = shuffle([("d", k) for k in range(1, n_dec + 1)] +
                    [("m", k) for k in range(1, n_mpnn + 1)], 42)
    items = []
    for kind, k in kinds:
        if kind == "d":
            items.append(("d", mx.decode_task(fd, prompt_tokens(k, 1, P_LEN, GPT2S.vocab), G_LEN)))
        else:
            mol = mol_cache[(k - 1) % len(mol_cache)]
            items.append(("m", mx.mpnn_task(fm, mol)))
    return items


def class_stats(res, kinds, mflops_mean, n_dec, n_mpnn):
    out = {}
    sp = span_s(res)
    for c, name in (("d", "decode"), ("m", "mpnn")):
        rr = [r for r, k in zip(res, kinds) if k == c]
        if not rr:
            continue
        s = lat(rr)
        s["tasks_per_s"] = round(len(rr) / sp, 3)
        out[name] = s
    dec_bytes = n_dec * decode_task_bytes(GPT2S, 1, P_LEN, G_LEN)
    out["decode_hbm_frac"] = round(dec_bytes / sp / 1e9 / peak_gbs(), 4)
    # share of the mixed run: MPNN flops over the whole makespan (decode dominates it)
    out["mpnn_tflops"] = round(n_mpnn * mflops_mean / sp / 1e12, 2)
    out["mpnn_tc_frac"] = round(out["mpnn_tflops"] / peak_bf16_tflops(), 4)
    # the MPNN kernel itself: one task's flops over its median service time on its partition
    if "mpnn" in out and out["mpnn"]["service_p50_ms"] > 0:
        kt = mflops_mean / (out["mpnn"]["service_p50_ms"] * 1e-3) / 1e12
        out["mpnn_kernel_tflops"] = round(kt, 2)
        out["mpnn_kernel_tc_frac"] = round(kt / peak_bf16_tflops(), 4)
    out["tasks_per_s"] = round(len(res) / sp, 3)
    out["span_s"] = round(sp, 4)
    return out


def cmd_c4(a, mx):
    fd = mx.fn_register(mx.decode_desc(GPT2S))
    fm = mx.fn_register(mx.mpnn_desc(MPNN, MOLS, MOLS * 30, MOLS * 32))
    mol_cache = [molecules(k, MOLS) for k in range(1, a.mol_variants + 1)]
    mfl = float(np.mean([mpnn_task_flops(m, MPNN.hidden, MPNN.steps) for m in mol_cache]))
    rows = {}
    for n in [int(x) for x in a.layouts.split(",")]:
        parts = [mx.part_create(0, s, 1 << 30) for s in LAYOUTS_FILL[n]]
        for p in parts:
            mx.fn_load(fd, p)
            mx.fn_load(fm, p)
        warm = mixed_items(mx, fd, fm, len(parts), len(parts), mol_cache)
        closed_batch(mx, [(mx.MX_PART_ANY, t) for _, t in warm])
        items = mixed_items(mx, fd, fm, a.decode, a.mpnn, mol_cache)
        res, wall = closed_batch(mx, [(mx.MX_PART_ANY, t) for _, t in items])
        rows[str(n)] = {"sms": LAYOUTS_FILL[n], **class_stats(res, [k for k, _ in items], mfl,
                                                              a.decode, a.mpnn),
                        "e2e_tasks_per_s": round(len(res) / wall, 3)}
        for p in parts:
            mx.part_destroy(p)
    if "1" in rows:
        for k, v in rows.items():
            v["ratio_vs_1_partition"] = round(v["tasks_per_s"] / rows["1"]["tasks_per_s"], 3)
    return {"suite": "D4 c4", "workload": f"configs[3]: {a.decode} GPT-2s decode (B1 P16 G32) + "
            f"{a.mpnn} MPNN ({MOLS} molecules) tasks shuffled (seed 42), WLAW placement, both "
            "functions loaded on every partition", "mpnn_flops_per_task": mfl,
            "peak_gbs": peak_gbs(), "peak_bf16_tflops": peak_bf16_tflops(), "layouts": rows}




def cmd_c5(a, mx):
    """D5 task farm (tools/farm.py). The correctness checks of the same farm run
    (trace vs the simulator, invariants I1-I5, 2 % sampled oracle parity) are
    tests/test_gpu_farm_d5.py: only tests/ may execute oracle/."""
    from tools.farm import Farm, FILL7, LAYOUT_B
    farm = Farm(mx, a.mol_variants)
    mfl = float(np.mean([mpnn_task_flops(m, MPNN.hidden, MPNN.steps) for m in farm.mol_cache]))
    out = {"suite": "D5 c5", "workload": f"configs[4]: task farm of {a.tasks} tasks, 50/50 "
           "GPT-2s decode / MPNN, shuffled (seed 42), WLAW over 7 fill partitions, layout "
           f"alternating fill-7 <-> {LAYOUT_B} via part_resize between waves of "
           f"{a.resize_every} submissions (wave w+2 is submitted after wave w completes)",
           "peak_gbs": peak_gbs()}
    for label, sizes, n_tasks, every in (("partitioned", FILL7, a.tasks, a.resize_every),
                                         ("1_partition", [148], a.base_tasks, 0)):
        r = farm.run(sizes, n_tasks, every)
        res = r["results"]
        assert all(x["status"] == 0 for x in res)
        st = class_stats(res, [k for k, _, _ in r["items"]], mfl, n_tasks // 2, n_tasks - n_tasks // 2)
        st["tasks"] = n_tasks
        st["e2e_tasks_per_s"] = round(n_tasks / r["wall_s"], 3)
        if r["resize_ms"]:
            rm = r["resize_ms"]
            st["part_resize_ms"] = {"n": len(rm), **{k: round(v, 3) for k, v in percentiles(rm).items()},
                                    "max": round(max(rm), 3)}
        out[label] = st
    out["ratio_vs_1_partition"] = round(out["partitioned"]["tasks_per_s"]
                                        / out["1_partition"]["tasks_per_s"], 3)
    return out


# ---------------------------------------------------------------------------
# N1: partitioned (green contexts) vs unpartitioned-concurrent vs time-shared
# ---------------------------------------------------------------------------

def cmd_modes(a, mx):
    """PAPER.md Table 1 and Figs. 4-5 compare time-
    sharing, MPS and MIG. Here, for N concurrent function instances:
      partitioned  : N green-context partitions (fill layout, SM-isolated)
      concurrent   : N shared streams, grid = 148/N CTAs each, hardware-placed
                     (default-MPS analog: concurrent, no isolation)
      timeshared   : N shared streams, grid = 148 CTAs each (every task wants
                     the whole GPU, so tasks take turns: time-slicing analog)
    Same closed batch of GPT-2s decode tasks, STATIC (k-1) mod N placement."""
    cfg = GPT2S
    fn = mx.fn_register(mx.decode_desc(cfg))
    tb = decode_task_bytes(cfg, 1, P_LEN, G_LEN)
    rows = []
    for n in [int(x) for x in a.ns.split(",")]:
        for mode in ("partitioned", "concurrent", "timeshared"):
            if mode == "partitioned":
                parts = [mx.part_create(0, s, 512 << 20) for s in LAYOUTS_FILL[n]]
            else:
                grid = 148 if mode == "timeshared" else max(1, 148 // n)
                parts = [mx.part_create_shared(0, grid, 512 << 20) for _ in range(n)]
            for p in parts:
                mx.fn_load(fn, p)
            closed_batch(mx, [(p, mx.decode_task(fn, prompt_tokens(1, 1, P_LEN, cfg.vocab), G_LEN))
                              for p in parts])
            items = [(parts[(k - 1) % n], mx.decode_task(fn, prompt_tokens(k, 1, P_LEN, cfg.vocab),
                                                         G_LEN)) for k in range(1, a.tasks + 1)]
            res, _ = closed_batch(mx, items)
            sp = span_s(res)
            rows.append({"n": n, "mode": mode, "grid": mx.part_query(parts[0])["n_ctas"],
                         "tasks_per_s": round(a.tasks / sp, 3),
                         "hbm_frac": round(a.tasks * tb / sp / 1e9 / peak_gbs(), 4), **lat(res)})
            for p in parts:
                mx.part_destroy(p)
    return {"suite": "N1 modes", "workload": f"configs[1] GPT-2s decode B1 P16 G32, {a.tasks} "
            "tasks per point, STATIC placement", "peak_gbs": peak_gbs(), "rows": rows}


# ---------------------------------------------------------------------------
# N3: shared read-only weights across partitions (§7, §6)
# ---------------------------------------------------------------------------

def cmd_n3(a, mx):
    """Same closed batches with one weight copy per partition (the paper's
    one-model-per-process setup) vs ONE copy per GPU referenced by all
    partitions. Reports tasks/s, algorithmic-bytes HBM fraction (may exceed 1
    when partitions hit each other's weights in L2), cold-start time of the
    layout and the HBM held by weights."""
    rows = []
    pool_fn = {}   # model -> bytes of its shared copy in the weight pool
    for cfg, B, layouts, ntask, q_priv, q_sh in (
            (GPT2S, 1, [int(x) for x in a.gpt2s_layouts.split(",")], a.gpt2s_tasks,
             512 << 20, 64 << 20),
            (LLAMA7B, 1, [int(x) for x in a.llama_layouts.split(",")], a.llama_tasks,
             14 << 30, 1 << 30)):
        tb = decode_task_bytes(cfg, B, P_LEN, G_LEN)
        fns = {"private": mx.fn_register(mx.decode_desc(cfg, max_batch=B)),
               "shared": mx.fn_register(mx.decode_desc(cfg, max_batch=B, shared_weights=True))}
        for n in layouts:
            sizes = LAYOUTS_FILL[n]
            for mode in ("private", "shared"):
                quota = q_priv if mode == "private" else q_sh
                if mode == "private" and n * quota > (170 << 30):
                    rows.append({"model": cfg.name, "partitions": n, "mode": mode,
                                 "skipped": f"{n} private copies exceed device memory"})
                    continue
                fn = fns[mode]
                pool0 = mx.weight_pool_query(0)["used_bytes"]
                parts = [mx.part_create(0, s, quota) for s in sizes]
                t0 = time.perf_counter()
                for p in parts:
                    mx.fn_load(fn, p)
                load_s = time.perf_counter() - t0
                grown = mx.weight_pool_query(0)["used_bytes"] - pool0
                if mode == "shared" and grown:
                    pool_fn[cfg.name] = grown
                held = sum(mx.part_query(p)["hbm_used"] for p in parts) + \
                    (pool_fn.get(cfg.name, 0) if mode == "shared" else 0)
                eq = len(set(sizes)) == 1
                closed_batch(mx, [(p, mx.decode_task(fn, prompt_tokens(9000 + i, B, P_LEN, cfg.vocab),
                                                     G_LEN)) for i, p in enumerate(parts)])
                items = [(parts[(k - 1) % n] if eq else mx.MX_PART_ANY,
                          mx.decode_task(fn, prompt_tokens(k, B, P_LEN, cfg.vocab), G_LEN))
                         for k in range(1, ntask + 1)]
                res, wall = closed_batch(mx, items)
                sp = span_s(res)
                rows.append({"model": cfg.name, "partitions": n, "sms": sizes, "mode": mode,
                             "tasks": ntask, "tasks_per_s": round(ntask / sp, 3),
                             "gen_tok_per_s": round(ntask * B * G_LEN / sp, 1),
                             "hbm_frac_algorithmic": round(ntask * tb / sp / 1e9 / peak_gbs(), 4),
                             "load_s": round(load_s, 3), "hbm_held_gib": round(held / 2**30, 2),
                             **lat(res)})
                for p in parts:
                    mx.part_destroy(p)
    return {"suite": "N3 shared weights", "workload": "configs[1] GPT-2s and configs[2] 7B "
            "decode, B=1 P=16 G=32, fill layouts; private = one weight copy per partition, "
            "shared = one copy per GPU (MX_FN_SHARED_WEIGHTS)", "peak_gbs": peak_gbs(),
            "rows": rows}


def main():
    ap = argparse.ArgumentParser()
    sub = ap.add_subparsers(dest="cmd", required=True)
    s = sub.add_parser("smsweep")
    s.add_argument("--sms", default="4,8,12,16,24,32,48,64,72,96,120,144,148")
    s.add_argument("--tasks", type=int, default=4)
    s = sub.add_parser("c3")
    s.add_argument("--layouts", default="1,2,4")
    s.add_argument("--batches", default="1,2,4,8")
    s.add_argument("--tasks", type=int, default=100)
    s = sub.add_parser("c4")
    s.add_argument("--layouts", default="1,7")
    s.add_argument("--decode", type=int, default=700)
    s.add_argument("--mpnn", type=int, default=700)
    s.add_argument("--mol-variants", type=int, default=16)
    s = sub.add_parser("c5")
    s.add_argument("--tasks", type=int, default=10000)
    s.add_argument("--base-tasks", type=int, default=1000)
    s.add_argument("--resize-every", type=int, default=1000)
    s.add_argument("--mol-variants", type=int, default=16)
    s = sub.add_parser("n3")
    s.add_argument("--gpt2s-layouts", default="14,18,37")
    s.add_argument("--gpt2s-tasks", type=int, default=296)
    s.add_argument("--llama-layouts", default="1,4,7,14")
    s.add_argument("--llama-tasks", type=int, default=28)
    s = sub.add_parser("modes")
    s.add_argument("--ns", default="1,2,4,7,14")
    s.add_argument("--tasks", type=int, default=140)
    a = ap.parse_args()
    from paper_conf_sc_dhakalrwercfm23_b200 import mx
    mx.mx_init([0])
    try:
        out = globals()[f"cmd_{a.cmd}"](a, mx)
    finally:
        mx.mx_shutdown()
    print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
