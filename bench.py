#!/usr/bin/env python3
"""Headline benchmark: multiplexed small-function throughput on B200 partitions.

BASELINE.json metric: "tasks/sec and p50/p99 completion time vs #partitions;
decode tok/s; HBM % peak". Workload = configs[1]: GPT-2-
small-shaped Llama decode (random bf16 weights generated on device), batch 1,
P = 16 prompt + G = 32 greedy tokens per task, 700 tasks per closed batch
(§5.2: a fixed set of completions divided over the processes).

One bench step = one closed batch of N_TASKS tasks submitted through the C ABI
(fn_submit with host prompt buffers) and collected with fn_wait (host token
buffers) on the chosen partition layout of each GPU. Before the timed run a
short sweep measures the 1 / 2 / 4 / 7 / 14-partition layouts (D0 "fill") and
the finer 18 / 37-partition layouts (4-SM groups) — the paper's Fig. 4
comparison; the timed run's layout is chosen by N2 right-sizing (fn_rightsize:
the task measured alone on each candidate size).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--layout auto|sweep|1|2|4|7|14|18|37]
    python bench.py --impl reference      # the CPU oracle on a bounded sample

Multi-GPU (torchrun, one rank per GPU): tasks are independent, so every rank
runs the same per-GPU batch on its own GPU (weak scaling, no data-path
collective); rank 0 reports the total over ranks / the max span over ranks.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")   # before any CUDA init
ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

from workloads.configs import GPT2S, LAYOUTS_FILL, LAYOUTS_EQUAL  # noqa: E402
from workloads.inputs import prompt_tokens  # noqa: E402

P_LEN, G_LEN, N_TASKS = 16, 32, 700
QUOTA = 512 << 20
METRIC = "tasks/sec (p50/p99 completion, decode tok/s, HBM % peak) vs #partitions"
UNIT = "tasks/s"


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def task_bytes(cfg, B, P, G):
    """Algorithmic HBM bytes of one task (mirrors include/mx.h cost rule)."""
    d, q, kv, ff = cfg.d_model, cfg.q_dim, cfg.kv_dim, cfg.d_ff
    layer = 2 * (d * q + 2 * d * kv + q * d + 3 * d * ff) + 4 * d
    head = 2 * cfg.vocab * d + 2 * d
    S = P + G - 1
    kvpos = cfg.n_layers * 2 * kv * 2
    return (S * cfg.n_layers * layer + G * head + S * B * 2 * d + B * kvpos * (S * (S + 1) // 2)
            + S * B * kvpos)


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""

    def __init__(self, gpus):
        self.gpus = [gpus] if isinstance(gpus, int) else list(gpus)
        self.proc = None
        self.path = os.path.join(ROOT, "gpurun_out", f"clocks_gpu{self.gpus[0]}.csv")

    def __enter__(self):
        os.makedirs(os.path.dirname(self.path), exist_ok=True)
        q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
             "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap,"
             "utilization.memory")
        try:
            self.f = open(self.path, "w")
            self.proc = subprocess.Popen(["nvidia-smi", "-i", ",".join(map(str, self.gpus)),
                                          f"--query-gpu={q}",
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=self.f, stderr=subprocess.DEVNULL)
        except Exception:
            self.proc = None
        return self

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            self.proc.wait()
            self.f.close()

    def summary(self):
        if not self.proc:
            return None
        sm, mx_, reasons, mem = [], None, set(), []
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        try:
            for line in open(self.path):
                c = [x.strip() for x in line.split(",")]
                if len(c) < 9:
                    continue
                sm.append(float(c[1]))
                mx_ = float(c[2])
                for n, v in zip(names, c[5:9]):
                    if v.lower().startswith("active"):
                        reasons.add(n)
                if len(c) >= 10:
                    try:
                        mem.append(float(c[9]))
                    except ValueError:
                        pass
        except Exception:
            return None
        if not sm:
            return None
        out = {"sm_mhz": statistics.median(sm), "sm_max_mhz": mx_, "reasons": sorted(reasons),
               "samples": len(sm), "gpus": self.gpus}
        if mem:
            # nvidia-smi utilization.memory: % of time device memory was being read or
            # written (a coarse hardware-side check of the HBM-bound step; nsys is absent)
            out["mem_busy_pct_median"] = statistics.median(mem)
        return out


# ---------------------------------------------------------------------------
# GPU arm
# ---------------------------------------------------------------------------

def max_over_ranks(values, dist):
    """Element-wise max of per-rank timings (host-side gloo collective; the
    data path itself has no collective: tasks are independent replicas)."""
    if not dist:
        return [float(v) for v in values]
    import torch
    t = torch.tensor([float(v) for v in values], dtype=torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return [float(v) for v in t]


def sum_over_ranks(values, dist):
    """Element-wise sum of per-rank counts (tasks, GPUs) over ranks."""
    if not dist:
        return [float(v) for v in values]
    import torch
    t = torch.tensor([float(v) for v in values], dtype=torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.SUM)
    return [float(v) for v in t]


def local_devices(n_gpus: int, world: int, local_rank: int):
    """Device ordinals this process drives: one per rank under torchrun
    (world > 1), else all N requested GPUs in this process (one dispatcher
    thread per GPU, global placement over every partition of every GPU)."""
    if world > 1:
        return [local_rank]
    return list(range(max(1, n_gpus)))


def make_layout(mx, gpus, n, kind):
    """The same partition layout on every library GPU; partitions ordered by
    (gpu, part id) as the STATIC rule orders them."""
    sizes = (LAYOUTS_FILL if kind == "fill" else LAYOUTS_EQUAL)[n]
    return make_sized(mx, gpus, sizes)


def make_sized(mx, gpus, sizes):
    return [mx.part_create(g, s, QUOTA) for g in gpus for s in sizes]


# N2 right-sizing candidates (SM counts; 4-SM group multiples)
N2_CAND = [4, 8, 12, 16, 20, 24, 36, 40, 48, 72, 148]


def run_batch(mx, fn, parts, n_tasks, equal_sizes, prompts):
    """Submit a closed batch (all at t0) and wait for all. Returns per-task results."""
    tasks = []
    for k in range(1, n_tasks + 1):
        t = mx.decode_task(fn, prompts[(k - 1) % len(prompts)], G_LEN)
        part = parts[(k - 1) % len(parts)] if equal_sizes else mx.MX_PART_ANY
        mx.fn_submit(part, t)
        tasks.append(t)
    res = [mx.fn_wait(t) for t in tasks]
    for r in res:
        if r["status"] != 0:
            raise RuntimeError(f"task {r['task']} failed with status {r['status']}")
    return res, tasks


def summarize(res, n_steps):
    t_sub0 = min(r["t_submit_ns"] for r in res)
    t_start = min(r["t_start_ns"] for r in res)
    t_end = max(r["t_end_ns"] for r in res)
    comp = [(r["t_end_ns"] - r["t_submit_ns"]) / 1e6 for r in res]
    serv = [(r["t_end_ns"] - r["t_start_ns"]) / 1e6 for r in res]
    per_gpu = {}
    for r in res:
        g = per_gpu.setdefault(r["gpu"], [r["t_start_ns"], r["t_end_ns"], 0])
        g[0], g[1], g[2] = min(g[0], r["t_start_ns"]), max(g[1], r["t_end_ns"]), g[2] + 1
    return dict(span_s=(t_end - t_start) / 1e9, wall_s=(t_end - t_sub0) / 1e9,
                p50_ms=float(np.percentile(comp, 50)), p99_ms=float(np.percentile(comp, 99)),
                service_p50_ms=float(np.percentile(serv, 50)),
                service_p99_ms=float(np.percentile(serv, 99)),
                kernel_ms_mean=float(np.mean([r["kernel_ns"] for r in res]) / 1e6),
                per_gpu={g: dict(span_s=(v[1] - v[0]) / 1e9, tasks=v[2])
                         for g, v in sorted(per_gpu.items())})


def choose_layout(mx, fn, args, sweep, prompts):
    """Partition sizes of the timed run. 'auto' = N2 right-sizing (fn_rightsize:
    the task measured alone on each candidate size, throughput objective);
    'sweep' = the best fill layout of the D2 sweep; an integer = that fill layout."""
    if args.layout == "auto":
        sample = mx.decode_task(fn, prompts[0], G_LEN)
        r = mx.fn_rightsize(fn, 0, sample, N2_CAND, hbm_bytes=QUOTA, reps=2, objective=1)
        n2 = {"chosen_sms": r["sm"], "partitions": r["parts"],
              "predicted_tasks_per_s": round(r["rate_per_s"], 2),
              "curve_ms": [(sm, round(t / 1e6, 3)) for sm, t in r["curve"]],
              "rule": "mx_rightsize objective 1: argmax floor(148/s)/t(s) over the measured "
                      "single-instance service times t(s)"}
        return [r["sm"]] * r["parts"], n2
    if args.layout == "sweep":
        n = max(sweep, key=lambda d: d["tasks_per_s"])["partitions"] if sweep else 37
        return LAYOUTS_FILL[n], None
    return LAYOUTS_FILL[int(args.layout)], None


def gpu_arm(args, rank, world, local_rank, dist):
    from paper_conf_sc_dhakalrwercfm23_b200 import mx
    devices = local_devices(args.gpus, world, local_rank)
    if args.devices:
        # explicit device list for this process (e.g. "0,0": the in-process
        # multi-GPU path on one physical device — two dispatchers, one placement)
        devices = [int(x) for x in args.devices.split(",")]
    mx.mx_init(devices)
    gpus = list(range(len(devices)))          # library GPU indices
    ng = len(gpus)
    cfg = GPT2S
    fn = mx.fn_register(mx.decode_desc(cfg))
    prompts = [prompt_tokens(k, 1, P_LEN, cfg.vocab) for k in range(1, N_TASKS + 1)]
    bytes_task = task_bytes(cfg, 1, P_LEN, G_LEN)
    peak, peak_src = peaks()
    n_step = N_TASKS * ng                     # tasks per step in this process

    def load(parts):
        for p in parts:
            mx.fn_load(fn, p)

    def sweep_one(n, kind):
        parts = make_layout(mx, gpus, n, kind)
        load(parts)
        sizes = (LAYOUTS_FILL if kind == "fill" else LAYOUTS_EQUAL)[n]
        eq = len(set(sizes)) == 1
        tasks = sweep_tasks * ng
        run_batch(mx, fn, parts, min(tasks, 2 * len(parts)), eq, prompts)   # warm
        res, _ = run_batch(mx, fn, parts, tasks, eq, prompts)
        s = summarize(res, 1)
        for p in parts:
            mx.part_destroy(p)
        return dict(partitions=n, sms=sizes, tasks=tasks, tasks_per_s=tasks / s["span_s"],
                    p50_ms=s["p50_ms"], p99_ms=s["p99_ms"],
                    hbm_frac=tasks * bytes_task / s["span_s"] / (peak * 1e9 * ng))

    # --- partition sweep (Fig. 4 analog: 1 vs 2/4/7/14 partitions) ----------------
    sweep_tasks = 148
    sweep = [sweep_one(n, "fill") for n in args.sweep]
    # equal (MIG-like) layouts of the same N: STATIC (k-1) mod N placement
    sweep_equal = [sweep_one(n, "equal") for n in args.sweep if n in LAYOUTS_EQUAL and n != 1]
    sizes, n2 = choose_layout(mx, fn, args, sweep, prompts)
    n_main = len(sizes)

    # --- main timed run ------------------------------------------------------------
    parts = make_sized(mx, gpus, sizes)
    load(parts)
    eq = len(set(sizes)) == 1
    for _ in range(args.warmup):
        run_batch(mx, fn, parts, n_step, eq, prompts)
    if dist:
        dist.barrier()
    l0 = mx.launch_count()
    all_res = []
    with ClockSampler(devices) as clk:
        h0 = time.perf_counter()
        for _ in range(args.steps):
            res, _ = run_batch(mx, fn, parts, n_step, eq, prompts)
            all_res += res
        h1 = time.perf_counter()
    launches = mx.launch_count() - l0
    if dist:
        dist.barrier()
    s = summarize(all_res, args.steps)
    span, wall = max_over_ranks([s["span_s"], h1 - h0], dist)
    n_total, gpus_total, launches_total = sum_over_ranks([n_step * args.steps, ng, launches], dist)
    n_total, gpus_total = int(n_total), int(gpus_total)
    priv_held = sum(mx.part_query(p)["hbm_used"] for p in parts)
    for p in parts:
        mx.part_destroy(p)
    # --- N3: the same layout with ONE shared read-only weight copy per GPU ------
    n3 = None
    if args.n3:
        fs = mx.fn_register(mx.decode_desc(cfg, shared_weights=True))
        sparts = [mx.part_create(g, sz, 64 << 20) for g in gpus for sz in sizes]
        for p in sparts:
            mx.fn_load(fs, p)
        held = sum(mx.part_query(p)["hbm_used"] for p in sparts) + \
            sum(mx.weight_pool_query(g)["used_bytes"] for g in gpus)
        run_batch(mx, fs, sparts, n_step, eq, prompts)   # warm
        n3_steps = min(args.steps, 2)
        n3_res = []
        for _ in range(n3_steps):
            r, _ = run_batch(mx, fs, sparts, n_step, eq, prompts)
            n3_res += r
        s3 = summarize(n3_res, n3_steps)
        (span3,) = max_over_ranks([s3["span_s"]], dist)
        v3 = n_total / args.steps * n3_steps / span3
        n3 = {"tasks_per_s": round(v3, 3), "steps": n3_steps,
              "hbm_frac_algorithmic": round(bytes_task * v3 / gpus_total / 1e9 / peak, 4),
              "p50_ms": round(s3["p50_ms"], 3), "p99_ms": round(s3["p99_ms"], 3),
              "hbm_held_gib": round(held / 2**30, 3),
              "private_hbm_held_gib": round(priv_held / 2**30, 3),
              "note": "SURVEY.md §8(f) N3: one weight copy per GPU shared by all partitions "
                      "(MX_FN_SHARED_WEIGHTS); algorithmic bytes still count every "
                      "partition's weight stream, so L2 hits between partitions can lift "
                      "the fraction"}
        for p in sparts:
            mx.part_destroy(p)
    mx.mx_shutdown()
    if rank != 0:
        return None
    value = n_total / span
    achieved_gbs = bytes_task * n_total / span / 1e9 / gpus_total   # per GPU
    out = {
        "metric": METRIC, "value": round(value, 3), "unit": UNIT, "n_gpus": gpus_total,
        "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": round(span / args.steps * 1e3, 3), "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "bf16 weights/KV, fp32 math",
        "data": "synthetic (seeded bf16 weights generated on device, seeded prompts)",
        "config": {"workload": "configs[1]: GPT-2-small-shaped Llama decode, batch 1, P=16, G=32",
                   "model": "gpt2s-llama (L12 d768 H12 d_ff2048 V50257)",
                   "tasks_per_step_per_gpu": N_TASKS, "partitions_per_gpu": n_main,
                   "partition_sms": sizes,
                   "layout": ("N2 right-sizing (fn_rightsize)" if n2 else
                              f"fill layout {n_main}" if args.layout != "sweep" else "best of sweep"),
                   "placement": ("STATIC (k-1) mod P" if eq else "WLAW (C5)") +
                                (" over all partitions of all GPUs" if ng > 1 else ""),
                   "parallelism": (f"replicas x{gpus_total}: " +
                                   (f"{world} ranks (torchrun), one GPU each" if world > 1 else
                                    f"one process, {ng} GPU dispatcher threads") +
                                   " (independent tasks, no collective)"),
                   "l2": "inputs larger than L2: 324 MB of weights per partition copy"},
        "p50_ms": round(s["p50_ms"], 3), "p99_ms": round(s["p99_ms"], 3),
        "service_p50_ms": round(s["service_p50_ms"], 3),
        "service_p99_ms": round(s["service_p99_ms"], 3),
        "gen_tok_per_s": round(value * G_LEN, 1),
        "hbm_frac": round(achieved_gbs / peak, 4),
        "per_gpu": [{"gpu": devices[g], "tasks": v["tasks"], "span_s": round(v["span_s"], 4),
                     "hbm_frac": round(v["tasks"] * bytes_task / v["span_s"] / 1e9 / peak, 4)}
                    for g, v in s["per_gpu"].items()],
        "partitions_sweep": sweep,
        "partitions_sweep_equal": sweep_equal,
        "roofline": {"bound": "hbm", "achieved": round(achieved_gbs, 1), "peak": peak,
                     "unit": "GB/s", "frac": round(achieved_gbs / peak, 4),
                     "traffic": decode_traffic(),
                     "kernel": "decode_kernel (persistent megakernel, all partitions together)",
                     "algorithmic_bytes_per_launch": bytes_task,
                     "kernel_ms_mean_per_launch": round(s["kernel_ms_mean"], 3),
                     "peak_source": peak_src},
        "e2e": {"value": round(n_total / wall, 3), "unit": UNIT,
                "h2d_bytes_per_step": int(n_total / args.steps) * P_LEN * 4,
                "d2h_bytes_per_step": int(n_total / args.steps) * (G_LEN * 4 + 24)},
        "gpu_launches": int(launches_total),
        "timing": "value: device %globaltimer span (first kernel start -> last kernel end, "
                  "over all GPUs of the process) over the K steps, max over ranks; kernel_ms "
                  "from the kernels' own timestamps; e2e: host wall clock fn_submit -> last "
                  "fn_wait (prompts H2D, tokens D2H inside)",
    }
    if sweep:
        base = [d for d in sweep if d["partitions"] == 1]
        if base:
            out["ratio_vs_1_partition"] = round(max(d["tasks_per_s"] for d in sweep)
                                                / base[0]["tasks_per_s"], 3)
    if n3:
        out["n3_shared_weights"] = n3
    if n2:
        n2["measured_tasks_per_s_per_gpu"] = round(value / gpus_total, 2)
        out["n2_rightsize"] = n2
    out["clocks"] = clk.summary()
    if args.cpu_baseline and gpus_total == 1:
        out["cpu_baseline"] = cpu_baseline(args)
    return out


def decode_traffic():
    """dram bytes per decode launch from the committed ncu capture, only if it
    was taken on the current kernel source (stamp = hash of decode_impl.cuh)."""
    tp = os.path.join(ROOT, "profiles", "decode_traffic.json")
    try:
        d = json.load(open(tp))
    except Exception:
        return None
    if d.get("source_sha256") != kernel_source_hash():
        return None
    return d.get("dram_bytes_per_launch")


def kernel_source_hash():
    """sha256 of the decode kernel's code (decode_impl.cuh + common.cuh) with
    comments and blank lines removed, so documentation edits keep the stamp."""
    import hashlib
    import re
    h = hashlib.sha256()
    for f in ("decode_impl.cuh", "common.cuh"):
        with open(os.path.join(ROOT, "paper_conf_sc_dhakalrwercfm23_b200", "csrc", "kernels", f)) as fh:
            src = re.sub(r"/\*.*?\*/", "", fh.read(), flags=re.S)
        lines = (re.sub(r"//.*$", "", ln).rstrip() for ln in src.splitlines())
        h.update("\n".join(ln for ln in lines if ln).encode())
    return h.hexdigest()


# ---------------------------------------------------------------------------
# CPU oracle (cpu_baseline leg and --impl reference arm)
# ---------------------------------------------------------------------------

def _threads():
    try:
        from threadpoolctl import threadpool_info
        info = threadpool_info()
        return max([i.get("num_threads", 1) for i in info] or [1])
    except Exception:
        return os.cpu_count() or 1


def cpu_baseline(args, n_tasks: int = 1):
    from oracle import decode as od
    from workloads.weights import decode_weights
    w = decode_weights(GPT2S)
    t0 = time.perf_counter()
    for k in range(1, n_tasks + 1):
        od.greedy_task(GPT2S, w, prompt_tokens(k, 1, P_LEN, GPT2S.vocab), G_LEN)
    dt = time.perf_counter() - t0
    return {"value": round(n_tasks / dt, 5), "unit": UNIT, "cores": _threads(), "kind": "oracle",
            "sample": f"{n_tasks} full task(s) of the same workload (GPT-2s decode, P=16, G=32), "
                      f"fp64 NumPy oracle, weight generation excluded; {dt:.1f} s"}


# --- D6: the CPU oracle on the box's host cores, per workload ----
_CPU = {}


def _cpu_decode_task(k):
    from threadpoolctl import threadpool_limits
    from oracle import decode as od
    cfg, w, P, G = _CPU["decode"]
    with threadpool_limits(1):
        t0 = time.perf_counter()
        od.greedy_task(cfg, w, prompt_tokens(k, 1, P, cfg.vocab), G)
        return time.perf_counter() - t0


def _cpu_mpnn_task(k):
    from threadpoolctl import threadpool_limits
    from oracle import mpnn as om
    from workloads.configs import MPNN
    from workloads.inputs import molecules
    w, M = _CPU["mpnn"]
    mol = molecules(k, M)
    with threadpool_limits(1):
        t0 = time.perf_counter()
        om.mpnn_task(w, mol, MPNN.steps)
        return time.perf_counter() - t0


def cpu_suite():
    """D6: one task per process, one BLAS thread per process, a pool of all host
    cores; bounded samples of C1, C2, C4 (one wave each) and a 7B one-layer
    decode step with BLAS on all cores (reported per layer-step: the full 7B
    oracle would need ~27 GB of fp32 weights on the host; no extrapolation is
    folded into the reported numbers)."""
    import multiprocessing as mp
    import platform
    from oracle import decode as od
    from workloads.configs import TINY, LLAMA7B, MPNN
    from workloads.weights import decode_weights, mpnn_weights
    cores = os.cpu_count() or 1
    try:
        model = [l.split(":", 1)[1].strip() for l in open("/proc/cpuinfo") if l.startswith("model name")][0]
    except Exception:
        model = platform.processor()
    out = {"suite": "D6 cpu oracle", "host_cores": cores, "cpu_model": model, "rows": []}
    ctx = mp.get_context("fork")
    for name, cfg, P, G, n in (("C1 tiny decode", TINY, 8, 16, 4), ("C2 GPT-2s decode", GPT2S, P_LEN, G_LEN, cores)):
        _CPU["decode"] = (cfg, decode_weights(cfg), P, G)
        with ctx.Pool(min(n, cores)) as pool:
            t0 = time.perf_counter()
            per = pool.map(_cpu_decode_task, range(1, n + 1))
            wall = time.perf_counter() - t0
        out["rows"].append({"workload": name, "tasks": n, "procs": min(n, cores),
                            "tasks_per_s": round(n / wall, 4), "task_s_median": round(float(np.median(per)), 3),
                            "gen_tok_per_s": round(n * G / wall, 2)})
    _CPU["mpnn"] = (mpnn_weights(MPNN), 1024)
    n = cores
    with ctx.Pool(n) as pool:
        t0 = time.perf_counter()
        per = pool.map(_cpu_mpnn_task, range(1, n + 1))
        wall = time.perf_counter() - t0
    out["rows"].append({"workload": "C4 MPNN inference (1024 molecules per task)", "tasks": n,
                        "procs": n, "tasks_per_s": round(n / wall, 4),
                        "task_s_median": round(float(np.median(per)), 3)})
    from dataclasses import replace
    cfg1 = replace(LLAMA7B.with_layers(1), vocab=1024)   # the layer's cost does not depend on V
    w1 = decode_weights(cfg1)
    st = od.DecodeState(cfg1, 64)
    t0 = time.perf_counter()
    for s in range(4):
        od.decode_step(cfg1, w1, st, int(prompt_tokens(1, 1, 4, cfg1.vocab)[0, s]), s, want_logits=False)
    per_layer_step = (time.perf_counter() - t0) / 4
    out["rows"].append({"workload": "C3 7B decode, ONE layer (L=1 slice, vocab 1024), B=1, BLAS on all cores",
                        "layer_step_ms": round(per_layer_step * 1e3, 2),
                        "note": "a full 7B step is 32 such layers + the LM head; not measured"})
    return out


def reference_arm(args, rank, world):
    if rank != 0:
        return None
    from oracle import decode as od
    from workloads.weights import decode_weights
    w = decode_weights(GPT2S)
    for k in range(args.warmup):
        od.greedy_task(GPT2S, w, prompt_tokens(k + 1, 1, P_LEN, GPT2S.vocab), G_LEN)
    t0 = time.perf_counter()
    for k in range(args.steps):
        od.greedy_task(GPT2S, w, prompt_tokens(k + 1, 1, P_LEN, GPT2S.vocab), G_LEN)
    dt = time.perf_counter() - t0
    v = args.steps / dt
    cores = _threads()
    return {"impl": "reference", "metric": METRIC, "value": round(v, 5), "unit": UNIT,
            "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": round(dt / args.steps * 1e3, 1), "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": "configs[1]: GPT-2-small-shaped Llama decode, batch 1, P=16, G=32",
                       "sample": "1 task per step on the host CPU"},
            "cpu_baseline": {"value": round(v, 5), "unit": UNIT, "cores": cores, "kind": "oracle",
                             "sample": "1 full task per step (fp64 NumPy oracle)"},
            "e2e": {"value": round(v, 5), "unit": UNIT, "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="mx", choices=["mx", "reference"])
    ap.add_argument("--devices", default="",
                    help="explicit device ordinals for this process (default: --gpus / LOCAL_RANK)")
    ap.add_argument("--layout", default="auto")
    ap.add_argument("--sweep", default="1,2,4,7,14,18,37",
                    help="comma list of partition counts for the pre-run sweep ('' = none)")
    ap.add_argument("--no-cpu-baseline", dest="cpu_baseline", action="store_false")
    ap.add_argument("--cpu-suite", action="store_true",
                    help="D6: time the CPU oracle per workload on the host cores and exit")
    ap.add_argument("--no-n3", dest="n3", action="store_false",
                    help="skip the shared-weights (N3) measurement of the chosen layout")
    args = ap.parse_args()
    args.sweep = [int(x) for x in args.sweep.split(",") if x.strip()]
    if args.warmup < 3 and args.impl == "mx":
        print("warning: the timing rules want >= 3 warm-up steps", file=sys.stderr)
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    dist = None
    if world > 1:
        import torch.distributed as tdist
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        tdist.init_process_group("gloo", rank=rank, world_size=world)
        dist = tdist
    if args.cpu_suite:
        if rank == 0:
            print(json.dumps(cpu_suite()), flush=True)
        return
    if args.impl == "reference":
        out = reference_arm(args, rank, world)
    else:
        out = gpu_arm(args, rank, world, local_rank, dist)
    if out is not None:
        print(json.dumps(out), flush=True)
    if dist:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
