"""Reporting metrics (§5.2 Figs. 4-5).

Closed batch of N tasks submitted at t0 (A24). makespan = max t_end - t0;
tasks/s = N / makespan; completion = t_end - t_submit; service = t_end -
t_start (A7). The paper's two headline numbers are linked by
1/(1 - 0.60) = 2.5 (A1): `throughput_ratio` and `completion_reduction`
are written so that identity holds.
"""
from __future__ import annotations

import numpy as np


def throughput_ratio(t_base: float, t_new: float) -> float:
    """Throughput of the new layout over the baseline for the same work."""
    return t_base / t_new


def completion_reduction(t_base: float, t_new: float) -> float:
    """Fractional reduction of total completion time ('up to 60% lower')."""
    return 1.0 - t_new / t_base


def percentiles(values, qs=(50, 99)) -> dict:
    v = np.asarray(values, dtype=np.float64)
    if v.size == 0:
        return {f"p{q}": None for q in qs}
    return {f"p{q}": float(np.percentile(v, q)) for q in qs}


def summarize(results, n_generated_tokens: int, algo_bytes: int, peak_gbs: float) -> dict:
    """results: list of dicts with t_submit, t_start, t_end (ns, one clock)."""
    t0 = min(r["t_submit"] for r in results)
    t_first = min(r["t_start"] for r in results)
    t_last = max(r["t_end"] for r in results)
    makespan = (t_last - t0) * 1e-9
    dev_span = (t_last - t_first) * 1e-9
    comp = [(r["t_end"] - r["t_submit"]) * 1e-6 for r in results]
    serv = [(r["t_end"] - r["t_start"]) * 1e-6 for r in results]
    out = dict(n_tasks=len(results), makespan_s=makespan, device_span_s=dev_span,
               tasks_per_s=len(results) / makespan,
               gen_tok_per_s=n_generated_tokens / makespan,
               completion_ms=percentiles(comp), service_ms=percentiles(serv))
    if algo_bytes:
        out["hbm_gbs"] = algo_bytes / dev_span * 1e-9
        out["hbm_frac"] = out["hbm_gbs"] / peak_gbs
    return out
