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


def decode_task_bytes(cfg, B: int, P: int, G: int) -> int:
    """Algorithmic HBM bytes of one greedy decode task (SURVEY.md §8(d) D0,
    DESIGN.md §6): every weight once per step (LM head only at the G steps that
    produce a token), the embedding row, and the KV cache read/written."""
    d, q, kv, ff = cfg.d_model, cfg.q_dim, cfg.kv_dim, cfg.d_ff
    layer = 2 * (d * q + 2 * d * kv + q * d + 3 * d * ff) + 4 * d
    head = 2 * cfg.vocab * d + 2 * d
    S = P + G - 1
    kvpos = cfg.n_layers * 2 * kv * 2
    return (S * cfg.n_layers * layer + G * head + S * B * 2 * d + B * kvpos * (S * (S + 1) // 2)
            + S * B * kvpos)


def mpnn_task_flops(task: dict, F: int, T: int) -> int:
    """Algorithmic flops of one MPNN task, summed over its
    molecules: T*(2F^2*(n + D_ub) + E_dir*F + 2n*F) + n*F + 2F^2 + 4F, with
    D_ub the number of distinct (atom, incident bond type) pairs."""
    ao = np.asarray(task["atom_off"], dtype=np.int64)
    eo = np.asarray(task["edge_off"], dtype=np.int64)
    e = task["edges"]
    M = len(ao) - 1
    n = np.diff(ao)
    E = np.diff(eo)
    mol_of_edge = np.repeat(np.arange(M), E)
    base = ao[:-1][mol_of_edge]
    b = e["bond"].astype(np.int64)
    gu = (base + e["u"].astype(np.int64)) * 4 + b
    gv = (base + e["v"].astype(np.int64)) * 4 + b
    D = len(np.unique(np.concatenate([gu, gv])))
    tot_n, tot_E = int(n.sum()), int(E.sum())
    return int(T * (2 * F * F * (tot_n + D) + 2 * tot_E * F + 2 * tot_n * F) + tot_n * F
               + M * (2 * F * F + 4 * F))
