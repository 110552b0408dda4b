"""Algorithmic work per task and the default placement cost (integers).

SURVEY.md §8(d) D0 defines the algorithmic work; §8(c) C5 the default cost
"as an integer in ns at nominal roofline on a whole GPU". Readings (DESIGN.md
§3, R5): a generated token needs the LM head only at steps s >= P-1 (the
prompt steps' logits are never read), so the LM-head bytes are counted G
times, not P+G-1 times.
"""
from __future__ import annotations


def decode_layer_weight_bytes(cfg) -> int:
    d, q, kv, ff = cfg.d_model, cfg.q_dim, cfg.kv_dim, cfg.d_ff
    return 2 * (d * q + 2 * d * kv + q * d + 3 * d * ff) + 2 * (2 * d)


def decode_head_bytes(cfg) -> int:
    return 2 * cfg.vocab * cfg.d_model + 2 * cfg.d_model


def decode_task_bytes(cfg, batch: int, prompt_len: int, gen_len: int) -> int:
    """HBM bytes one greedy task must move: weights streamed once per step, the
    embedding row, the KV cache read (positions 0..t) and written (position t)."""
    S = prompt_len + gen_len - 1
    L, B = cfg.n_layers, batch
    kv_pos = L * 2 * cfg.kv_dim * 2          # K and V, bf16, all layers, one position
    return (S * L * decode_layer_weight_bytes(cfg) + gen_len * decode_head_bytes(cfg)
            + S * B * 2 * cfg.d_model
            + B * kv_pos * (S * (S + 1) // 2)
            + S * B * kv_pos)


def decode_task_flops(cfg, batch: int, prompt_len: int, gen_len: int) -> int:
    """2 flops per weight per sequence (GEMV), attention 4*hd per (head, position)."""
    S = prompt_len + gen_len - 1
    wl = decode_layer_weight_bytes(cfg) // 2 - 2 * cfg.d_model
    head = cfg.vocab * cfg.d_model
    attn = batch * cfg.n_layers * cfg.n_heads * 4 * cfg.head_dim * (S * (S + 1) // 2)
    return 2 * batch * (S * cfg.n_layers * wl + gen_len * head) + attn


def mpnn_molecule_flops(types, edges, F: int, T: int) -> int:
    """T*(2F^2*(n + D_ub) + E_dir*F + 2n*F) + n*F + 2F^2 + 4F  (D0)."""
    n = len(types)
    pairs = set()
    for (u, v, b) in edges:
        pairs.add((u, b))
        pairs.add((v, b))
    D = len(pairs)
    e_dir = 2 * len(edges)
    return T * (2 * F * F * (n + D) + e_dir * F + 2 * n * F) + n * F + 2 * F * F + 4 * F


def mpnn_task_flops(task: dict, F: int, T: int) -> int:
    from workloads.inputs import molecule_of
    M = len(task["atom_off"]) - 1
    return sum(mpnn_molecule_flops(*molecule_of(task, m), F, T) for m in range(M))


def ceil_div(a: int, b: int) -> int:
    return -(-a // b)


def decode_default_cost(cfg, batch, prompt_len, gen_len) -> int:
    return ceil_div(decode_task_bytes(cfg, batch, prompt_len, gen_len), 8000)


def mpnn_default_cost(task: dict, F: int, T: int) -> int:
    return ceil_div(mpnn_task_flops(task, F, T), 75000)


def mpnn_train_default_cost(task: dict, F: int, T: int) -> int:
    """Placement cost of one emulator training step (N4, reading R10): forward
    plus backward ~ 3x the forward contractions, same 75 TFLOP/s unit as C5."""
    return ceil_div(3 * mpnn_task_flops(task, F, T), 75000)
