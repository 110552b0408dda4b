"""Oracle: one greedy LLM decode task (the paper's LLaMa-2 text completion).

PAPER.md §3.2: LLaMa2 "is mostly based on the predecessor LLaMa1
which is based on the transformer architecture"; §3.4 "text completion
tasks for 20-word sentences"; §5.2 "complete a paragraph of
text 100 times". The block is written out from SURVEY.md §8(c) C2 (Llama-2
conventions A8, A11, A15, A16; greedy A10):

    x = E[token]
    for l in 0..L-1:
        h = RMSNorm(x, g_attn[l]);  q = Wq h; k = Wk h; v = Wv h
        q, k = rope(q, t), rope(k, t)
        Kc[l][t] = bf16(k); Vc[l][t] = bf16(v)
        o_hh = sum_j softmax_j(q_hh . Kc[l][j] / sqrt(hd)) Vc[l][j]   (j = 0..t)
        x = x + Wo o
        h = RMSNorm(x, g_mlp[l]);  x = x + Wdown(silu(Wgate h) * (Wup h))
    logits = Wlm RMSNorm(x, g_final);   token = argmax (ties -> lowest index)

Arithmetic in float64. Two decisions follow the kernel's precision (fp32), as
the task rules require when floating point decides a discrete value: the KV
rounding (fp64 -> fp32 -> bf16 RNE) and the argmax (taken on fp32 logits).
"""
from __future__ import annotations

import numpy as np

from .numerics import bf16_rne


def rmsnorm(x: np.ndarray, g: np.ndarray, eps: float) -> np.ndarray:
    """RMSNorm: normalise, then scale; eps inside the sqrt (C2; hf_llama:53-66)."""
    x = np.asarray(x, dtype=np.float64)
    return x / np.sqrt(np.mean(x * x) + eps) * np.asarray(g, dtype=np.float64)


def rope_angles(t: int, head_dim: int, theta: float) -> np.ndarray:
    """a_i = fl32(t * inv_freq_i), inv_freq_i = fl32(1 / theta^(2i/hd)) (A11)."""
    expo = (np.arange(0, head_dim, 2, dtype=np.int64).astype(np.float32)
            / np.float32(head_dim))
    inv_freq = (np.float32(1.0) / (np.float32(theta) ** expo)).astype(np.float32)
    return (np.float32(t) * inv_freq).astype(np.float32).astype(np.float64)


def rope(x: np.ndarray, t: int, theta: float) -> np.ndarray:
    """Rotate-half RoPE on one head vector x[hd] at position t (A11).

    y_i = x_i cos a_i - x_{i+hd/2} sin a_i ;  y_{i+hd/2} = x_{i+hd/2} cos a_i + x_i sin a_i
    """
    hd = x.shape[-1]
    a = rope_angles(t, hd, theta)
    c, s = np.cos(a), np.sin(a)
    x1, x2 = x[..., : hd // 2], x[..., hd // 2:]
    return np.concatenate([x1 * c - x2 * s, x2 * c + x1 * s], axis=-1)


def softmax(s: np.ndarray) -> np.ndarray:
    e = np.exp(s - np.max(s))
    return e / np.sum(e)


def attention(q: np.ndarray, kc: np.ndarray, vc: np.ndarray) -> np.ndarray:
    """One head: o = sum_j softmax_j(q . K_j / sqrt(hd)) V_j over cached j = 0..t."""
    s = kc @ q / np.sqrt(q.shape[-1])
    return softmax(s) @ vc


def silu(z: np.ndarray) -> np.ndarray:
    return z / (1.0 + np.exp(-z))


class DecodeState:
    """Per-sequence KV cache: K[l][kvh][pos][hd], V likewise (float64 holding bf16 values)."""

    def __init__(self, cfg, max_pos: int):
        self.k = np.zeros((cfg.n_layers, cfg.n_kv_heads, max_pos, cfg.head_dim))
        self.v = np.zeros_like(self.k)


def decode_step(cfg, w: dict, st: DecodeState, token: int, t: int,
                want_logits: bool, kv_bf16: bool = True):
    """One decode step of one sequence at position t. Returns float64 logits or None."""
    hd, H, Hkv = cfg.head_dim, cfg.n_heads, cfg.n_kv_heads
    group = H // Hkv
    x = w["embed"][token].astype(np.float64)
    for l, lw in enumerate(w["layers"]):
        h = rmsnorm(x, lw["g_attn"], cfg.rms_eps)
        q = lw["wq"].astype(np.float64) @ h
        k = lw["wk"].astype(np.float64) @ h
        v = lw["wv"].astype(np.float64) @ h
        q = rope(q.reshape(H, hd), t, cfg.rope_theta)
        k = rope(k.reshape(Hkv, hd), t, cfg.rope_theta)
        v = v.reshape(Hkv, hd)
        if kv_bf16:
            k = bf16_rne(k).astype(np.float64)
            v = bf16_rne(v).astype(np.float64)
        st.k[l, :, t] = k
        st.v[l, :, t] = v
        o = np.empty((H, hd))
        for hh in range(H):
            kvh = hh // group
            o[hh] = attention(q[hh], st.k[l, kvh, : t + 1], st.v[l, kvh, : t + 1])
        x = x + lw["wo"].astype(np.float64) @ o.reshape(-1)
        h = rmsnorm(x, lw["g_mlp"], cfg.rms_eps)
        a = silu(lw["w_gate"].astype(np.float64) @ h) * (lw["w_up"].astype(np.float64) @ h)
        x = x + lw["w_down"].astype(np.float64) @ a
    if not want_logits:
        return None
    return w["lm_head"].astype(np.float64) @ rmsnorm(x, w["g_final"], cfg.rms_eps)


def argmax_fp32(logits64: np.ndarray) -> tuple[int, float]:
    """Greedy choice on fp32 logits, ties -> lowest index (A10). Returns (token, margin)."""
    l32 = np.asarray(logits64, dtype=np.float32)
    tok = int(np.argmax(l32))
    top2 = np.partition(logits64, -2)[-2:]
    margin = float((top2[1] - top2[0]) / max(np.max(np.abs(logits64)), 1e-30))
    return tok, margin


def greedy_task(cfg, w: dict, prompt: np.ndarray, gen_len: int, kv_bf16: bool = True,
                forced: np.ndarray | None = None):
    """Greedy task for prompt[B][P].

    Steps s = 0..P+G-2 at positions t = s; input token = prompt[s] for s < P,
    else the token generated at step s-1; generated token j (1-based) is the
    argmax at step P-2+j. Logits are only needed at steps s >= P-1.

    Returns tokens[B][G] int32, logits[G][B][V] float32, margins[G][B].
    `forced` (teacher forcing with given tokens[B][G]) is a debugging aid only.
    """
    prompt = np.asarray(prompt)
    B, P = prompt.shape
    G = gen_len
    V = cfg.vocab
    tokens = np.zeros((B, G), dtype=np.int32)
    logits = np.zeros((G, B, V), dtype=np.float32)
    margins = np.zeros((G, B))
    for b in range(B):
        st = DecodeState(cfg, P + G)
        prev = None
        for s in range(P + G - 1):
            tok_in = int(prompt[b, s]) if s < P else prev
            want = s >= P - 1
            lg = decode_step(cfg, w, st, tok_in, s, want, kv_bf16)
            if want:
                j = s - (P - 1)
                tok, m = argmax_fp32(lg)
                tokens[b, j] = tok
                logits[j, b] = lg.astype(np.float32)
                margins[j, b] = m
                prev = tok if forced is None else int(forced[b, j])
    return tokens, logits, margins
