"""Seeded model weights as numpy arrays in canonical (logical) layout.

W[out][in] element i = row*in + col, E[tok][col] i = tok*d + col, gains i = col
(SURVEY.md §8(c) C1). Values are exactly representable in bf16. The CUDA
library generates the same values on device into its own physical layout with
its own implementation of the generator.
"""
from __future__ import annotations

import numpy as np

from .configs import (DecodeCfg, MpnnCfg, T_EMBED, T_WQ, T_WK, T_WV, T_WO, T_WGATE, T_WUP,
                      T_WDOWN, T_GATTN, T_GMLP, layer_tid, gfinal_tid, lmhead_tid,
                      M_EATOM, M_WB0, M_U, M_C, M_W1, M_C1, M_W2, M_C2)
from .prng import weight_values, gain_values


def matrix(seed: int, tid: int, rows: int, cols: int) -> np.ndarray:
    return weight_values(seed, tid, rows * cols).reshape(rows, cols)


def decode_layer(cfg: DecodeCfg, layer: int) -> dict:
    s, d = cfg.seed, cfg.d_model
    t = lambda w: layer_tid(layer, w)
    return dict(
        wq=matrix(s, t(T_WQ), cfg.q_dim, d),
        wk=matrix(s, t(T_WK), cfg.kv_dim, d),
        wv=matrix(s, t(T_WV), cfg.kv_dim, d),
        wo=matrix(s, t(T_WO), d, cfg.q_dim),
        w_gate=matrix(s, t(T_WGATE), cfg.d_ff, d),
        w_up=matrix(s, t(T_WUP), cfg.d_ff, d),
        w_down=matrix(s, t(T_WDOWN), d, cfg.d_ff),
        g_attn=gain_values(s, t(T_GATTN), d),
        g_mlp=gain_values(s, t(T_GMLP), d),
    )


def decode_weights(cfg: DecodeCfg) -> dict:
    """All decoder tensors: {'embed', 'layers': [...], 'g_final', 'lm_head'}."""
    return dict(
        embed=matrix(cfg.seed, T_EMBED, cfg.vocab, cfg.d_model),
        layers=[decode_layer(cfg, l) for l in range(cfg.n_layers)],
        g_final=gain_values(cfg.seed, gfinal_tid(cfg), cfg.d_model),
        lm_head=matrix(cfg.seed, lmhead_tid(cfg), cfg.vocab, cfg.d_model),
    )


def mpnn_weights(cfg: MpnnCfg) -> dict:
    s, F = cfg.seed, cfg.hidden
    return dict(
        e_atom=matrix(s, M_EATOM, cfg.n_atom_types, F),
        w_b=np.stack([matrix(s, M_WB0 + b, F, F) for b in range(cfg.n_bond_types)]),
        u=matrix(s, M_U, F, F),
        c=weight_values(s, M_C, F),
        w1=matrix(s, M_W1, F, F),
        c1=weight_values(s, M_C1, F),
        w2=weight_values(s, M_W2, F),
        c2=weight_values(s, M_C2, 1)[0],
    )
