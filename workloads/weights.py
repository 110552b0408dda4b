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
from .prng import weight_values, weight_levels, gain_values


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


class LazyDecodeLayers:
    """The per-layer dicts of `decode_layer`, generated on first access and held
    as int8 levels (1 byte per weight; values = level * 2^-12, exact), so a
    32-layer 7B-shaped model (6.5 G weights) fits a test host. Indexing and
    iteration return the same float32 arrays `decode_layer` would."""

    _MATS = (("wq", T_WQ, "q", "d"), ("wk", T_WK, "kv", "d"), ("wv", T_WV, "kv", "d"),
             ("wo", T_WO, "d", "q"), ("w_gate", T_WGATE, "ff", "d"), ("w_up", T_WUP, "ff", "d"),
             ("w_down", T_WDOWN, "d", "ff"))

    def __init__(self, cfg: DecodeCfg):
        self.cfg = cfg
        self._lv = {}

    def __len__(self):
        return self.cfg.n_layers

    def _dims(self):
        c = self.cfg
        return {"q": c.q_dim, "kv": c.kv_dim, "d": c.d_model, "ff": c.d_ff}

    def __getitem__(self, l: int) -> dict:
        if not 0 <= l < self.cfg.n_layers:
            raise IndexError(l)
        c, dims = self.cfg, self._dims()
        if l not in self._lv:
            self._lv[l] = {name: weight_levels(c.seed, layer_tid(l, t), dims[r] * dims[k])
                           for name, t, r, k in self._MATS}
        out = {name: (self._lv[l][name].astype(np.float32) * np.float32(2.0 ** -12)).reshape(
            dims[r], dims[k]) for name, t, r, k in self._MATS}
        out["g_attn"] = gain_values(c.seed, layer_tid(l, T_GATTN), c.d_model)
        out["g_mlp"] = gain_values(c.seed, layer_tid(l, T_GMLP), c.d_model)
        return out

    def __iter__(self):
        for l in range(len(self)):
            yield self[l]


def decode_weights_lazy(cfg: DecodeCfg) -> dict:
    """`decode_weights` with the layers generated on demand (LazyDecodeLayers)."""
    return dict(
        embed=matrix(cfg.seed, T_EMBED, cfg.vocab, cfg.d_model),
        layers=LazyDecodeLayers(cfg),
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
