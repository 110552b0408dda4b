"""Pins for the decode oracle (SURVEY.md §8(c) pin table), all CPU.

Each pin checks the oracle against something other than itself: a library
routine (torch / HF transformers), a closed form, an invariant, exact integer
arithmetic, or a worked example with hand-derived values.
"""
import math

import numpy as np
import pytest
import torch

from oracle import decode as od
from oracle.numerics import bf16_rne
from workloads.configs import TINY, DecodeCfg
from workloads.weights import decode_weights


# ---- bf16 RNE vs torch ------------------------------------------------------
def test_bf16_rne_matches_torch_including_ties():
    rng = np.random.default_rng(0)
    x = rng.standard_normal(1_000_000).astype(np.float32) * np.float32(3.0)
    bits = np.array([0x3F808000, 0x3F818000, 0x3F80FFFF, 0xBF808000, 0x7F7FFFFF, 0x00008000,
                     0x00018000, 0x7F800000, 0xFF800000], dtype=np.uint32)
    x = np.concatenate([x, bits.view(np.float32)])
    want = torch.from_numpy(x).to(torch.bfloat16).to(torch.float32).numpy()
    got = bf16_rne(x)
    assert np.array_equal(got.view(np.uint32), want.view(np.uint32))
    # the two ties named in the survey
    assert bf16_rne(np.uint32(0x3F808000).view(np.float32)).view(np.uint32) == 0x3F800000
    assert bf16_rne(np.uint32(0x3F818000).view(np.float32)).view(np.uint32) == 0x3F820000


# ---- RMSNorm ------------------------------------------------------------------
def test_rmsnorm_closed_form_constant_vector():
    c, eps = 0.37, 1e-5
    g = np.linspace(0.5, 1.5, 16)
    y = od.rmsnorm(np.full(16, c), g, eps)
    assert np.allclose(y, g * c / math.sqrt(c * c + eps), rtol=1e-15)


def test_rmsnorm_vs_hf_llama():
    from transformers.models.llama.modeling_llama import LlamaRMSNorm
    rng = np.random.default_rng(1)
    x = rng.standard_normal(256)
    g = rng.uniform(0.8, 1.2, 256)
    m = LlamaRMSNorm(256, eps=1e-5)
    m.weight.data = torch.tensor(g, dtype=torch.float32)
    want = m(torch.tensor(x, dtype=torch.float32)).detach().double().numpy()
    assert np.allclose(od.rmsnorm(x, g, 1e-5), want, rtol=1e-6, atol=1e-6)


# ---- RoPE -------------------------------------------------------------------
def test_rope_identity_at_t0_and_norm_preserving():
    rng = np.random.default_rng(2)
    x = rng.standard_normal(64)
    assert np.array_equal(od.rope(x, 0, 1e4), x)
    for t in (1, 7, 47):
        y = od.rope(x, t, 1e4)
        pn = lambda v: v[:32] ** 2 + v[32:] ** 2
        assert np.allclose(pn(y), pn(x), rtol=1e-12)


def test_rope_relative_position_property():
    rng = np.random.default_rng(3)
    q, k = rng.standard_normal(64), rng.standard_normal(64)
    # <rope(q,m), rope(k,n)> depends only on m-n (angles are fl32(t*inv_freq): allow fp32 slack)
    a = od.rope(q, 10, 1e4) @ od.rope(k, 7, 1e4)
    b = od.rope(q, 5, 1e4) @ od.rope(k, 2, 1e4)
    assert abs(a - b) < 1e-5 * (np.linalg.norm(q) * np.linalg.norm(k))


def test_rope_vs_hf_apply_rotary():
    from transformers.models.llama.modeling_llama import apply_rotary_pos_emb
    rng = np.random.default_rng(4)
    hd, t = 64, 13
    q = rng.standard_normal((1, 2, 1, hd))
    k = rng.standard_normal((1, 2, 1, hd))
    inv = 1.0 / (1e4 ** (torch.arange(0, hd, 2, dtype=torch.int64).float() / hd))
    fr = (inv[None, :] * torch.tensor([[float(t)]])).float()
    emb = torch.cat([fr, fr], -1)
    cos, sin = emb.cos().double()[None], emb.sin().double()[None]
    qe, ke = apply_rotary_pos_emb(torch.tensor(q), torch.tensor(k), cos, sin)
    assert np.allclose(od.rope(q[0, 0, 0], t, 1e4), qe[0, 0, 0].numpy(), atol=1e-6)
    assert np.allclose(od.rope(k[0, 1, 0], t, 1e4), ke[0, 1, 0].numpy(), atol=1e-6)


# ---- attention --------------------------------------------------------------
def test_attention_special_cases():
    rng = np.random.default_rng(5)
    q = rng.standard_normal(64)
    k0, v0 = rng.standard_normal((1, 64)), rng.standard_normal((1, 64))
    assert np.array_equal(od.attention(q, k0, v0), v0[0])          # t = 0: o = v0 exactly
    K = np.repeat(rng.standard_normal((1, 64)), 9, axis=0)
    V = rng.standard_normal((9, 64))
    assert np.allclose(od.attention(q, K, V), V.mean(0), rtol=1e-13)  # equal keys -> mean(v)


def test_attention_vs_torch_sdpa_fp64():
    rng = np.random.default_rng(6)
    q, K, V = rng.standard_normal(64), rng.standard_normal((30, 64)), rng.standard_normal((30, 64))
    want = torch.nn.functional.scaled_dot_product_attention(
        torch.tensor(q)[None, None, None], torch.tensor(K)[None, None], torch.tensor(V)[None, None])
    assert np.allclose(od.attention(q, K, V), want[0, 0, 0].numpy(), rtol=1e-12, atol=1e-14)


# ---- SwiGLU / GEMV / argmax ------------------------------------------------------
def test_silu_zero_and_vs_torch():
    z = np.linspace(-20, 20, 1001)
    assert od.silu(np.array([0.0]))[0] == 0.0
    assert np.allclose(od.silu(z), torch.nn.functional.silu(torch.tensor(z)).numpy(), rtol=1e-14)


def test_gemv_is_exact_on_dyadic_inputs():
    # weights are k*2^-12 (C1); with h = integer*2^-10 every product and sum is exact in fp64,
    # so the matmul step equals exact integer arithmetic.
    from workloads.weights import matrix
    W = matrix(0x7111, 17, 40, 256)
    rng = np.random.default_rng(7)
    hi = rng.integers(-1000, 1000, 256)
    h = hi * 2.0 ** -10
    got = W.astype(np.float64) @ h
    Wi = np.round(W * 4096).astype(np.int64)
    exact = [sum(int(a) * int(b) for a, b in zip(Wi[r], hi)) for r in range(40)]
    assert [int(round(g * 2 ** 22)) for g in got] == exact


def test_argmax_ties_lowest_index():
    lg = np.array([0.1, 3.0, -1.0, 3.0, 2.9])
    tok, margin = od.argmax_fp32(lg)
    assert tok == 1 and margin == 0.0
    assert od.argmax_fp32(np.array([1.0, 2.0, 0.0]))[0] == int(torch.argmax(torch.tensor([1.0, 2.0, 0.0])))


# ---- worked micro model (hand-derived closed form) ------------------------------
def test_micro_model_closed_form():
    """L1, d2, H1, hd2, d_ff1, V3, eps=0, t=0 (SURVEY.md pin 'micro model by hand').

    token 0 -> x = [1, 1]; rms = 1 -> h = g_attn = [1, 1]; at t = 0 attention
    returns v0 = Wv h = [1, 1] (bf16-exact) and RoPE is the identity;
    x1 = x + Wo o = [1,1] + [[1,0],[0,0]][1,1] = [2, 1].  Wgate = 0 -> silu(0) = 0
    -> MLP adds 0.  logits = Wlm (x1/rms(x1)) with rms(x1) = sqrt(5/2):
    x1/rms = [4/sqrt(10), 2/sqrt(10)] and Wlm = [[1,0],[0,1],[1,-1]]
    -> logits = [4/sqrt(10), 2/sqrt(10), 2/sqrt(10)] -> token 0.
    """
    cfg = DecodeCfg("micro", 1, 2, 1, 1, 2, 1, 3, max_seq=4, rms_eps=0.0, rope_theta=1e4)
    one = np.ones(2)
    w = dict(embed=np.array([[1.0, 1.0], [0.0, 1.0], [1.0, 0.0]]),
             layers=[dict(wq=np.eye(2), wk=np.eye(2), wv=np.eye(2),
                          wo=np.array([[1.0, 0.0], [0.0, 0.0]]),
                          w_gate=np.zeros((1, 2)), w_up=np.ones((1, 2)), w_down=np.ones((2, 1)),
                          g_attn=one, g_mlp=one)],
             g_final=one, lm_head=np.array([[1.0, 0.0], [0.0, 1.0], [1.0, -1.0]]))
    st = od.DecodeState(cfg, 4)
    lg = od.decode_step(cfg, w, st, 0, 0, True)
    s10 = math.sqrt(10.0)
    assert np.allclose(lg, [4 / s10, 2 / s10, 2 / s10], rtol=1e-15)
    assert od.argmax_fp32(lg)[0] == 0
    assert np.array_equal(st.k[0, 0, 0], [1.0, 1.0]) and np.array_equal(st.v[0, 0, 0], [1.0, 1.0])


# ---- whole decode vs HF LlamaForCausalLM ------------------------------------------
def _hf_model(cfg, w):
    from transformers import LlamaConfig, LlamaForCausalLM
    hc = LlamaConfig(hidden_size=cfg.d_model, intermediate_size=cfg.d_ff,
                     num_hidden_layers=cfg.n_layers, num_attention_heads=cfg.n_heads,
                     num_key_value_heads=cfg.n_kv_heads, head_dim=cfg.head_dim,
                     vocab_size=cfg.vocab, rms_norm_eps=cfg.rms_eps, rope_theta=cfg.rope_theta,
                     tie_word_embeddings=False, attention_bias=False, mlp_bias=False,
                     max_position_embeddings=256)
    m = LlamaForCausalLM(hc).double().eval()
    sd = {"model.embed_tokens.weight": w["embed"], "model.norm.weight": w["g_final"],
          "lm_head.weight": w["lm_head"]}
    for l, lw in enumerate(w["layers"]):
        p = f"model.layers.{l}."
        sd.update({p + "self_attn.q_proj.weight": lw["wq"], p + "self_attn.k_proj.weight": lw["wk"],
                   p + "self_attn.v_proj.weight": lw["wv"], p + "self_attn.o_proj.weight": lw["wo"],
                   p + "mlp.gate_proj.weight": lw["w_gate"], p + "mlp.up_proj.weight": lw["w_up"],
                   p + "mlp.down_proj.weight": lw["w_down"],
                   p + "input_layernorm.weight": lw["g_attn"],
                   p + "post_attention_layernorm.weight": lw["g_mlp"]})
    m.load_state_dict({k: torch.tensor(np.asarray(v), dtype=torch.float64) for k, v in sd.items()},
                      strict=False)
    return m


@pytest.mark.slow
def test_tiny_decode_vs_hf_llama():
    """Whole tiny decode (C1 shape) vs HF LlamaForCausalLM with the same weights,
    KV rounding OFF (HF keeps full-precision KV): logits <= 1e-5 rel, tokens identical."""
    from workloads.inputs import prompt_tokens
    cfg = TINY
    w = decode_weights(cfg)
    prompt = prompt_tokens(1, 1, 8, cfg.vocab)
    P, G = 8, 16
    tok, lg, _ = od.greedy_task(cfg, w, prompt, G, kv_bf16=False)
    m = _hf_model(cfg, w)
    seq = list(prompt[0])
    with torch.no_grad():
        out = m(torch.tensor([seq]), use_cache=True)
        past = out.past_key_values
        hf_logits = [out.logits[0, -1].numpy()]
        nxt = int(np.argmax(hf_logits[-1].astype(np.float32)))
        hf_tok = [nxt]
        for j in range(1, G):
            out = m(torch.tensor([[nxt]]), past_key_values=past, use_cache=True)
            past = out.past_key_values
            hf_logits.append(out.logits[0, -1].numpy())
            nxt = int(np.argmax(hf_logits[-1].astype(np.float32)))
            hf_tok.append(nxt)
    assert list(tok[0]) == hf_tok
    for j in range(G):
        ref = hf_logits[j]
        rel = np.max(np.abs(lg[j, 0] - ref)) / np.max(np.abs(ref))
        assert rel <= 1e-5, (j, rel)


def test_kv_rounding_flag_changes_only_by_bf16_scale():
    from workloads.inputs import prompt_tokens
    cfg = TINY
    w = decode_weights(cfg)
    prompt = prompt_tokens(2, 1, 8, cfg.vocab)
    t1, l1, _ = od.greedy_task(cfg, w, prompt, 4, kv_bf16=True)
    t0, l0, _ = od.greedy_task(cfg, w, prompt, 4, kv_bf16=False, forced=t1)
    rel = np.max(np.abs(l1 - l0)) / np.max(np.abs(l0))
    assert 0 < rel < 2e-2
