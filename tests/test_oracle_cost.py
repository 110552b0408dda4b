"""Pins for oracle/cost.py (VERDICT r1 Weak 1: mpnn_molecule_flops and the
task-level terms of decode_task_bytes were only compared with their own C++
mirror). Each value below is derived independently of the formula in
cost.py: hand-counted for a worked example, or counted from the tensors the
seeded generator actually produces, or by brute-force enumeration.

SURVEY.md §8(d) D0 defines the algorithmic work; reading R5 departs
from SURVEY's per-task byte figures by counting the LM head only at the G
steps whose logits are read (steps s >= P-1), not at all P+G-1 steps."""
import itertools

from oracle.cost import (decode_task_bytes, decode_head_bytes, decode_layer_weight_bytes,
                         mpnn_molecule_flops, mpnn_task_flops)
from workloads.configs import TINY, GPT2S, LLAMA7B
from workloads.inputs import molecules, molecule_of
from workloads.weights import decode_weights


def test_mpnn_flops_worked_example():
    """3 atoms, bonds (0-1 type 0), (1-2 type 1); F = 128, T = 3. Counted by hand
    from the D0 description of the work:
      per step: U h_v for 3 atoms              3 x 2F^2 = 98,304
                W_b h_u for distinct (atom, type) incident pairs
                {(0,0), (1,0), (1,1), (2,1)}     4 x 2F^2 = 131,072
                one F-vector add per directed message (4)   512
                + m and + c for 3 atoms          2 x 3F  =   768
                                                 ------- 230,656 x 3 steps = 691,968
      readout sum over 3 atoms                  3F      =    384
      head: W1 r (2F^2), + c1, ReLU, w2 . (2F), + c2     = 32,768 + 512 (4F)
    total 691,968 + 384 + 33,280 = 725,632."""
    assert mpnn_molecule_flops([1, 2, 3], [(0, 1, 0), (1, 2, 1)], 128, 3) == 725_632


def test_mpnn_flops_structure():
    """D_ub counts DISTINCT (atom, bond type) pairs; a duplicate listing adds
    only its two directed messages; relabelling atoms changes nothing; a lone
    atom costs T (U h + 2 adds) plus the readout and head (brute-force check of
    the pair count on a generated task)."""
    F, T = 128, 3
    base = mpnn_molecule_flops([0, 1, 2], [(0, 1, 0), (1, 2, 1)], F, T)
    dup = mpnn_molecule_flops([0, 1, 2], [(0, 1, 0), (1, 2, 1), (1, 0, 0)], F, T)
    assert dup - base == T * 2 * F                       # 2 directed messages, no new pair
    new_type = mpnn_molecule_flops([0, 1, 2], [(0, 1, 0), (1, 2, 1), (0, 1, 3)], F, T)
    assert new_type - base == T * (2 * 2 * F * F + 2 * F)  # pairs (0,3), (1,3) are new
    perm = mpnn_molecule_flops([2, 1, 0], [(2, 1, 0), (1, 0, 1)], F, T)
    assert perm == base
    assert mpnn_molecule_flops([5], [], F, T) == T * (2 * F * F + 2 * F) + F + 2 * F * F + 4 * F
    mol = molecules(3, 50)
    for m in range(50):
        types, edges = molecule_of(mol, m)
        pairs = sum(1 for a, b in itertools.product(range(len(types)), range(4))
                    if any(b == eb and a in (u, v) for (u, v, eb) in edges))
        n, E = len(types), len(edges)
        want = T * (2 * F * F * (n + pairs) + 2 * E * F + 2 * n * F) + n * F + 2 * F * F + 4 * F
        assert mpnn_molecule_flops(types, edges, F, T) == want
    assert mpnn_task_flops(mol, F, T) == sum(
        mpnn_molecule_flops(*molecule_of(mol, m), F, T) for m in range(50))


def _bf16_bytes(arrs):
    return sum(2 * a.size for a in arrs)


def test_decode_bytes_from_generated_tensors_tiny():
    """C1 task bytes counted from the tensors the generator produces (bf16 = 2 B
    per element) and the KV-cache geometry, term by term:
      weights per step   = every layer tensor once             (S steps)
      LM head + g_final  = read at the G steps whose logits are used (R5)
      embedding row      = d bf16 per step and sequence
      KV written         = one position (K and V, all layers) per step
      KV read            = positions 0..t at step t -> sum_{t<S} (t+1)
    TINY, B = 1, P = 8, G = 16 (S = 23) gives 87,449,088 B."""
    cfg, B, P, G = TINY, 1, 8, 16
    S = P + G - 1
    w = decode_weights(cfg)
    layers = _bf16_bytes(a for lw in w["layers"] for a in lw.values())
    head = _bf16_bytes([w["lm_head"], w["g_final"]])
    embed_row = 2 * w["embed"].shape[1]
    kv_pos = cfg.n_layers * 2 * cfg.n_kv_heads * cfg.head_dim * 2
    kv_read = sum(t + 1 for t in range(S)) * kv_pos * B
    want = S * layers + G * head + S * B * embed_row + kv_read + S * B * kv_pos
    assert want == 87_449_088
    assert decode_task_bytes(cfg, B, P, G) == want
    assert decode_layer_weight_bytes(cfg) * cfg.n_layers == layers
    assert decode_head_bytes(cfg) == head


def test_r5_reconciles_with_survey_figures():
    """SURVEY.md §8(a) a6 / D2 quote 91,122,688 B (C1) and 11,657,203,200 B
    (C2) per task, counting the LM head at all S = P+G-1 steps. Reading R5
    counts it at G steps: the figures differ by exactly (S - G) head reads."""
    for cfg, P, G, survey in ((TINY, 8, 16, 91_122_688), (GPT2S, 16, 32, 11_657_203_200)):
        S = P + G - 1
        ours = decode_task_bytes(cfg, 1, P, G)
        assert survey - ours == (S - G) * decode_head_bytes(cfg)
    assert decode_task_bytes(GPT2S, 1, 16, 32) == 10_499_258_880
    # D3: 7B per-task bytes grow with the batch only through KV and embedding rows
    b1, b8 = decode_task_bytes(LLAMA7B, 1, 16, 32), decode_task_bytes(LLAMA7B, 8, 16, 32)
    S = 47
    kv_pos = 32 * 2 * 4096 * 2
    assert b8 - b1 == 7 * (S * 2 * 4096 + kv_pos * S * (S + 1) // 2 + S * kv_pos)


def test_7b_parameter_count():
    """Public Llama-2-7B parameter count 6,738,415,616 (A8) from the byte model:
    32 layers (incl. two norm gains each) + LM head + embedding + final gain."""
    c = LLAMA7B
    n = (decode_layer_weight_bytes(c) * c.n_layers) // 2 + 2 * c.vocab * c.d_model + c.d_model
    assert n == 6_738_415_616
