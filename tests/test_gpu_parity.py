"""GPU parity: the CUDA path (through the C ABI) vs the fp64 oracle on the same
seeded weights and inputs. Tolerances: BASELINE.json north_star — logits within
2e-2 max relative error (normalised by the max |oracle logit| per step and
sequence, reading A18), greedy tokens identical; MPNN outputs within 2e-2
normalised by max |y| (C7)."""
import numpy as np
import pytest

from oracle import decode as od
from oracle import mpnn as om
from oracle import sched as S
from workloads.configs import TINY, GPT2S, RAGGED, LLAMA7B, MPNN, SPLITK
from workloads.inputs import prompt_tokens, molecules
from workloads.weights import decode_weights, mpnn_weights

pytestmark = pytest.mark.gpu

TOL = 2e-2


def _check_decode(cfg, w, prompt, G, tokens, logits):
    o_tok, o_lg, margins = od.greedy_task(cfg, w, prompt, G)
    for j in range(G):
        for b in range(prompt.shape[0]):
            ref = o_lg[j, b].astype(np.float64)
            rel = np.max(np.abs(logits[j, b] - ref)) / np.max(np.abs(ref))
            assert rel <= TOL, (j, b, rel)
    if not np.array_equal(tokens, o_tok):
        bad = np.argwhere(tokens != o_tok)
        j, b = bad[0][1], bad[0][0]
        pytest.fail(f"token mismatch at seq {b} step {j}: gpu {tokens[b, j]} oracle {o_tok[b, j]}"
                    f" (oracle top-2 margin {margins[j, b]:.2e})")
    return max(float(np.max(np.abs(logits[j, b] - o_lg[j, b])) / np.max(np.abs(o_lg[j, b])))
               for j in range(G) for b in range(prompt.shape[0]))


def test_c1_tiny_four_tasks_two_partitions(mxlib, parts):
    """configs[0] (D1): tiny decoder, 4 tasks x 16 greedy tokens on 2 partitions,
    STATIC placement (tasks 1,3 -> p0; 2,4 -> p1; Fig. 4)."""
    cfg = TINY
    p0, p1 = parts(72), parts(72)
    fn = mxlib.fn_register(mxlib.decode_desc(cfg))
    w = decode_weights(cfg)
    tasks = []
    for k in range(1, 5):
        t = mxlib.decode_task(fn, prompt_tokens(k, 1, 8, cfg.vocab), 16, want_logits=True,
                              vocab=cfg.vocab)
        mxlib.fn_submit([p0, p1][S.static_part(k, 2)], t)
        tasks.append((k, t))
    for k, t in tasks:
        r = mxlib.fn_wait(t)
        assert r["status"] == 0
        assert r["part"] == [p0, p1][S.static_part(k, 2)]
        rel = _check_decode(cfg, w, prompt_tokens(k, 1, 8, cfg.vocab), 16, t.tokens, t.logits)
        print(f"C1 task {k}: max rel logit err {rel:.2e}, kernel {r['kernel_ns'] / 1e3:.1f} us")


def test_ragged_gqa_batch3(mxlib, parts):
    """Ragged shapes (d=264, q_dim=192, d_ff=712, V=1031: partial 256-col chunks
    and tiles), GQA (6 heads / 2 KV heads, hd 32), batch 3, on a 24-SM partition."""
    cfg = RAGGED
    p = parts(24)
    fn = mxlib.fn_register(mxlib.decode_desc(cfg, max_batch=3))
    w = decode_weights(cfg)
    prompt = prompt_tokens(5, 3, 5, cfg.vocab)
    t = mxlib.decode_task(fn, prompt, 9, want_logits=True, vocab=cfg.vocab)
    mxlib.fn_submit(p, t)
    assert mxlib.fn_wait(t)["status"] == 0
    _check_decode(cfg, w, prompt, 9, t.tokens, t.logits)


@pytest.mark.parametrize("cfg,B,sm", [(RAGGED, 5, 12), (TINY, 4, 8), (RAGGED, 8, 40)])
def test_tensor_core_batches(mxlib, parts, cfg, B, sm):
    """Batch >= 4 runs the GEMVs on the tensor cores (K7, bf16 hi/lo activations):
    ragged K (264 -> padded 288, masked), ragged rows, GQA, B = 4 / 5 / 8."""
    p = parts(sm)
    fn = mxlib.fn_register(mxlib.decode_desc(cfg, max_batch=B))
    w = decode_weights(cfg)
    prompt = prompt_tokens(40 + B, B, 6, cfg.vocab)
    t = mxlib.decode_task(fn, prompt, 7, want_logits=True, vocab=cfg.vocab)
    mxlib.fn_submit(p, t)
    assert mxlib.fn_wait(t)["status"] == 0
    rel = _check_decode(cfg, w, prompt, 7, t.tokens, t.logits)
    print(f"TC {cfg.name} B={B}: max rel err {rel:.2e}")


def test_single_token_generation_and_single_prompt(mxlib, parts):
    """Degenerate shapes: G = 1 (one LM-head step) and P = 1 (no prompt steps)."""
    cfg = TINY
    p = parts(8)
    fn = mxlib.fn_register(mxlib.decode_desc(cfg))
    w = decode_weights(cfg)
    for P, G in [(6, 1), (1, 5)]:
        prompt = prompt_tokens(9, 1, P, cfg.vocab)
        t = mxlib.decode_task(fn, prompt, G, want_logits=True, vocab=cfg.vocab)
        mxlib.fn_submit(p, t)
        assert mxlib.fn_wait(t)["status"] == 0
        _check_decode(cfg, w, prompt, G, t.tokens, t.logits)


def test_results_identical_across_partition_sizes(mxlib, parts):
    """Row ownership + fixed reduction order => bit-identical outputs for any SM
    budget (8, 40, whole-device-sized 144 SMs)."""
    cfg = TINY
    fn = mxlib.fn_register(mxlib.decode_desc(cfg))
    prompt = prompt_tokens(11, 1, 8, cfg.vocab)
    outs = []
    for sm in (8, 40, 96):
        p = parts(sm)
        t = mxlib.decode_task(fn, prompt, 12, want_logits=True, vocab=cfg.vocab)
        mxlib.fn_submit(p, t)
        assert mxlib.fn_wait(t)["status"] == 0
        outs.append((t.tokens.copy(), t.logits.copy()))
        mxlib.part_destroy(p)
    for tok, lg in outs[1:]:
        assert np.array_equal(tok, outs[0][0])
        assert np.array_equal(lg.view(np.uint32), outs[0][1].view(np.uint32))


@pytest.mark.parametrize("B,sms", [(1, (36, 148)), (8, (36, 148)), (3, (52, 100))])
def test_llama7b_width_identical_chained_vs_distributed(mxlib, parts, B, sms):
    """7B widths (2 layers): on 36 SMs every CTA chains the K segments of its
    own rows; on 148 SMs the O/DOWN pieces are spread over the CTAs and
    finished by other CTAs, and the attention runs key-block split. The row
    sums keep the segment order either way, so tokens and logits must be
    bit-identical; and both match the oracle."""
    cfg = LLAMA7B.with_layers(2)
    fn = mxlib.fn_register(mxlib.decode_desc(cfg, max_batch=B))
    prompt = prompt_tokens(40 + B, B, 5, cfg.vocab)
    outs = []
    for sm in sms:
        p = parts(sm, hbm=4 << 30)
        t = mxlib.decode_task(fn, prompt, 4, want_logits=True, vocab=cfg.vocab)
        mxlib.fn_submit(p, t)
        assert mxlib.fn_wait(t)["status"] == 0
        outs.append((t.tokens.copy(), t.logits.copy()))
        mxlib.part_destroy(p)
    assert np.array_equal(outs[0][0], outs[1][0])
    assert np.array_equal(outs[0][1].view(np.uint32), outs[1][1].view(np.uint32))
    _check_decode(cfg, decode_weights(cfg), prompt, 4, outs[1][0], outs[1][1])


def test_shared_partitions_time_share_and_concurrent(mxlib):
    """N1 modes (unpartitioned streams, cooperative launches): two time-shared
    streams (148-CTA grids competing for every SM) and two concurrent ones
    (74-CTA grids) give outputs bit-identical to a green-context partition."""
    cfg = TINY
    fn = mxlib.fn_register(mxlib.decode_desc(cfg))
    ref_p = mxlib.part_create(0, 16, 256 << 20)
    prompts = [prompt_tokens(20 + k, 1, 8, cfg.vocab) for k in range(6)]
    ref = []
    for pr in prompts:
        t = mxlib.decode_task(fn, pr, 10, want_logits=True, vocab=cfg.vocab)
        mxlib.fn_submit(ref_p, t)
        assert mxlib.fn_wait(t)["status"] == 0
        ref.append((t.tokens.copy(), t.logits.copy()))
    mxlib.part_destroy(ref_p)
    for grid in (148, 74):
        sp = [mxlib.part_create_shared(0, grid, 256 << 20) for _ in range(2)]
        info = mxlib.part_query(sp[0])
        assert info["shared"] == 1 and info["group_mask"] == 0 and info["n_ctas"] == grid
        ts = []
        for k, pr in enumerate(prompts):
            t = mxlib.decode_task(fn, pr, 10, want_logits=(k % 2 == 0), vocab=cfg.vocab)
            mxlib.fn_submit(sp[k % 2], t)
            ts.append(t)
        for k, t in enumerate(ts):
            r = mxlib.fn_wait(t)
            assert r["status"] == 0, r
            assert np.array_equal(t.tokens, ref[k][0])
            if k % 2 == 0:
                assert np.array_equal(t.logits.view(np.uint32), ref[k][1].view(np.uint32))
        for p in sp:
            mxlib.part_destroy(p)


def test_c2_gpt2s_one_task_full_size(mxlib, parts):
    """configs[1] shape at full size (12 layers, d=768, V=50257, P=16, G=32)."""
    cfg = GPT2S
    p = parts(16, hbm=1 << 30)
    fn = mxlib.fn_register(mxlib.decode_desc(cfg))
    w = decode_weights(cfg)
    prompt = prompt_tokens(1, 1, 16, cfg.vocab)
    t = mxlib.decode_task(fn, prompt, 32, want_logits=True, vocab=cfg.vocab)
    mxlib.fn_submit(p, t)
    r = mxlib.fn_wait(t)
    assert r["status"] == 0
    rel = _check_decode(cfg, w, prompt, 32, t.tokens, t.logits)
    print(f"C2 gpt2s: max rel err {rel:.2e}, kernel {r['kernel_ns'] / 1e6:.2f} ms on 16 SMs")


def test_c3_llama7b_width_two_layers(mxlib, parts):
    """configs[2] widths (d=4096, H=32, hd=128, d_ff=11008, V=32000) with 2 layers
    (the oracle cannot afford 32 fp64 layers in a test), batch 2."""
    cfg = LLAMA7B.with_layers(2)
    p = parts(32, hbm=4 << 30)
    fn = mxlib.fn_register(mxlib.decode_desc(cfg, max_batch=2))
    w = decode_weights(cfg)
    prompt = prompt_tokens(2, 2, 4, cfg.vocab)
    t = mxlib.decode_task(fn, prompt, 3, want_logits=True, vocab=cfg.vocab)
    mxlib.fn_submit(p, t)
    assert mxlib.fn_wait(t)["status"] == 0
    _check_decode(cfg, w, prompt, 3, t.tokens, t.logits)


def test_split_k_batch8_ragged_segments(mxlib, parts):
    """Split-K (inputs wider than the 64 KiB activation staging at batch 8):
    d_model 2056 and d_ff 2600 run as 2 K segments each, the second ragged;
    GQA, separate attention phase. Also batch 3 on the same instance."""
    cfg = SPLITK
    p = parts(20, hbm=1 << 30)
    fn = mxlib.fn_register(mxlib.decode_desc(cfg, max_batch=8))
    w = decode_weights(cfg)
    for B, P, G in ((8, 5, 4), (3, 3, 3)):
        prompt = prompt_tokens(31 + B, B, P, cfg.vocab)
        t = mxlib.decode_task(fn, prompt, G, want_logits=True, vocab=cfg.vocab)
        mxlib.fn_submit(p, t)
        assert mxlib.fn_wait(t)["status"] == 0
        rel = _check_decode(cfg, w, prompt, G, t.tokens, t.logits)
        print(f"split-K B={B}: max rel err {rel:.2e}")


def test_split_k_chained_vs_distributed_small(mxlib, parts):
    """The distributed DOWN phase (3 K segments, d = 2056 rows < 64 x 40 CTAs)
    and the key-block split attention at a size compute-sanitizer can afford:
    20 SMs (chained) vs 40 SMs (distributed) give bit-identical outputs, and
    both match the oracle."""
    cfg = SPLITK
    fn = mxlib.fn_register(mxlib.decode_desc(cfg, max_batch=8))
    prompt = prompt_tokens(77, 8, 5, cfg.vocab)
    outs = []
    for sm in (20, 40):
        p = parts(sm, hbm=1 << 30)
        t = mxlib.decode_task(fn, prompt, 4, want_logits=True, vocab=cfg.vocab)
        mxlib.fn_submit(p, t)
        assert mxlib.fn_wait(t)["status"] == 0
        outs.append((t.tokens.copy(), t.logits.copy()))
        mxlib.part_destroy(p)
    assert np.array_equal(outs[0][0], outs[1][0])
    assert np.array_equal(outs[0][1].view(np.uint32), outs[1][1].view(np.uint32))
    _check_decode(cfg, decode_weights(cfg), prompt, 4, outs[1][0], outs[1][1])


def test_c3_llama7b_width_batch8(mxlib, parts):
    """configs[2] widths at batch 8 (every phase but O runs split-K), 2 layers."""
    cfg = LLAMA7B.with_layers(2)
    p = parts(48, hbm=4 << 30)
    fn = mxlib.fn_register(mxlib.decode_desc(cfg, max_batch=8))
    w = decode_weights(cfg)
    prompt = prompt_tokens(3, 8, 3, cfg.vocab)
    t = mxlib.decode_task(fn, prompt, 2, want_logits=True, vocab=cfg.vocab)
    mxlib.fn_submit(p, t)
    assert mxlib.fn_wait(t)["status"] == 0
    _check_decode(cfg, w, prompt, 2, t.tokens, t.logits)


def test_mpnn_parity(mxlib, parts):
    """The scientific function (C4) vs the literal oracle on 96 molecules."""
    p = parts(16)
    mol = molecules(3, 96)
    fn = mxlib.fn_register(mxlib.mpnn_desc(MPNN, 1024, 1024 * 30, 1024 * 32))
    t = mxlib.mpnn_task(fn, mol)
    mxlib.fn_submit(p, t)
    assert mxlib.fn_wait(t)["status"] == 0
    y = om.mpnn_task(mpnn_weights(MPNN), mol, MPNN.steps)
    rel = np.max(np.abs(t.ip - y)) / np.max(np.abs(y))
    print(f"MPNN max rel err {rel:.2e}")
    assert rel <= TOL


def test_mixed_colocation_any_placement(mxlib, parts):
    """Decode and MPNN tasks sharing partitions (configs[3] shape, small), WLAW."""
    ps = [parts(24), parts(16), parts(16)]
    fd = mxlib.fn_register(mxlib.decode_desc(TINY))
    fm = mxlib.fn_register(mxlib.mpnn_desc(MPNN, 64, 64 * 30, 64 * 32))
    w = decode_weights(TINY)
    mw = mpnn_weights(MPNN)
    ts = []
    for k in range(1, 9):
        if k % 2:
            t = mxlib.decode_task(fd, prompt_tokens(k, 1, 8, TINY.vocab), 6)
        else:
            t = mxlib.mpnn_task(fm, molecules(k, 16))
        mxlib.fn_submit(S.MX_PART_ANY, t)
        ts.append((k, t))
    for k, t in ts:
        r = mxlib.fn_wait(t)
        assert r["status"] == 0 and r["part"] in ps
        if k % 2:
            o_tok, _, _ = od.greedy_task(TINY, w, prompt_tokens(k, 1, 8, TINY.vocab), 6)
            assert np.array_equal(t.tokens, o_tok)
        else:
            y = om.mpnn_task(mw, molecules(k, 16), MPNN.steps)
            assert np.max(np.abs(t.ip - y)) / np.max(np.abs(y)) <= TOL
