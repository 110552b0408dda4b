"""GPU tests of shared read-only weights across partitions (
PAPER.md §7 P:250 "share the model weights", §6 P:240 cold start). One weight
copy per GPU, referenced by every partition's instance: outputs must equal the
oracle exactly as with private copies (tokens identical, logits within 2e-2),
and partition quotas hold only task slots."""
import numpy as np
import pytest

from oracle import decode as od
from oracle import invariants as I
from oracle import mpnn as om
from workloads.configs import TINY, GPT2S, MPNN
from workloads.inputs import prompt_tokens, molecules
from workloads.weights import decode_weights, mpnn_weights

pytestmark = pytest.mark.gpu

TOL = 2e-2


def test_shared_tiny_parity_and_accounting(mxlib, parts):
    """Three partitions share one tiny-decoder weight copy: the pool grows by the
    weights once, partition usage excludes them, every partition's tasks match
    the oracle (C2/C3), and the tensors read back from any partition are the
    same bf16 values (C1)."""
    before = mxlib.weight_pool_query(0)
    ps = [parts(16, hbm=64 << 20) for _ in range(3)]
    fn = mxlib.fn_register(mxlib.decode_desc(TINY, shared_weights=True))
    for p in ps:
        mxlib.fn_load(fn, p)
    after = mxlib.weight_pool_query(0)
    w = decode_weights(TINY)
    wbytes = sum(int(np.asarray(v).size) for v in _tensors(w)) * 2
    grown = after["used_bytes"] - before["used_bytes"]
    assert after["n_fns"] == before["n_fns"] + 1
    assert wbytes <= grown < wbytes + (4 << 20), (grown, wbytes)   # one copy (+ RoPE, alignment)
    for p in ps:
        q = mxlib.part_query(p)
        assert q["hbm_used"] < wbytes, q   # slots only
        assert I.i3_quota([{"part": p, **q}]) == []
    emb = [mxlib.fn_read_tensor(fn, p, 0, TINY.vocab * TINY.d_model) for p in ps]
    assert all(np.array_equal(emb[0], e) for e in emb[1:])
    tasks = []
    for k in range(1, 7):
        prompt = prompt_tokens(k, 1, 8, TINY.vocab)
        t = mxlib.decode_task(fn, prompt, 12, want_logits=True, vocab=TINY.vocab)
        mxlib.fn_submit(ps[(k - 1) % 3], t)
        tasks.append((prompt, t))
    for prompt, t in tasks:
        assert mxlib.fn_wait(t)["status"] == 0
        o_tok, o_lg, _ = od.greedy_task(TINY, w, prompt, 12)
        assert np.array_equal(t.tokens, o_tok)
        rel = np.max(np.abs(t.logits - o_lg)) / np.max(np.abs(o_lg))
        assert rel <= TOL, rel


def _tensors(w):
    """Every array of the oracle's weight dict (nested dicts / lists)."""
    if isinstance(w, dict):
        return [a for v in w.values() for a in _tensors(v)]
    if isinstance(w, (list, tuple)):
        return [a for v in w for a in _tensors(v)]
    return [w]


def test_shared_gpt2s_small_quotas_bit_identical_to_private(mxlib, parts):
    """GPT-2s weights (324 MB) do not fit a 64 MiB quota privately (MX_ENOMEM),
    but four 64 MiB partitions run it from the shared copy; their tokens and
    logits are bit-identical to a private instance's (same kernel, same bf16
    weights, row ownership independent of the partition size)."""
    small = parts(8, hbm=64 << 20)
    fp = mxlib.fn_register(mxlib.decode_desc(GPT2S))
    with pytest.raises(mxlib.MxError) as e:
        mxlib.fn_load(fp, small)
    assert e.value.code == mxlib.MX_ENOMEM
    fs = mxlib.fn_register(mxlib.decode_desc(GPT2S, shared_weights=True))
    ps = [parts(8, hbm=64 << 20) for _ in range(4)]
    priv = parts(16, hbm=512 << 20)
    prompt = prompt_tokens(3, 1, 16, GPT2S.vocab)
    ref = mxlib.decode_task(fp, prompt, 8, want_logits=True, vocab=GPT2S.vocab)
    mxlib.fn_submit(priv, ref)
    ts = []
    for p in ps:
        t = mxlib.decode_task(fs, prompt, 8, want_logits=True, vocab=GPT2S.vocab)
        mxlib.fn_submit(p, t)
        ts.append(t)
    assert mxlib.fn_wait(ref)["status"] == 0
    for p, t in zip(ps, ts):
        assert mxlib.fn_wait(t)["status"] == 0
        assert np.array_equal(t.tokens, ref.tokens)
        assert np.array_equal(t.logits, ref.logits)
        assert mxlib.part_query(p)["hbm_peak"] <= 64 << 20


def test_shared_mpnn_and_resize_keeps_weights(mxlib, parts):
    """A shared MPNN function on two partitions matches the oracle (C4/C7), and
    part_resize neither moves nor regenerates the shared weights (a9)."""
    ps = [parts(8, hbm=32 << 20), parts(8, hbm=32 << 20)]
    fm = mxlib.fn_register(mxlib.mpnn_desc(MPNN, 64, 64 * 30, 64 * 32, shared_weights=True))
    for p in ps:
        mxlib.fn_load(fm, p)
    used = mxlib.weight_pool_query(0)["used_bytes"]
    mxlib.part_resize(ps[1], 16, 0)
    mw = mpnn_weights(MPNN)
    for k, p in enumerate(ps):
        mol = molecules(40 + k, 64)
        t = mxlib.mpnn_task(fm, mol)
        mxlib.fn_submit(p, t)
        assert mxlib.fn_wait(t)["status"] == 0
        y = om.mpnn_task(mw, mol, MPNN.steps)
        assert np.max(np.abs(t.ip - y)) / np.max(np.abs(y)) <= TOL
    assert mxlib.weight_pool_query(0)["used_bytes"] == used
