"""N2 right-sizing on the GPU (Fig. 2 P:150,
P:161 "LLaMa2 can only properly utilize about 20 SMs", future work P:252):
fn_rightsize measures the function alone on each candidate partition size and
its choice must equal the policy (mx_rightsize, pinned on hand-computed cases
in test_abi_host.py) applied to that measured curve; the chosen layout then
serves tasks whose outputs match the oracle."""
import numpy as np
import pytest

from oracle import decode as od
from workloads.configs import TINY
from workloads.inputs import prompt_tokens
from workloads.weights import decode_weights

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("objective,slack", [(1, 0.0), (0, 0.10)])
def test_fn_rightsize_matches_policy_on_measured_curve(mxlib, objective, slack):
    cfg = TINY
    fn = mxlib.fn_register(mxlib.decode_desc(cfg))
    sample = mxlib.decode_task(fn, prompt_tokens(1, 1, 8, cfg.vocab), 8)
    cand = [4, 8, 16, 36, 72, 148]
    r = mxlib.fn_rightsize(fn, 0, sample, cand, hbm_bytes=256 << 20, reps=2,
                           objective=objective, slack=slack)
    sms = [c for c, _ in r["curve"]]
    t = [v for _, v in r["curve"]]
    assert sms == cand and all(v > 0 for v in t)
    want = mxlib.rightsize(sms, t, total_sms=148, max_parts=64, objective=objective, slack=slack)
    assert (r["sm"], r["parts"]) == want[:2]
    assert r["parts"] * r["sm"] <= 148
    # the sample's outputs are real results
    o_tok, _, _ = od.greedy_task(cfg, decode_weights(cfg), prompt_tokens(1, 1, 8, cfg.vocab), 8)
    assert np.array_equal(sample.tokens, o_tok)
    # the chosen layout serves tasks
    parts = [mxlib.part_create(0, r["sm"], 256 << 20) for _ in range(min(r["parts"], 8))]
    try:
        ts = []
        for k in range(2 * len(parts)):
            t_ = mxlib.decode_task(fn, prompt_tokens(10 + k, 1, 8, cfg.vocab), 4)
            mxlib.fn_submit(mxlib.MX_PART_ANY, t_)
            ts.append((k, t_))
        for k, t_ in ts:
            assert mxlib.fn_wait(t_)["status"] == 0
            o, _, _ = od.greedy_task(cfg, decode_weights(cfg), prompt_tokens(10 + k, 1, 8, cfg.vocab), 4)
            assert np.array_equal(t_.tokens, o)
    finally:
        for p in parts:
            mxlib.part_destroy(p)
    print(f"N2 objective {objective}: curve {r['curve']} -> {r['parts']} x {r['sm']} SMs")


def test_fn_rightsize_rejects_bad_arguments(mxlib):
    fn = mxlib.fn_register(mxlib.decode_desc(TINY))
    other = mxlib.fn_register(mxlib.decode_desc(TINY))
    sample = mxlib.decode_task(fn, prompt_tokens(1, 1, 4, TINY.vocab), 2)
    for cand in ([8, 4], [0, 8]):
        with pytest.raises(mxlib.MxError) as e:
            mxlib.fn_rightsize(fn, 0, sample, cand)
        assert e.value.code == mxlib.MX_EINVAL
    with pytest.raises(mxlib.MxError) as e:
        mxlib.fn_rightsize(other, 0, sample, [4, 8])   # sample is a task of another fn
    assert e.value.code == mxlib.MX_EINVAL
