"""Fault paths of the C ABI (SURVEY.md §8(b) error table; §4b.7; §4.2
P:136 isolation, §2.2.1 P:63 futures): every task completes exactly once with
a status, errors never lose or duplicate a task, and a partition keeps serving
correct results after a device error on one of its tasks."""
import numpy as np
import pytest

from oracle import decode as od
from oracle import mpnn as om
from workloads.configs import TINY, GPT2S, MPNN
from workloads.inputs import prompt_tokens, molecules
from workloads.weights import decode_weights, mpnn_weights

pytestmark = pytest.mark.gpu


def test_wait_timeout_leaves_task_waitable(mxlib, parts):
    """MX_ETIMEDOUT: a GPT-2s task on 4 SMs runs ~60 ms; a 1 us wait times out,
    the task stays waitable, the next wait succeeds once, then MX_ENOENT."""
    p = parts(4)
    fn = mxlib.fn_register(mxlib.decode_desc(GPT2S))
    mxlib.fn_load(fn, p)
    t = mxlib.decode_task(fn, prompt_tokens(1, 1, 16, GPT2S.vocab), 32)
    mxlib.fn_submit(p, t)
    with pytest.raises(mxlib.MxError) as e:
        mxlib.fn_wait(t, timeout_ns=1000)
    assert e.value.code == mxlib.MX_ETIMEDOUT
    r = mxlib.fn_wait(t)
    assert r["status"] == 0
    with pytest.raises(mxlib.MxError) as e:
        mxlib.fn_wait(t)
    assert e.value.code == mxlib.MX_ENOENT


def test_destroy_with_pending_work_is_busy(mxlib):
    """part_destroy while a task is queued or in flight: MX_EBUSY; the task
    still completes, then the destroy succeeds."""
    p = mxlib.part_create(0, 4, 1 << 30)
    fn = mxlib.fn_register(mxlib.decode_desc(GPT2S))
    mxlib.fn_load(fn, p)
    ts = [mxlib.decode_task(fn, prompt_tokens(k, 1, 16, GPT2S.vocab), 32) for k in (1, 2, 3)]
    for t in ts:
        mxlib.fn_submit(p, t)
    with pytest.raises(mxlib.MxError) as e:
        mxlib.part_destroy(p)
    assert e.value.code == mxlib.MX_EBUSY
    assert all(mxlib.fn_wait(t)["status"] == 0 for t in ts)
    mxlib.part_destroy(p)


def test_bad_device_and_handles(mxlib):
    """MX_ENODEV for a GPU index outside the initialised set; MX_EINVAL for
    unknown partitions, functions and non-positive SM counts."""
    n = mxlib.mx_gpu_count()
    for call, code in ((lambda: mxlib.part_create(n, 8, 1 << 28), mxlib.MX_ENODEV),
                       (lambda: mxlib.part_create(-1, 8, 1 << 28), mxlib.MX_ENODEV),
                       (lambda: mxlib.mx_gpu_query(n), mxlib.MX_ENODEV),
                       (lambda: mxlib.part_create(0, 0, 1 << 28), mxlib.MX_EINVAL),
                       (lambda: mxlib.part_destroy(9999), mxlib.MX_EINVAL),
                       (lambda: mxlib.part_resize(9999, 8, 0), mxlib.MX_EINVAL),
                       (lambda: mxlib.fn_load(9999, 0), mxlib.MX_EINVAL),
                       (lambda: mxlib.fn_wait(10 ** 12), mxlib.MX_ENOENT)):
        with pytest.raises(mxlib.MxError) as e:
            call()
        assert e.value.code == code, (e.value.code, code)


@pytest.mark.parametrize("logits", [False, True])
def test_device_error_completes_once_and_partition_recovers(mxlib, parts, logits):
    """A task whose kernel reports a device error (mx_debug_inject_error: the
    same completion-record path as a bounded-wait timeout) completes exactly
    once with MX_EDEVICE, in FIFO order; the partition's next tasks on the same
    slot produce oracle-identical outputs. Both completion modes: host flag
    (no logits) and event + copy (parity mode)."""
    cfg = TINY
    p = parts(8)
    fn = mxlib.fn_register(mxlib.decode_desc(cfg))
    mxlib.fn_load(fn, p)
    w = decode_weights(cfg)
    mxlib.debug_inject_error(p, 7)
    ts = []
    for k in range(1, 5):
        t = mxlib.decode_task(fn, prompt_tokens(k, 1, 8, cfg.vocab), 6, want_logits=logits,
                              vocab=cfg.vocab)
        mxlib.fn_submit(p, t)
        ts.append((k, t))
    res = [mxlib.fn_wait(t) for _, t in ts]
    assert res[0]["status"] == mxlib.MX_EDEVICE
    assert [r["status"] for r in res[1:]] == [0, 0, 0]
    assert [r["seq_in_part"] for r in res] == sorted(r["seq_in_part"] for r in res)
    for k, t in ts[1:]:
        o_tok, _, _ = od.greedy_task(cfg, w, prompt_tokens(k, 1, 8, cfg.vocab), 6)
        assert np.array_equal(t.tokens, o_tok)
    for _, t in ts:
        with pytest.raises(mxlib.MxError):
            mxlib.fn_wait(t)


def test_mpnn_device_error_then_recovery(mxlib, parts):
    p = parts(8)
    fn = mxlib.fn_register(mxlib.mpnn_desc(MPNN, 64, 64 * 32, 64 * 64))
    mol = molecules(9, 40)
    mxlib.debug_inject_error(p, 3)
    a, b = mxlib.mpnn_task(fn, mol), mxlib.mpnn_task(fn, mol)
    mxlib.fn_submit(p, a)
    mxlib.fn_submit(p, b)
    assert mxlib.fn_wait(a)["status"] == mxlib.MX_EDEVICE
    assert mxlib.fn_wait(b)["status"] == 0
    y = om.mpnn_task(mpnn_weights(MPNN), mol, MPNN.steps)
    assert np.max(np.abs(b.ip - y)) / np.max(np.abs(y)) <= 2e-2


def test_inject_error_rejects_bad_arguments(mxlib, parts):
    p = parts(4)
    for part, code in ((p, 0), (p, -1), (9999, 5)):
        with pytest.raises(mxlib.MxError) as e:
            mxlib.debug_inject_error(part, code)
        assert e.value.code == mxlib.MX_EINVAL
