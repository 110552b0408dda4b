"""CPU-side checks of the C-ABI library: it loads, exports every symbol that
include/mx.h declares, refuses to run without a GPU, and its placement engine
(the same C++ object the runtime uses) reproduces the oracle simulator's
canonical trace byte for byte."""
import os
import re

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

from paper_conf_sc_dhakalrwercfm23_b200 import mx
from oracle import sched as S
from oracle.cost import decode_default_cost, mpnn_default_cost, mpnn_train_default_cost
from workloads.configs import TINY, GPT2S, LLAMA7B, MPNN
from workloads.inputs import molecules, prompt_tokens, ip_targets

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared_functions():
    txt = open(os.path.join(ROOT, "include", "mx.h")).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    names = re.findall(r"^\s*(?:const\s+)?[\w\s\*]+?\b(\w+)\s*\(", txt, flags=re.M)
    return sorted(set(n for n in names if n not in ("if", "while", "sizeof")))


def test_library_exports_every_declared_symbol():
    L = mx.lib()
    names = _declared_functions()
    assert "part_create" in names and "fn_submit" in names and "mx_sched_trace" in names
    missing = [n for n in names if not hasattr(L, n)]
    assert missing == []
    assert set(names) <= set(mx._SIGS)


def test_device_calls_refuse_without_init():
    assert mx.lib().mx_gpu_count(None) == mx.MX_ESTATE
    with pytest.raises(mx.MxError) as e:
        mx.part_create(0, 8, 1 << 30)
    assert e.value.code == mx.MX_ESTATE


def _replay(events, n_gpus=2):
    sim = S.Sim(n_gpus, mem_bytes=1000)
    cpp = mx.HostSched(n_gpus, 18, 8, 148, 1000)
    for kind, a, b, c in events:
        rs = rc = None
        try:
            if kind == "c":
                sim.create(a % n_gpus, b, c)
            elif kind == "x":
                sim.create_shared(a % n_gpus, b, c)
            elif kind == "r":
                sim.resize(a % max(1, len(sim.parts)), b, c)
            elif kind == "d":
                sim.destroy(a % max(1, len(sim.parts)))
            else:
                sim.submit(1 + a % 2, S.MX_PART_ANY if b % 3 else a % max(1, len(sim.parts)), c)
        except S.SchedError as e:
            rs = e.code
        try:
            if kind == "c":
                cpp.create(a % n_gpus, b, c)
            elif kind == "x":
                cpp.create_shared(a % n_gpus, b, c)
            elif kind == "r":
                cpp.resize(a % max(1, len(sim.parts)), b, c)
            elif kind == "d":
                cpp.destroy(a % max(1, len(sim.parts)))
            else:
                cpp.submit(1 + a % 2, S.MX_PART_ANY if b % 3 else a % max(1, len(sim.parts)), c)
        except mx.MxError as e:
            rc = e.code
        assert rs == rc, (kind, a, b, c, rs, rc)
    return sim, cpp


def test_cpp_placement_trace_equals_simulator_fixed():
    ev = [("c", 0, 72, 100), ("c", 0, 72, 100), ("c", 1, 16, 10), ("s", 0, 1, 500),
          ("s", 1, 2, 700), ("r", 0, 40, 0), ("s", 2, 1, 50), ("d", 2, 0, 0), ("s", 3, 1, 9),
          ("c", 1, 148, 10), ("c", 1, 8, 10), ("c", 0, 20, 999), ("x", 0, 37, 10),
          ("x", 0, 500, 10), ("s", 1, 1, 77), ("r", 4, 74, 0), ("x", 1, 0, 5)]
    sim, cpp = _replay(ev)
    assert cpp.trace_bytes() == sim.trace_bytes()


@settings(max_examples=200, deadline=None)
@given(st.lists(st.tuples(st.sampled_from("crdsx"), st.integers(0, 20), st.integers(-5, 160),
                          st.integers(0, 400)), max_size=50))
def test_cpp_placement_trace_equals_simulator_random(events):
    sim, cpp = _replay(events)
    assert cpp.trace_bytes() == sim.trace_bytes()


def test_default_cost_matches_oracle():
    for cfg, B, P, G in [(TINY, 1, 8, 16), (GPT2S, 1, 16, 32), (LLAMA7B, 2, 16, 32)]:
        desc = mx.decode_desc(cfg, max_batch=B)
        t = mx.decode_task(1, prompt_tokens(1, B, P, cfg.vocab), G)
        assert mx.task_default_cost(desc, t) == decode_default_cost(cfg, B, P, G)
    mol = molecules(4, 40)
    desc = mx.mpnn_desc(MPNN, 64, 64 * 32, 64 * 64)
    t = mx.mpnn_task(1, mol)
    assert mx.task_default_cost(desc, t) == mpnn_default_cost(mol, MPNN.hidden, MPNN.steps)


def test_training_and_shared_weight_descriptors_host_side():
    """N4 cost rule (3x forward flops) and descriptor validation (N3/N4) are
    pure host logic in libmx.so (no GPU needed)."""
    mol = molecules(6, 24)
    tdesc = mx.mpnn_train_desc(MPNN, 32, 32 * 32, 32 * 64)
    t = mx.mpnn_train_task(1, mol, ip_targets(6, 24), 0.1)
    assert mx.task_default_cost(tdesc, t) == mpnn_train_default_cost(mol, MPNN.hidden, MPNN.steps)
    # a training step without targets is rejected
    t.desc.targets = None
    with pytest.raises(mx.MxError) as e:
        mx.task_default_cost(tdesc, t)
    assert e.value.code == mx.MX_EINVAL
    # training state is per instance: shared weights are rejected for it
    tdesc.flags = mx.MX_FN_SHARED_WEIGHTS
    with pytest.raises(mx.MxError):
        mx.task_default_cost(tdesc, mx.mpnn_train_task(1, mol, ip_targets(6, 24), 0.1))
    # shared weights are accepted for inference functions, unknown flags are not
    sdesc = mx.decode_desc(TINY, shared_weights=True)
    td = mx.decode_task(1, prompt_tokens(1, 1, 8, TINY.vocab), 4)
    assert mx.task_default_cost(sdesc, td) == decode_default_cost(TINY, 1, 8, 4)
    sdesc.flags = 0x80
    with pytest.raises(mx.MxError):
        mx.task_default_cost(sdesc, td)


def test_task_validation_rejects_bad_inputs():
    desc = mx.decode_desc(TINY, max_batch=1)
    bad = mx.decode_task(1, np.array([[TINY.vocab]], dtype=np.int32), 4)
    with pytest.raises(mx.MxError) as e:
        mx.task_default_cost(desc, bad)
    assert e.value.code == mx.MX_EINVAL
    too_long = mx.decode_task(1, np.zeros((1, 60), dtype=np.int32), 8)   # 67 > max_seq 64
    with pytest.raises(mx.MxError):
        mx.task_default_cost(desc, too_long)
    big = mx.decode_desc(LLAMA7B, max_batch=8)   # split-K: wide inputs at batch 8 are valid
    assert mx.task_default_cost(big, mx.decode_task(1, np.zeros((8, 4), dtype=np.int32), 4)) > 0
    over = mx.decode_desc(LLAMA7B, max_batch=9)  # batch > 8
    with pytest.raises(mx.MxError):
        mx.task_default_cost(over, mx.decode_task(1, np.zeros((9, 4), dtype=np.int32), 4))


def test_rightsize_policy_n2():
    """N2 right-sizing (mx_rightsize), pinned on hand-computed cases: the
    throughput objective maximises floor(148/s)/t(s); the latency objective
    takes the smallest size within (1+slack) of the fastest; ties and the
    max_parts cap; invalid inputs."""
    # D2b-shaped curve (GPT-2s decode, ms per task alone on s SMs)
    sms = [4, 8, 12, 16, 24, 32, 48, 64, 72, 96, 120, 148]
    t = [62.1, 38.9, 31.7, 27.3, 23.9, 22.1, 20.0, 19.8, 19.5, 19.3, 18.8, 18.96]
    s, n, rate = mx.rightsize(sms, t, objective=1)
    assert (s, n) == (4, 37) and abs(rate - 37 / 62.1) < 1e-12
    s, n, _ = mx.rightsize(sms, t, objective=0, slack=0.10)   # <= 20.68 ms
    assert (s, n) == (48, 3)
    s, n, _ = mx.rightsize(sms, t, objective=0, slack=0.0)    # the fastest point
    assert (s, n) == (120, 1)
    # efficiency peaking in the middle: 37/100, 18/30, 9/20 -> 8 SMs
    assert mx.rightsize([4, 8, 16], [100.0, 30.0, 20.0])[:2] == (8, 18)
    # exact tie 2/2 == 1/1 -> the larger partition
    assert mx.rightsize([4, 8], [2.0, 1.0], total_sms=8)[:2] == (8, 1)
    # max_parts caps the count: 2/1 vs 2/1.5 -> 4 SMs x 2
    assert mx.rightsize([4, 8], [1.0, 1.5], max_parts=2)[:2] == (4, 2)
    for bad in (dict(sms=[8, 4], t=[1.0, 1.0]), dict(sms=[4], t=[0.0]),
                dict(sms=[200], t=[1.0]), dict(sms=[4], t=[1.0], slack=-1.0, objective=0)):
        with pytest.raises(mx.MxError) as e:
            mx.rightsize(**bad)
        assert e.value.code == mx.MX_EINVAL
