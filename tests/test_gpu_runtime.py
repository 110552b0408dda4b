"""GPU tests of the partition layer, cold start and placement (SURVEY.md §8(a)
a1-a4, a8, a9; invariants I1-I6). Run on a B200 through gpurun."""
import os
import tempfile

import numpy as np
import pytest

from oracle import invariants as I
from oracle import sched as S
from workloads.configs import TINY, MPNN
from workloads.inputs import prompt_tokens
from workloads.weights import decode_weights, mpnn_weights

pytestmark = pytest.mark.gpu


def test_gpu_query_b200(mxlib):
    g = mxlib.mx_gpu_query(0)
    assert g["cc_major"] == 10
    assert g["sm_total"] == 148
    assert g["group_size"] in (4, 8) and g["n_groups"] * g["group_size"] <= 148
    print("gpu:", g)


def test_partition_sm_budget_and_isolation(mxlib, parts):
    """I2 + I6: concurrently running probes of two partitions land on disjoint SM
    sets, each no larger than its budget (§4.1: a GPU% caps the SMs)."""
    a, b = parts(72), parts(72)
    qa, qb = mxlib.part_query(a), mxlib.part_query(b)
    assert qa["sm_count"] == 72 and qb["sm_count"] == 72 and qa["group_mask"] & qb["group_mask"] == 0
    sm = mxlib.probe_smids_concurrent([a, b], n_ctas=4 * 72, spin_ns=3_000_000)
    sa, sb = set(sm[0].tolist()), set(sm[1].tolist())
    print("partition SMs:", sorted(sa), sorted(sb))
    assert I.i6_smid_subset(sa, set(), qa["n_ctas"]) == []
    assert I.i6_smid_subset(sb, set(), qb["n_ctas"]) == []
    assert not (sa & sb)
    assert len(sa) == qa["n_ctas"] and len(sb) == qb["n_ctas"]


def test_small_partition_probe(mxlib, parts):
    p = parts(8)
    s = set(mxlib.probe_smids(p, 64, 100_000).tolist())
    assert 1 <= len(s) <= mxlib.part_query(p)["n_ctas"] <= 8 + 0


def test_sm_budget_exhaustion_enosm(mxlib, parts):
    g = mxlib.mx_gpu_query(0)
    gs, ng = g["group_size"], g["n_groups"]
    ps = [parts((ng // 2) * gs), parts((ng // 2) * gs)]
    with pytest.raises(mxlib.MxError) as e:
        parts((ng - 2 * (ng // 2) + 1) * gs)
    assert e.value.code == mxlib.MX_ENOSM
    assert sum(mxlib.part_query(p)["sm_count"] for p in ps) <= 148


def test_weights_generated_on_device_bit_exact(mxlib, parts):
    """K1: the device generator reproduces workloads/prng.py bit for bit (C1)."""
    p = parts(16)
    fn = mxlib.fn_register(mxlib.decode_desc(TINY))
    mxlib.fn_load(fn, p)
    w = decode_weights(TINY)
    checks = [(0, w["embed"]), (16 + 0, w["layers"][0]["wq"]), (16 + 2, w["layers"][0]["wv"]),
              (32 + 6, w["layers"][1]["w_down"]), (32 + 7, w["layers"][1]["g_attn"]),
              (48, w["g_final"]), (49, w["lm_head"])]
    for tid, ref in checks:
        got = mxlib.fn_read_tensor(fn, p, tid, ref.size)
        want = (np.ascontiguousarray(ref, dtype=np.float32).view(np.uint32) >> 16).astype(np.uint16)
        assert np.array_equal(got, want.ravel()), tid
    fm = mxlib.fn_register(mxlib.mpnn_desc(MPNN, 8, 256, 512))
    mxlib.fn_load(fm, p)
    mw = mpnn_weights(MPNN)
    for tid, ref in [(0, mw["e_atom"]), (3, mw["w_b"][2]), (5, mw["u"]), (10, np.array([mw["c2"]]))]:
        got = mxlib.fn_read_tensor(fm, p, tid, ref.size)
        want = (np.ascontiguousarray(ref, dtype=np.float32).view(np.uint32) >> 16).astype(np.uint16)
        assert np.array_equal(got, want.ravel()), tid


def test_quota_enforced_enomem(mxlib, parts):
    """I3: loading weights beyond the partition quota fails with MX_ENOMEM
    (MIG memory slice analog, §4.2; reading A23)."""
    p = parts(8, hbm=2 << 20)
    fn = mxlib.fn_register(mxlib.decode_desc(TINY))
    with pytest.raises(mxlib.MxError) as e:
        mxlib.fn_load(fn, p)
    assert e.value.code == mxlib.MX_ENOMEM
    q = mxlib.part_query(p)
    assert I.i3_quota([{"part": p, **q}]) == []


def test_resize_shrink_below_used_is_busy(mxlib, parts):
    p = parts(16, hbm=64 << 20)
    fn = mxlib.fn_register(mxlib.decode_desc(TINY))
    mxlib.fn_load(fn, p)
    used = mxlib.part_query(p)["hbm_used"]
    with pytest.raises(mxlib.MxError) as e:
        mxlib.part_resize(p, 0, used // 2)
    assert e.value.code == mxlib.MX_EBUSY


def test_wait_semantics(mxlib, parts):
    p = parts(16)
    fn = mxlib.fn_register(mxlib.decode_desc(TINY))
    t = mxlib.decode_task(fn, prompt_tokens(1, 1, 8, TINY.vocab), 4)
    mxlib.fn_submit(p, t)
    r = mxlib.fn_wait(t)
    assert r["status"] == 0 and r["part"] == p
    with pytest.raises(mxlib.MxError) as e:
        mxlib.fn_wait(t)
    assert e.value.code == mxlib.MX_ENOENT
    with pytest.raises(mxlib.MxError) as e:
        mxlib.part_destroy(10_000)
    assert e.value.code == mxlib.MX_EINVAL


def test_trace_matches_simulator_with_resize(mxlib):
    """Bit-exact canonical trace (C5) for a create / submit / resize / destroy
    stream, tasks running on the device; I1, I2, I4 on the results."""
    mxlib.mx_shutdown()
    mxlib.mx_init([0])
    g = mxlib.mx_gpu_query(0)
    sim = S.Sim(1, n_groups=g["n_groups"], group_size=g["group_size"], total_sms=g["sm_total"],
                mem_bytes=g["mem_bytes"])
    fn = mxlib.fn_register(mxlib.decode_desc(TINY))
    quota = 256 << 20
    pa = mxlib.part_create(0, 72, quota)
    pb = mxlib.part_create(0, 40, quota)
    sim.create(0, 72, quota)
    sim.create(0, 40, quota)
    tasks, ids = [], []
    for k in range(1, 13):
        if k == 7:
            mxlib.part_resize(pa, 32, 0)
            sim.resize(pa, 32, 0)
        t = mxlib.decode_task(fn, prompt_tokens(k, 1, 8, TINY.vocab), 8)
        part = S.MX_PART_ANY if k % 3 else S.static_part(k, 2)
        mxlib.fn_submit(part, t)
        cost = mxlib.task_default_cost(mxlib.decode_desc(TINY), t)
        sim.submit(fn, part, cost)
        tasks.append(t)
        ids.append(t.id)
    res = [mxlib.fn_wait(t) for t in tasks]
    mxlib.part_destroy(pb)
    sim.destroy(pb)
    with tempfile.TemporaryDirectory() as d:
        path = os.path.join(d, "trace.bin")
        mxlib.mx_trace_write(path)
        data = open(path, "rb").read()
        assert os.path.exists(path + ".timing")
    assert data == sim.trace_bytes()
    recs = S.parse_trace(data)
    assert I.i1_exactly_once(ids, res) == []
    assert I.i2_sm_budget(recs, g["sm_total"]) == []
    assert I.i4_fifo([{"part": r["part"], "seq": r["seq_in_part"], "t_end": r["t_end_ns"],
                       "task": r["task"]} for r in res]) == []
    assert all(r["status"] == 0 for r in res)
    mxlib.part_destroy(pa)
