"""Pins for the placement simulator and invariants (C6)."""
import itertools

import pytest
from hypothesis import given, settings, strategies as st

from oracle import sched as S
from oracle import invariants as I
from oracle.cost import decode_task_bytes, decode_layer_weight_bytes, decode_head_bytes
from workloads.configs import TINY, GPT2S, LLAMA7B


def test_static_is_round_robin_from_task_1():
    # P:195 "each process will complete 25 text completion tasks" for 4 processes
    counts = [0] * 4
    for k in range(1, 101):
        counts[S.static_part(k, 4)] += 1
    assert counts == [25] * 4 and S.static_part(1, 4) == 0 and S.static_part(2, 4) == 1


def test_wlaw_equal_sizes_equal_costs_is_round_robin():
    sim = S.Sim(1)
    ps = [sim.create(0, 16, 1 << 30) for _ in range(7)]
    parts = [sim.submit(1, S.MX_PART_ANY, 1000)[1] for _ in range(70)]
    assert parts == [ps[i % 7] for i in range(70)]


def _brute_force_wlaw(sizes, costs):
    """Enumerate the choice at each step: the chosen part must minimise (A+c)/s with the
    lowest id among ties; exact rational comparison via fractions."""
    from fractions import Fraction
    A = [0] * len(sizes)
    out = []
    for c in costs:
        vals = [Fraction(A[p] + c, sizes[p]) for p in range(len(sizes))]
        best = min(range(len(sizes)), key=lambda p: (vals[p], p))
        out.append(best)
        A[best] += c
    return out


def test_wlaw_brute_force_small():
    for sizes in itertools.product([8, 16, 24], repeat=3):
        for costs in itertools.product([1, 2, 5], repeat=4):
            sim = S.Sim(1)
            ps = [sim.create(0, s, 1) for s in sizes]
            got = [sim.submit(1, S.MX_PART_ANY, c)[1] for c in costs]
            assert got == [ps[i] for i in _brute_force_wlaw(sizes, costs)]


def test_group_allocation_layouts_and_errors():
    sim = S.Sim(1)
    fill14 = [16, 16, 16, 16] + [8] * 10
    ids = [sim.create(0, s, 1) for s in fill14]
    assert sum(sim.parts[i].sm_count for i in ids) == 144
    with pytest.raises(S.SchedError) as e:
        sim.create(0, 8, 1)
    assert e.value.code == S.MX_ENOSM
    with pytest.raises(S.SchedError) as e:
        sim.create(1, 8, 1)
    assert e.value.code == S.MX_ENODEV
    # whole device needs every group free
    sim2 = S.Sim(1)
    w = sim2.create(0, 148, 1)
    assert sim2.parts[w].sm_count == 148 and sim2.parts[w].whole
    with pytest.raises(S.SchedError):
        sim2.create(0, 8, 1)
    # odd requests round up to 8-SM groups (A20)
    sim3 = S.Sim(1)
    assert sim3.parts[sim3.create(0, 20, 1)].sm_count == 24


def test_resize_releases_own_groups_first():
    sim = S.Sim(1)
    a = sim.create(0, 72, 1)        # groups 0..8
    b = sim.create(0, 72, 1)        # groups 9..17
    sim.resize(a, 40, 0)            # -> groups 0..4
    assert sim.parts[a].groups == [0, 1, 2, 3, 4] and sim.parts[a].epoch == 1
    with pytest.raises(S.SchedError):
        sim.resize(a, 80, 0)        # 10 groups, only 9 free incl. own
    assert sim.parts[a].groups == [0, 1, 2, 3, 4]
    sim.destroy(b)
    sim.resize(a, 148, 0)
    assert sim.parts[a].whole


def test_quota_sum_limit():
    sim = S.Sim(1, mem_bytes=100)
    sim.create(0, 8, 60)
    with pytest.raises(S.SchedError) as e:
        sim.create(0, 8, 41)
    assert e.value.code == S.MX_ENOMEM


def test_trace_format_roundtrip():
    sim = S.Sim(2)
    p0 = sim.create(0, 72, 5)
    p1 = sim.create(1, 72, 5)
    sim.submit(1, S.MX_PART_ANY, 3)
    sim.resize(p0, 40, 0)
    sim.destroy(p1)
    recs = S.parse_trace(sim.trace_bytes())
    assert recs[0][:3] == (S.REC_HEADER, S.TRACE_VERSION, 2)
    assert [r[0] for r in recs[1:]] == [1, 1, 4, 2, 3]
    assert recs[3] == (S.REC_PLACE, 1, 1, 0, p0, 0, 0, 3)
    assert len(sim.trace_sha256()) == 64


events = st.lists(st.tuples(st.sampled_from(["c", "r", "d", "s", "x"]), st.integers(0, 2),
                            st.integers(1, 160), st.integers(1, 40)), min_size=1, max_size=60)


@settings(max_examples=150, deadline=None)
@given(events)
def test_random_event_streams_keep_invariants(evs):
    sim = S.Sim(3, mem_bytes=100)
    for kind, gpu, sm, x in evs:
        try:
            if kind == "c":
                sim.create(gpu, sm, x)
            elif kind == "x":
                sim.create_shared(gpu, sm, x)
            elif kind == "r" and sim.parts:
                sim.resize(x % len(sim.parts), sm, x)
            elif kind == "d" and sim.parts:
                sim.destroy(x % len(sim.parts))
            elif kind == "s":
                sim.submit(1, S.MX_PART_ANY, x)
        except S.SchedError:
            pass
    recs = S.parse_trace(sim.trace_bytes())
    assert I.i2_sm_budget(recs) == []
    assert I.i5_quota_sum(recs, 100) == []
    seqs = {}
    for r in recs:
        if r[0] == S.REC_PLACE:
            assert seqs.get(r[4], -1) + 1 == r[5]       # FIFO seq per partition
            seqs[r[4]] = r[5]


def test_shared_partitions_take_no_groups_and_weigh_by_grid():
    """N1 (Table 1): unpartitioned streams own
    no SM groups, so the whole device can still be partitioned next to them; their
    WLAW weight is the grid size: with grids 148 and 37 (4:1) and equal costs,
    the first 5 ANY placements go 4 to the big grid and 1 to the small one."""
    sim = S.Sim(1, n_groups=37, group_size=4)
    a = sim.create_shared(0, 148, 10)
    b = sim.create_shared(0, 37, 10)
    assert sim.parts[a].sm_count == 148 and sim.parts[a].groups == []
    assert sim.create_shared(0, 1000, 10) == 2 and sim.parts[2].sm_count == 148
    whole = sim.create(0, 148, 10)            # every group is still free
    assert sim.parts[whole].whole
    sim.destroy(whole)
    sim.destroy(2)
    got = [sim.submit(1, S.MX_PART_ANY, 100)[1] for _ in range(5)]
    assert sorted(got) == [a, a, a, a, b]
    sim.resize(b, 74, 0)                      # stays shared, grid 74
    assert sim.parts[b].groups == [] and sim.parts[b].sm_count == 74
    recs = S.parse_trace(sim.trace_bytes())
    assert [r[7] for r in recs if r[0] == S.REC_CREATE] == [2, 2, 2, 1]
    assert I.i2_sm_budget(recs) == []
    with pytest.raises(S.SchedError):
        sim.create_shared(0, 0, 10)


def test_invariant_checkers_detect_violations():
    assert I.i1_exactly_once([1, 2], [{"task": 1}, {"task": 1}]) != []
    assert I.i1_exactly_once([1, 2], [{"task": 1}, {"task": 2}]) == []
    bad = [(S.REC_CREATE, 0, 0, 80, 0b11, 1, 0, 0), (S.REC_CREATE, 1, 0, 80, 0b10, 1, 0, 0)]
    assert I.i2_sm_budget(bad) != []
    assert I.i3_quota([{"part": 0, "hbm_peak": 5, "hbm_quota": 4}]) != []
    res = [{"part": 0, "seq": 0, "t_end": 10, "task": 1}, {"part": 0, "seq": 1, "t_end": 5, "task": 2}]
    assert I.i4_fifo(res) != []
    assert I.i6_smid_subset({1, 2, 3}, {1, 2}, 8) != []


def test_decode_bytes_match_generated_tensor_sizes():
    """Independent count: bytes of the tiny model's tensors as actually generated."""
    from workloads.weights import decode_weights
    w = decode_weights(TINY)
    layer = sum(a.size for a in w["layers"][0].values()) * 2
    assert layer == decode_layer_weight_bytes(TINY)
    assert w["lm_head"].size * 2 + w["g_final"].size * 2 == decode_head_bytes(TINY)
    # 7B parameter count = the public Llama-2-7B count (A8)
    n7 = (LLAMA7B.n_layers * (decode_layer_weight_bytes(LLAMA7B) // 2)
          + 2 * LLAMA7B.vocab * LLAMA7B.d_model + LLAMA7B.d_model)
    assert n7 == 6_738_415_616


def test_metric_identity_60pct_is_2_5x():
    """P:230 (§5.2): 'reduce the time ... by up to 60%' <=> '2.5 times higher throughput'."""
    from paper_conf_sc_dhakalrwercfm23_b200.metrics import throughput_ratio, completion_reduction
    assert abs(throughput_ratio(100.0, 40.0) - 2.5) < 1e-12
    assert abs(completion_reduction(100.0, 40.0) - 0.60) < 1e-12
