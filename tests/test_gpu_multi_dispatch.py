"""The library's in-process multi-GPU path (one dispatcher
thread per GPU, one placement over all partitions of all GPUs, no collective)
exercised on a single B200 by initialising the same device twice: the library
then runs two GPU objects — two dispatchers, two SM splits, two weight pools —
exactly as it would on two devices. Placement, the canonical trace (vs the
simulator with n_gpus = 2), per-GPU FIFO and outputs vs the oracle are
checked; bench.py's `--devices 0,0` uses the same path."""
import os
import tempfile

import numpy as np
import pytest

from oracle import decode as od
from oracle import invariants as I
from oracle import sched as S
from workloads.configs import TINY
from workloads.inputs import prompt_tokens
from workloads.weights import decode_weights

pytestmark = pytest.mark.gpu


def test_two_dispatchers_one_process_global_placement(mxlib):
    mxlib.mx_shutdown()
    mxlib.mx_init([0, 0])
    try:
        assert mxlib.mx_gpu_count() == 2
        g = mxlib.mx_gpu_query(0)
        sim = S.Sim(2, n_groups=g["n_groups"], group_size=g["group_size"], total_sms=g["sm_total"],
                    mem_bytes=g["mem_bytes"])
        fn = mxlib.fn_register(mxlib.decode_desc(TINY))
        quota = 128 << 20
        sizes = [(0, 40), (0, 16), (1, 24), (1, 16), (1, 8)]
        parts = []
        for gpu, sm in sizes:
            parts.append(mxlib.part_create(gpu, sm, quota))
            sim.create(gpu, sm, quota)
        tasks = []
        desc = mxlib.decode_desc(TINY)
        for k in range(1, 25):
            t = mxlib.decode_task(fn, prompt_tokens(k, 1, 8, TINY.vocab), 6)
            part = S.MX_PART_ANY if k % 4 else parts[k % len(parts)]
            mxlib.fn_submit(part, t)
            sim.submit(fn, part, mxlib.task_default_cost(desc, t))
            tasks.append((k, t))
        res = [mxlib.fn_wait(t) for _, t in tasks]
        assert all(r["status"] == 0 for r in res)
        assert {r["gpu"] for r in res} == {0, 1}, "WLAW must place onto both GPUs' partitions"
        for r in res:
            assert r["gpu"] == sizes[parts.index(r["part"])][0]
        w = decode_weights(TINY)
        for (k, t), r in zip(tasks, res):
            o, _, _ = od.greedy_task(TINY, w, prompt_tokens(k, 1, 8, TINY.vocab), 6)
            assert np.array_equal(t.tokens, o), (k, r["gpu"], r["part"])
        for p in parts:
            mxlib.part_destroy(p)
            sim.destroy(p)
        with tempfile.TemporaryDirectory() as d:
            path = os.path.join(d, "trace.bin")
            mxlib.mx_trace_write(path)
            data = open(path, "rb").read()
        assert data == sim.trace_bytes()
        recs = S.parse_trace(data)
        assert I.i2_sm_budget(recs, g["sm_total"]) == []
        assert I.i4_fifo([{"part": r["part"], "seq": r["seq_in_part"], "t_end": r["t_end_ns"],
                           "task": r["task"]} for r in res]) == []
    finally:
        mxlib.mx_shutdown()
        mxlib.mx_init([0])
