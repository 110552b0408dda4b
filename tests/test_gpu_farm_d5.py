"""D5 (SURVEY.md §8(d), configs[4]) correctness on the full task farm: 10,000
mixed tasks (50/50 GPT-2s decode / 1024-molecule MPNN, seed-42 shuffle, WLAW
over 7 fill partitions, live part_resize between waves of 1,000 submissions —
PAPER.md §5.2 P:195 "work was divided equally", §7 P:248 live reconfiguration),
run by the same driver as tools/suite.py c5 (tools/farm.py). Checks:
  * the canonical trace equals the oracle simulator's replay of the same event
    stream byte for byte (C5; timing excluded by construction);
  * invariants I1 (exactly once), I2 (SM budget, disjoint groups after every
    create/resize), I3 (quota), I4 (per-partition FIFO), I5 (quota sum);
  * outputs of a seeded 2 % sample of the tasks equal the oracle (decode tokens
    identical; MPNN within 2e-2 of max |y|), computed on all host cores.
"""
import multiprocessing as mp
import os
import sys
import tempfile
import time

import numpy as np
import pytest

from oracle import decode as od
from oracle import invariants as I
from oracle import mpnn as om
from oracle import sched as S
from workloads.configs import GPT2S, MPNN
from workloads.inputs import prompt_tokens
from workloads.prng import draw, key
from workloads.weights import decode_weights, mpnn_weights

sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tools"))
from farm import Farm, FILL7, P_LEN, G_LEN  # noqa: E402

pytestmark = pytest.mark.gpu

N_TASKS = int(os.environ.get("MX_D5_TASKS", "10000"))
RESIZE_EVERY = N_TASKS // 10

_W = {}


def _init_worker():
    from threadpoolctl import threadpool_limits
    _W["limits"] = threadpool_limits(1)   # one BLAS thread per worker process
    _W["d"] = decode_weights(GPT2S)
    _W["m"] = mpnn_weights(MPNN)


def _oracle_decode(k):
    tok, _, margins = od.greedy_task(GPT2S, _W["d"], prompt_tokens(k, 1, P_LEN, GPT2S.vocab), G_LEN)
    return tok, margins


def _oracle_forced(args):
    """Teacher-forced oracle along the GPU's own tokens: at each step, how far
    (relative to max |logit|) the GPU's token is below the oracle's best."""
    k, gpu_tok = args
    _, lg, _ = od.greedy_task(GPT2S, _W["d"], prompt_tokens(k, 1, P_LEN, GPT2S.vocab), G_LEN,
                              forced=gpu_tok)
    lg = lg[:, 0].astype(np.float64)
    return [float((l.max() - l[t]) / np.abs(l).max()) for l, t in zip(lg, gpu_tok[0])]


# A greedy token may differ from the oracle's only at a near-tie: the GPU's
# logits differ from the oracle's by up to ~3e-4 of max |logit| at GPT-2s depth
# (bf16 KV rounding-boundary flips, A16; tests/test_gpu_parity.py C2), so an
# argmax whose oracle top-2 margin is below that can flip (reading R13,
# DESIGN.md). NEAR_TIE bounds the accepted gap with a 6x margin; it is far
# inside the 2e-2 logit tolerance of C7.
NEAR_TIE = 2e-3


def _oracle_mpnn(mol):
    return om.mpnn_task(_W["m"], mol, MPNN.steps)


def test_d5_task_farm_trace_invariants_sampled_parity(mxlib):
    mxlib.mx_shutdown()
    mxlib.mx_init([0])
    g = mxlib.mx_gpu_query(0)
    farm = Farm(mxlib)
    t0 = time.perf_counter()
    r = farm.run(FILL7, N_TASKS, RESIZE_EVERY)
    print(f"farm run {time.perf_counter() - t0:.1f} s", flush=True)
    res, items = r["results"], r["items"]
    assert len(res) == N_TASKS and all(x["status"] == 0 for x in res)
    assert len(r["resize_ms"]) > 0, "the layout must have been resized live"

    # --- canonical trace vs the simulator's replay -----------------------------
    sim = S.Sim(1, n_groups=g["n_groups"], group_size=g["group_size"], total_sms=g["sm_total"],
                mem_bytes=g["mem_bytes"])
    for ev in farm.events:
        getattr(sim, ev[0])(*ev[1:])
    with tempfile.TemporaryDirectory() as d:
        path = os.path.join(d, "trace.bin")
        mxlib.mx_trace_write(path)
        data = open(path, "rb").read()
    assert data == sim.trace_bytes(), "device trace differs from the simulator"
    recs = S.parse_trace(data)

    # --- invariants --------------------------------------------------------------
    ids = [t.id for _, _, t in items]
    assert I.i1_exactly_once(ids, res) == []
    assert I.i2_sm_budget(recs, g["sm_total"]) == []
    assert I.i3_quota([{"part": i, **q} for i, q in enumerate(r["parts_info"])]) == []
    assert I.i4_fifo([{"part": x["part"], "seq": x["seq_in_part"], "t_end": x["t_end_ns"],
                       "task": x["task"]} for x in res]) == []
    assert I.i5_quota_sum(recs, g["mem_bytes"]) == []

    # --- seeded 2 % output sample vs the oracle ------------------------------------
    n_s = max(2, N_TASKS // 50)
    kk = np.uint64(key(0xD5, 0))
    picks = sorted({int(draw(kk, np.uint64(i))) % N_TASKS for i in range(4 * n_s)})[:n_s]
    dec = [(i, items[i][1]) for i in picks if items[i][0] == "d"]
    mpn = [(i, items[i][1]) for i in picks if items[i][0] == "m"]
    # spawn (not fork): this process runs the library's dispatcher threads
    ctx = mp.get_context("spawn")
    t0 = time.perf_counter()
    with ctx.Pool(os.cpu_count() or 1, initializer=_init_worker) as pool:
        o_dec = pool.map(_oracle_decode, [k for _, k in dec])
        print(f"oracle decode sample {time.perf_counter() - t0:.1f} s", flush=True)
        o_mpn = pool.map(_oracle_mpnn, [farm.mol_of(k) for _, k in mpn])
        print(f"oracle mpnn sample {time.perf_counter() - t0:.1f} s", flush=True)
    bad, ties = [], []
    for (i, k), (o, margins) in zip(dec, o_dec):
        got = items[i][2].tokens
        if not np.array_equal(got, o):
            j = int(np.argwhere(got[0] != o[0])[0][0])
            bad.append((k, i, res[i]["part"], res[i]["epoch"], j, float(margins[j, 0])))
    if bad:
        with ctx.Pool(min(len(bad), os.cpu_count() or 1), initializer=_init_worker) as pool:
            gaps = pool.map(_oracle_forced, [(b[0], items[b[1]][2].tokens.copy()) for b in bad])
        ties = [(b, max(g)) for b, g in zip(bad, gaps) if max(g) <= NEAR_TIE]
        bad = [(b, max(g)) for b, g in zip(bad, gaps) if max(g) > NEAR_TIE]
    if bad:
        # re-run the failing tasks alone on a fresh partition: a near-tie flips
        # deterministically, a concurrency fault does not reproduce
        bad = [b for b, _ in bad]
        p = mxlib.part_create(0, 4, 1 << 30)
        alone = []
        for k, *_ in bad:
            t = mxlib.decode_task(farm.fd, prompt_tokens(k, 1, P_LEN, GPT2S.vocab), G_LEN)
            mxlib.fn_submit(p, t)
            mxlib.fn_wait(t)
            alone.append(t.tokens.copy())
        mxlib.part_destroy(p)
        det = [bool(np.array_equal(a, items[b[1]][2].tokens)) for a, b in zip(alone, bad)]
        pytest.fail(f"decode mismatches (task k, farm item, part, epoch, first step, oracle top-2 "
                    f"margin): {bad}; same tokens when re-run alone on 4 SMs: {det}")
    for (i, k), y in zip(mpn, o_mpn):
        ip = items[i][2].ip
        assert np.max(np.abs(ip - y)) / np.max(np.abs(y)) <= 2e-2, f"mpnn task {k}"
    print(f"D5 farm: {N_TASKS} tasks, {len(r['resize_ms'])} live resizes, trace SHA equal to the "
          f"simulator ({S.Sim.__name__}), I1-I5 hold, {len(dec)} decode + {len(mpn)} MPNN sampled "
          f"outputs equal the oracle; {len(ties)} decode sample(s) follow a near-tie (gap <= "
          f"{NEAR_TIE} of max |logit| under teacher forcing): {ties}")
