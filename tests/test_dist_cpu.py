"""Multi-rank host logic of bench.py on CPU (gloo, world_size 2): the timing
reduction is a max over ranks, and task counts add up (weak scaling)."""
import os
import socket

import pytest
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import bench
    span, wall = bench.max_over_ranks([1.0 + rank, 5.0 - rank], dist)
    q.put((rank, span, wall))
    dist.barrier()
    dist.destroy_process_group()


def test_max_over_ranks_gloo_world2():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(120)
        assert p.exitcode == 0
    got = sorted(q.get() for _ in range(2))
    assert got == [(0, 2.0, 5.0), (1, 2.0, 5.0)]


def test_single_rank_passthrough():
    import bench
    assert bench.max_over_ranks([3, 4], None) == [3.0, 4.0]
