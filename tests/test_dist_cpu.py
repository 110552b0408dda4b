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
    tasks, gpus = bench.sum_over_ranks([700 * 3, 1], dist)
    q.put((rank, span, wall, tasks, gpus))
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
    # spans: max over ranks; task and GPU counts: summed (weak scaling)
    assert got == [(0, 2.0, 5.0, 4200.0, 2.0), (1, 2.0, 5.0, 4200.0, 2.0)]


def test_single_rank_passthrough():
    import bench
    assert bench.max_over_ranks([3, 4], None) == [3.0, 4.0]
    assert bench.sum_over_ranks([3, 4], None) == [3.0, 4.0]


def test_local_devices_one_process_or_one_rank_per_gpu():
    """`bench.py --gpus N` without torchrun drives N GPUs from one process (the
    library's own multi-GPU path: one dispatcher per GPU, global placement);
    under torchrun each rank drives its LOCAL_RANK GPU."""
    import bench
    assert bench.local_devices(1, 1, 0) == [0]
    assert bench.local_devices(8, 1, 0) == list(range(8))
    assert bench.local_devices(8, 8, 5) == [5]
    assert bench.local_devices(0, 1, 0) == [0]
