"""N > 1 host logic on CPU: chunk-aligned global slices and the failure-count
all-reduce, with world_size-2 gloo process groups (no GPU needed)."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

import synth
from paper_conf_ipps_gatesklpd17_b200 import multi_gpu


@pytest.mark.parametrize("B", [0, 1, 31, 32, 1000, 4096, 1 << 20, (1 << 25) + 7])
@pytest.mark.parametrize("world", [1, 2, 3, 4, 8])
@pytest.mark.parametrize("chunk", [0, 32, 64, 512])
def test_rank_slices_partition_the_batch(B, world, chunk):
    C = chunk if chunk > 0 else 32
    nxt = 0
    for r in range(world):
        b0, cnt = multi_gpu.rank_slice(B, world, r, chunk)
        assert b0 == nxt and cnt >= 0
        if cnt and b0 + cnt < B:
            assert cnt % C == 0
        assert b0 % C == 0 or cnt == 0
        nxt = b0 + cnt
    assert nxt == B


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, n, B, chunk, P, q):
    import torch
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank),
                      WORLD_SIZE=str(world), LOCAL_RANK=str(rank))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    r, w, _ = multi_gpu.env_rank_world()
    b0, cnt = multi_gpu.rank_slice(B, w, r, chunk)
    # the per-rank count the kernel would produce, from the enumerated plan
    local = synth.expected_fail_count(n, 2018, P, b0, b0 + cnt)
    t = torch.tensor([local], dtype=torch.int32)
    total = multi_gpu.allreduce_count(t)
    q.put((rank, b0, cnt, local, total))
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_gloo_allreduce_of_failure_count(world):
    n, B, chunk, P = 32, 200_000, 32, 1009
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, n, B, chunk, P, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    expected = synth.expected_fail_count(n, 2018, P, 0, B)
    assert all(r[4] == expected for r in res)
    assert sum(r[3] for r in res) == expected
    assert sum(r[2] for r in res) == B


def _timing_worker(rank, world, port, q):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank),
                      WORLD_SIZE=str(world), LOCAL_RANK=str(rank))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    # rank r "measured" a step time of 10 + 5r ms and a mean launch of 2 - r ms
    total, launch = multi_gpu.max_over_ranks([10.0 + 5 * rank, 2.0 - rank])
    value = multi_gpu.job_throughput(1 << 20, world, total, 16 ** 3 / 3)
    q.put((rank, total, launch, value))
    dist.destroy_process_group()


def test_gloo_max_over_ranks_timing():
    """bench.py's rule: the job's step time is the MAX over ranks (every rank
    reports the same number) and the throughput is all ranks' units over it."""
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_timing_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted(q.get(timeout=120) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for _, total, launch, value in res:
        assert total == 15.0 and launch == 2.0
        assert abs(value - 2 * (1 << 20) * (16 ** 3 / 3) / 15e-3 / 1e9) < 1e-9
    assert multi_gpu.max_over_ranks([3.5]) == [3.5]          # world 1: identity
