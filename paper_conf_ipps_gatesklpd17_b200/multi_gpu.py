"""Multi-GPU batch split (north star (5)).

One process per GPU (torchrun).  The global batch of independent matrices is
cut into contiguous, chunk-aligned slices of GLOBAL indices -- in the chunked
layout such a slice is a contiguous byte range and itself a valid chunked
array of its local batch -- so there is no inter-GPU data traffic at all.  The
only collective is one ``all_reduce(SUM)`` of the int32 failure count that
the factorization kernel already reduced per rank (warp ballot + popc + one
atomic per warp).  The matrices are independent, so no other exchange exists
(DESIGN.md "Multi-GPU").
"""
from __future__ import annotations

import os


def rank_slice(batch_global: int, world: int, rank: int, chunk: int):
    """[b0, b0 + count) of global matrix indices owned by ``rank``.

    Slices are multiples of the chunk C (32 for simple interleaved, chunk 0, so
    that every rank's warps stay full), as equal as possible; trailing ranks
    may get fewer (or zero) matrices when the batch is small."""
    if world <= 0 or not (0 <= rank < world):
        raise ValueError("bad world/rank")
    if batch_global < 0:
        raise ValueError("bad batch")
    C = chunk if chunk > 0 else 32
    per = -(-batch_global // (world * C)) * C
    b0 = min(rank * per, batch_global)
    b1 = min(b0 + per, batch_global)
    return b0, b1 - b0


def env_rank_world():
    return int(os.environ.get("RANK", "0")), int(os.environ.get("WORLD_SIZE", "1")), \
        int(os.environ.get("LOCAL_RANK", "0"))


def allreduce_count(count, group=None):
    """Global failure count: SUM over ranks of each rank's int32 count tensor
    (a CUDA tensor under NCCL, a CPU tensor under gloo).  Returns a Python int
    (synchronising)."""
    import torch.distributed as dist
    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(count, op=dist.ReduceOp.SUM, group=group)
    return int(count.item())


def max_over_ranks(values, device=None, group=None):
    """Device timings of a multi-GPU step: the MAX over ranks of each value
    (the job is as slow as its slowest rank; bench.py's timing rule).  `values`
    is a list of floats; returns the list of maxima (identity at world 1)."""
    import torch
    import torch.distributed as dist
    t = torch.tensor([float(v) for v in values], dtype=torch.float64, device=device)
    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return [float(x) for x in t.tolist()]


def job_throughput(units_per_rank, world, max_ms_per_step, flops_per_unit, global_units=None):
    """Whole-job Gflop/s: every rank's units (or the global batch when the batch
    is split) over the max-over-ranks step time."""
    units = global_units if global_units is not None else units_per_rank * world
    return units * flops_per_unit / (max_ms_per_step * 1e-3) / 1e9


class RankBatch:
    """This rank's slice of a global synthetic batch, resident on its GPU."""

    def __init__(self, n, batch_global, chunk, kind="dd", seed=2017, fail_seed=0,
                 fail_period=0, device=None):
        import torch

        from . import batch_interleaved_elems, bspotrf_synth_generate
        rank, world, local = env_rank_world()
        self.n, self.chunk = n, chunk
        self.b0, self.count = rank_slice(batch_global, world, rank, chunk)
        self.device = device or torch.device("cuda", local)
        self.kind, self.seed, self.fail_seed, self.fail_period = kind, seed, fail_seed, fail_period
        elems = batch_interleaved_elems(n, self.count, chunk) if self.count else 0
        self.A = torch.empty(max(elems, 4), dtype=torch.float32, device=self.device)
        self.info = torch.empty(max(self.count, 1), dtype=torch.int32, device=self.device)
        self.nfailed = torch.zeros(1, dtype=torch.int32, device=self.device)
        self._gen = bspotrf_synth_generate

    def regenerate(self, stream=None):
        if self.count:
            self._gen(self.n, self.count, self.chunk, self.A, kind=self.kind, seed=self.seed,
                      b0=self.b0, fail_seed=self.fail_seed, fail_period=self.fail_period,
                      stream=stream)

    def factor(self, stream=None, tune=None, reset=True):
        """Factor this rank's slice (one kernel launch); the failure count is
        accumulated on the device (``reset`` zeroes it first)."""
        from . import batch_spotrf_interleaved_ex
        if reset:
            self.nfailed.zero_()
        if self.count:
            batch_spotrf_interleaved_ex(self.n, self.count, self.chunk, self.A, self.info,
                                        nfailed=self.nfailed, tune=tune, stream=stream)

    def reduce_failures(self, group=None):
        """Enqueue the one collective (SUM of the 4-byte count) without a host
        sync: after it, ``nfailed`` holds the global count on every rank."""
        import torch.distributed as dist
        if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
            dist.all_reduce(self.nfailed, op=dist.ReduceOp.SUM, group=group)

    def global_failures(self, group=None):
        return allreduce_count(self.nfailed, group)


def min_over_ranks(value: int, device=None, group=None) -> int:
    """The MIN over ranks of an integer (e.g. how many buffers fit in HBM), so
    every rank runs the same number of steps and collectives pair up."""
    import torch
    import torch.distributed as dist
    t = torch.tensor([int(value)], dtype=torch.int64, device=device)
    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MIN, group=group)
    return int(t.item())
