"""Multi-GPU plumbing: one process per GPU, photons sharded by id, one
all-reduce of the integer tallies.

Tasks are independent (every draw is keyed by task id), so sharding needs no
data-path exchange: rank r owns ids [task_offset_of(r), +per_rank).  The only
collective is the reduction of the GRID+COUNTERS workspace regions viewed as
int64 -- two's-complement addition is uint64 addition mod 2^64, so the result
is bit-identical for any rank count and any reduction order.
"""
from __future__ import annotations


def task_offset_of(rank: int, per_rank: int, base: int = 0) -> int:
    """First global task id of `rank` when every rank owns `per_rank` tasks."""
    if rank < 0 or per_rank < 0:
        raise ValueError("rank and per_rank must be >= 0")
    return base + rank * per_rank


def split_even(total: int, world: int, rank: int) -> tuple[int, int]:
    """(offset, count) of `rank`'s contiguous share of `total` tasks (strong scaling)."""
    q, r = divmod(total, world)
    count = q + (1 if rank < r else 0)
    offset = rank * q + min(rank, r)
    return offset, count


def allreduce_tallies(tallies, group=None, stream=None):
    """In-place SUM all-reduce of an int64 tensor view of GRID+COUNTERS.

    `stream`: the CUDA stream the kernels were enqueued on (NCCL runs on
    torch's current stream; it must be ordered after the kernels)."""
    import torch
    import torch.distributed as dist
    if not dist.is_initialized() or dist.get_world_size(group) == 1:
        return tallies
    if tallies.dtype != torch.int64:
        raise TypeError("tallies must be an int64 view")
    if stream is not None:
        with torch.cuda.stream(stream):
            dist.all_reduce(tallies, op=dist.ReduceOp.SUM, group=group)
    else:
        dist.all_reduce(tallies, op=dist.ReduceOp.SUM, group=group)
    return tallies
