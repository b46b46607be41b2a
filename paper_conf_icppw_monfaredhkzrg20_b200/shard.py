"""Instance-range sharding across GPUs (one process per GPU) and the two
collectives the path uses (sec. 5.4: seeds partitioned
equally across GPUs, output identical to a single GPU's).

No keystream ever crosses NVLink: each rank generates its own instance range.
The only exchange is the uint64 CHECKSUM sum and the max step time.
"""
from __future__ import annotations

MASK64 = (1 << 64) - 1


def weak_range(rank: int, n_per_rank: int) -> tuple[int, int]:
    """Weak scaling: rank r owns global instances [r*n, (r+1)*n)."""
    if n_per_rank % 32:
        raise ValueError("instances per rank must be a multiple of 32")
    return rank * n_per_rank, n_per_rank


def strong_range(rank: int, world: int, n_total: int) -> tuple[int, int]:
    """Strong scaling: a contiguous, 32-aligned partition of n_total instances
    (the last rank takes the remainder)."""
    groups = (n_total + 31) // 32
    per = groups // world
    extra = groups % world
    g0 = rank * per + min(rank, extra)
    g1 = g0 + per + (1 if rank < extra else 0)
    first = g0 * 32
    last = min(g1 * 32, n_total)
    return first, max(0, last - first)


def to_int64(u: int) -> int:
    """uint64 -> the int64 with the same bits (NCCL/gloo sum is then mod 2^64)."""
    u &= MASK64
    return u - (1 << 64) if u >= (1 << 63) else u


def allreduce_checksum(value_u64: int, device=None, group=None) -> int:
    """Sum per-rank CHECKSUM values mod 2^64 across the process group."""
    import torch
    import torch.distributed as dist
    t = torch.tensor([to_int64(value_u64)], dtype=torch.int64, device=device)
    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
    return int(t.item()) & MASK64


def allreduce_max(x: float, device=None, group=None) -> float:
    import torch
    import torch.distributed as dist
    t = torch.tensor([float(x)], dtype=torch.float64, device=device)
    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return float(t.item())
