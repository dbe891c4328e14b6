"""Multi-GPU sharding of the RHS batch: one contiguous slice
per rank, no collective on the data path.  torch.distributed is used only for
barriers and the max-over-ranks time reduction (NCCL on GPUs, gloo in tests).
"""
from __future__ import annotations


def shard_bounds(rank: int, world: int, total: int) -> tuple[int, int]:
    """[first, last) of rank's contiguous slice of `total` RHS; the remainder
    goes to the last ranks (sizes differ by at most one)."""
    if not (0 <= rank < world) or total < 0:
        raise ValueError((rank, world, total))
    base, rem = divmod(total, world)
    first = rank * base + max(0, rank - (world - rem))
    size = base + (1 if rank >= world - rem else 0)
    return first, first + size


def weak_bounds(rank: int, per_rank: int) -> tuple[int, int]:
    """Weak scaling: rank owns [rank*per_rank, (rank+1)*per_rank) of the
    global RHS index space (the index drives the RNG, so data do not depend
    on the number of ranks)."""
    return rank * per_rank, (rank + 1) * per_rank


def max_over_ranks(value: float, device=None) -> float:
    """All-reduce(MAX) of one float over the default process group (identity
    when torch.distributed is not initialised)."""
    import torch
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()):
        return float(value)
    t = torch.tensor([float(value)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())
