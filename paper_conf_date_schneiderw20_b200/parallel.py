"""Multi-GPU slot sharding (each stimulus under an operating point is
an independent simulation problem, so the slot space shards with no exchange
during simulation).  The only collective is the reduction of the per-rank
results: activity SUM and latest-arrival MAX.
"""
from __future__ import annotations


def shard_range(total_slots: int, rank: int, world: int) -> tuple:
    """Contiguous public-slot range [first, first + n) of `rank` (balanced)."""
    if world < 1 or not (0 <= rank < world):
        raise ValueError("bad rank / world")
    first = total_slots * rank // world
    end = total_slots * (rank + 1) // world
    return first, end - first


def shard_pairs(n_pairs: int, rank: int, world: int) -> tuple:
    """Pairs [first, first + n) of `rank` (balanced), simulated at every
    operating point (Context.set_pair_range): each shard keeps whole
    operating-point sweeps of its pairs, the layout the sweep is fastest on."""
    return shard_range(n_pairs, rank, world)


def reduce_results(activity, latest, dst: int = 0, group=None):
    """In-place reduce of rank-local results onto `dst` (torch tensors:
    activity int64 [n_signals][n_vdd] -> SUM, latest float32 [n_vdd] -> MAX)."""
    import torch.distributed as dist
    dist.reduce(activity, dst=dst, op=dist.ReduceOp.SUM, group=group)
    dist.reduce(latest, dst=dst, op=dist.ReduceOp.MAX, group=group)
    return activity, latest
