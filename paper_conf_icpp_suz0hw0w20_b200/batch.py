"""Multi-GPU host logic: independent systems sharded over ranks.

A single solve does not shard (its dependency DAG crosses every row partition), so the
multi-GPU path only distributes INDEPENDENT systems: system s -> rank s mod world, one
stream per device, no data-path collective.  torch.distributed (NCCL on GPUs, gloo in the
CPU tests) is used only for the barrier and the max-over-ranks of the timed region.
"""
from __future__ import annotations


def shard(n_systems: int, rank: int, world: int) -> list[int]:
    """Systems owned by `rank`: s with s % world == rank (round-robin, deterministic)."""
    if world < 1 or not 0 <= rank < world:
        raise ValueError("bad rank/world")
    return [s for s in range(n_systems) if s % world == rank]


def replica_seed(base_seed: int, rank: int) -> int:
    """Weak scaling: every rank solves its own system of the same shape, seed base + rank."""
    return base_seed + rank


def max_over_ranks(value: float, dist=None, device=None) -> float:
    """The timed region's length is the max over ranks (never a wall clock)."""
    if dist is None or not dist.is_initialized() or dist.get_world_size() == 1:
        return float(value)
    import torch
    t = torch.tensor([float(value)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def sum_over_ranks(value: float, dist=None, device=None) -> float:
    if dist is None or not dist.is_initialized() or dist.get_world_size() == 1:
        return float(value)
    import torch
    t = torch.tensor([float(value)], dtype=torch.float64, device=device)
    dist.all_reduce(t)
    return float(t.item())
