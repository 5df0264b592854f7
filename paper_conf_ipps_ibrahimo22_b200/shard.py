"""Data-parallel sharding of the decode path: one process per
GPU, each rank decodes its own sample shard, no data-path collective.  The only
communication is a barrier around the timed region and one MAX all-reduce of
the elapsed seconds (PAPER.md P:58/P:150 use NCCL for the model's gradients,
which is not on this path)."""
from __future__ import annotations


def shard_indices(n_total: int, rank: int, world: int) -> list[int]:
    """Samples {i : i mod world == rank} (a DistributedSampler-style split)."""
    if world < 1 or not 0 <= rank < world:
        raise ValueError("bad rank/world")
    return list(range(rank, n_total, world))


def rank_seed_base(seed: int, rank: int) -> int:
    """Weak scaling: each rank generates a disjoint block of seeds."""
    return seed + 1000 * rank


def max_over_ranks(seconds: float, dist=None, device=None) -> float:
    """Max of a per-rank elapsed time (device-timed), via one all-reduce."""
    if dist is None or not dist.is_initialized() or dist.get_world_size() == 1:
        return float(seconds)
    import torch
    if dist.get_backend() == "gloo":
        device = None  # gloo reduces host tensors
    t = torch.tensor([float(seconds)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def aggregate_throughput(units_per_rank: int, world: int, steps: int, max_seconds: float) -> float:
    """Whole-job throughput: units all ranks processed / max-over-ranks time."""
    return world * units_per_rank * steps / max_seconds
