"""Multi-GPU plumbing for the lookup path.

The lookup batch shards trivially: lookup i depends only on (grid spec, i)
(its random stream is FF(seed, 2i)), so rank r of R processes a contiguous
id range and the grid is replicated per GPU.  The only collective is A9:
one all-reduce (SUM) of the 16-byte verification vector {sum v, count}
over NCCL (NVLink/NVSwitch); the timing reduction (MAX over ranks) is
measurement, not part of the method.

Scaling modes:
  weak   - every rank owns `per_rank` lookups: ids [r*per_rank, (r+1)*per_rank)
  strong - a fixed total L split as [floor(r L / R), floor((r+1) L / R)), or
           (sorted batches, bench.py's default) energy-range shards: every rank
           samples all L lookups and looks up those with b_r <= p < b_{r+1}
           (xs_lookup_batch_shard), so each keeps the full batch's density
"""
from __future__ import annotations

import os


def shard_range(rank: int, world: int, lookups: int, scaling: str = "weak") -> tuple[int, int]:
    """(first_id, count) of this rank's shard."""
    if world < 1 or not 0 <= rank < world:
        raise ValueError("bad rank/world")
    if scaling == "weak":
        return rank * lookups, lookups
    if scaling == "strong":
        a = rank * lookups // world
        b = (rank + 1) * lookups // world
        return a, b - a
    raise ValueError(f"unknown scaling {scaling!r}")


def energy_shard_bounds(rank: int, world: int) -> tuple[float, float]:
    """[lo, hi) of energy shard `rank` of `world` as xs_lookup_batch_shard
    defines it: b_s = s / world in binary64, b_0 = -inf, b_world = +inf."""
    if world < 1 or not 0 <= rank < world:
        raise ValueError("bad rank/world")
    lo = rank / world if rank > 0 else float("-inf")
    hi = (rank + 1) / world if rank < world - 1 else float("inf")
    return lo, hi


def env_rank() -> tuple[int, int, int]:
    """(rank, world, local_rank) from the torchrun environment (1 process if unset)."""
    return (int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1)),
            int(os.environ.get("LOCAL_RANK", 0)))


def combine_vsum(vsum, group=None):
    """A9: in-place all-reduce (SUM) of the {sum v, count} vector (int64
    tensor of 2) across ranks; a no-op on a single process."""
    import torch.distributed as dist
    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(vsum, op=dist.ReduceOp.SUM, group=group)
    return vsum


def max_over_ranks(value: float, device=None, group=None) -> float:
    """Maximum of a per-rank scalar (e.g. elapsed ms) over all ranks."""
    import torch
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1):
        return float(value)
    t = torch.tensor([float(value)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return float(t.item())


def global_hash(vsum_global) -> int:
    """hash = (sum over all ranks of v) mod 999983, applied once after the
    global reduction (R13) — the library's xs_hash_finalize."""
    from .xs import xs_hash_finalize
    return int(xs_hash_finalize(int(vsum_global[0]) & 0xFFFFFFFFFFFFFFFF))
