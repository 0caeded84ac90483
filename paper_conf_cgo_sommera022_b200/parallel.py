"""Sample-batch sharding across the GPUs of one box.

Samples are independent, so a batch of N samples is split into contiguous
shards, one per rank (rank r gets [floor(rN/P), floor((r+1)N/P))); every rank
holds a full replica of the prepared plan and runs the same kernels on its
shard.  The only collective is the optional gather of the per-sample results
(log-likelihoods or class argmax) with NCCL (`all_gather_into_tensor` over
NVLink); there is no collective on the compute path.
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def shard_range(n: int, rank: int, world: int) -> tuple[int, int]:
    """Contiguous, balanced shard [lo, hi) of n samples for `rank`."""
    if not (0 <= rank < world):
        raise ValueError("rank out of range")
    return (n * rank) // world, (n * (rank + 1)) // world


def shard_sizes(n: int, world: int) -> list[int]:
    return [shard_range(n, r, world)[1] - shard_range(n, r, world)[0] for r in range(world)]


def gather_results(local: torch.Tensor, n_total: int, group=None) -> torch.Tensor:
    """Gather every rank's shard of a per-sample result ([n_r, ...] or [n_r])
    into the full [n_total, ...] tensor on every rank.  Shards may differ by
    one row (floor split): they are padded to the largest shard for the
    fixed-size all_gather and trimmed afterwards."""
    world = dist.get_world_size(group)
    sizes = shard_sizes(n_total, world)
    m = max(sizes)
    rank = dist.get_rank(group)
    if local.shape[0] != sizes[rank]:
        raise ValueError(f"rank {rank}: local shard has {local.shape[0]} rows, "
                         f"expected {sizes[rank]}")
    pad = torch.zeros((m,) + tuple(local.shape[1:]), dtype=local.dtype, device=local.device)
    pad[:local.shape[0]] = local
    full = torch.empty((world * m,) + tuple(local.shape[1:]), dtype=local.dtype,
                       device=local.device)
    dist.all_gather_into_tensor(full, pad, group=group)
    parts = [full[r * m:r * m + sizes[r]] for r in range(world)]
    return torch.cat(parts, dim=0)


def gather_into(full: torch.Tensor, local: torch.Tensor, group=None) -> torch.Tensor:
    """Gather equal shards ([n/P, ...] per rank) into a preallocated
    [n, ...] tensor on every rank with one all_gather_into_tensor (NCCL over
    NVLink on GPUs).  The bench calls this inside the timed step for the
    strong-scaling config (10M samples split evenly over 1/2/4/8 ranks)."""
    world = dist.get_world_size(group)
    if full.shape[0] != local.shape[0] * world or full.shape[1:] != local.shape[1:]:
        raise ValueError(f"gather_into: full {tuple(full.shape)} != {world} x {tuple(local.shape)}")
    dist.all_gather_into_tensor(full, local.contiguous(), group=group)
    return full


def sharded_infer(plan, x_full: torch.Tensor, marginal: bool = False, gather: bool = True,
                  group=None):
    """Evaluate this rank's shard of x_full with `plan` (a Plan on this
    rank's GPU) and optionally gather the results of all ranks.
    Returns (logp, argmax) -- full tensors if gather else this rank's shard."""
    world = dist.get_world_size(group) if dist.is_initialized() else 1
    rank = dist.get_rank(group) if dist.is_initialized() else 0
    lo, hi = shard_range(x_full.shape[0], rank, world)
    out, am = plan.infer(x_full[lo:hi], marginal=marginal)
    if gather and world > 1:
        out = gather_results(out, x_full.shape[0], group)
        if am is not None:
            am = gather_results(am, x_full.shape[0], group)
    return out, am
