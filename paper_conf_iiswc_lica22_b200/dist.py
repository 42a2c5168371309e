"""Multi-GPU plumbing for the scaling bench (one process per GPU, torch.distributed).

The method has no exchange step: every (batch, head) unit is independent (heads run in
parallel; each row's softmax is row-local). So ranks shard the batch and run the forward on
their shard with no data-path collective. Only the scaling bench gathers O (NCCL all_gather over
NVLink on B200; gloo in the CPU tests) to assemble the global result.
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def shard_range(global_batch: int, world: int, rank: int) -> tuple[int, int]:
    """Contiguous batch slice [lo, hi) of `rank` (strong scaling); the first ranks take the remainder."""
    if global_batch < 0 or world <= 0 or not 0 <= rank < world:
        raise ValueError("bad shard arguments")
    base, rem = divmod(global_batch, world)
    lo = rank * base + min(rank, rem)
    return lo, lo + base + (1 if rank < rem else 0)


def rank_seed(seed: int, rank: int) -> int:
    """Input seed of a rank in the weak-scaling bench (each rank draws its own batch)."""
    return seed + 1000 * rank


def gather_outputs(o: torch.Tensor, group=None) -> torch.Tensor:
    """all_gather of equally-shaped per-rank outputs along a new leading rank dimension."""
    world = dist.get_world_size(group)
    o = o.contiguous()
    out = torch.empty((world * o.shape[0],) + tuple(o.shape[1:]), dtype=o.dtype, device=o.device)
    dist.all_gather_into_tensor(out, o, group=group)   # concatenated along dim 0 (gloo and NCCL)
    return out.view((world,) + tuple(o.shape))


def gather_batches(o: torch.Tensor, global_batch: int, group=None) -> torch.Tensor:
    """Reassemble a strong-scaling result: ranks hold shard_range slices of the batch dimension
    (possibly uneven); returns the [global_batch, ...] tensor on every rank."""
    world = dist.get_world_size(group)
    rest = tuple(o.shape[1:])
    maxb = -(-global_batch // world)
    pad = torch.zeros((maxb,) + rest, dtype=o.dtype, device=o.device)
    pad[: o.shape[0]] = o
    allp = gather_outputs(pad, group)
    parts = []
    for r in range(world):
        lo, hi = shard_range(global_batch, world, r)
        parts.append(allp[r, : hi - lo])
    return torch.cat(parts, dim=0)
