"""Batch sharding across GPUs.

Inference images are independent and BN is folded with fixed statistics, so
the path shards by contiguous batch slices with no data-path exchange: rank r
of N runs images [r*B, (r+1)*B) through its own plan, and the only collective
is one all_gather of the fp32 logits (NCCL over NVLink on the GPU box, gloo in
the CPU tests).  Weak scaling: B per rank is fixed as N grows.
"""
from __future__ import annotations


def shard_range(rank: int, world: int, per_rank: int):
    """Global image indices [start, stop) of `rank`'s shard."""
    if not 0 <= rank < world or per_rank <= 0:
        raise ValueError("bad shard arguments")
    return rank * per_rank, (rank + 1) * per_rank


def gather_logits(local, world: int, out=None):
    """All-gather the per-rank logits [B, K] into [world * B, K] (rank order).

    Uses all_gather_into_tensor on NCCL (one collective into a preallocated
    buffer) and the list form elsewhere (gloo)."""
    import torch
    import torch.distributed as dist
    if world == 1:
        return local
    if out is None:
        out = torch.empty((world * local.shape[0],) + tuple(local.shape[1:]), dtype=local.dtype,
                          device=local.device)
    if dist.get_backend() == "nccl":
        dist.all_gather_into_tensor(out, local.contiguous())
    else:
        parts = [torch.empty_like(local) for _ in range(world)]
        dist.all_gather(parts, local.contiguous())
        torch.cat(parts, out=out)
    return out
