"""Data-parallel sharding by image: weak scaling, no data-path collective.

Each rank processes its own batch of `per_rank` images with global indices
[rank*per_rank, (rank+1)*per_rank) and regenerates them from the per-image seeds, so a
sharded run sees exactly the images a single process would.  The only collectives are the
barrier around the timed region, the max-over-ranks reduction of the measured times, and --
outside the timed region -- an all_gather of per-image fp64 checksums of y (the invariance
check: an image's y does not depend on which rank computed it) and the gather of every rank's
y into rank 0, timed on its own.
"""
from __future__ import annotations

import torch


def shard_images(rank: int, world: int, per_rank: int):
    if not (0 <= rank < world) or per_rank <= 0:
        raise ValueError("bad shard")
    return list(range(rank * per_rank, (rank + 1) * per_rank))


def shard_strong(rank: int, world: int, global_batch: int):
    """Strong scaling (config 5: a fixed global batch): contiguous image blocks, the first
    global_batch % world ranks take one extra image."""
    if not (0 <= rank < world) or global_batch < world:
        raise ValueError("bad shard")
    base, extra = divmod(global_batch, world)
    start = rank * base + min(rank, extra)
    return list(range(start, start + base + (1 if rank < extra else 0)))


def max_over_ranks(dist, values, device):
    """Element-wise max of a list of floats over all ranks (the job's wall time is the
    slowest rank's).  dist=None means single process."""
    t = torch.tensor(values, dtype=torch.float64, device=device)
    if dist is not None:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return [float(v) for v in t.cpu()]


def image_checksums(y: torch.Tensor) -> torch.Tensor:
    """Per-image fp64 checksum of y [n, ...]: (sum, sum of squares, sum of index-weighted values)
    per image, so a swapped or shifted image changes it."""
    f = y.reshape(y.shape[0], -1).to(torch.float64)
    idx = torch.arange(f.shape[1], dtype=torch.float64, device=f.device) / max(1, f.shape[1])
    return torch.stack([f.sum(1), (f * f).sum(1), (f * idx).sum(1)], dim=1)


def gather_checksums(dist, local: torch.Tensor) -> torch.Tensor:
    """All-gather the [n_local, 3] checksums of every rank -> [world * n_local, 3] in image order."""
    if dist is None:
        return local
    parts = [torch.empty_like(local) for _ in range(dist.get_world_size())]
    dist.all_gather(parts, local.contiguous())
    return torch.cat(parts)


def gather_outputs(dist, y: torch.Tensor):
    """Every rank's y [n_local, ...] into one [world * n_local, ...] tensor (all ranks receive it;
    rank 0 is the consumer).  Returns y itself in a single process."""
    if dist is None:
        return y
    out = torch.empty((dist.get_world_size() * y.shape[0],) + tuple(y.shape[1:]), dtype=y.dtype, device=y.device)
    dist.all_gather_into_tensor(out, y.contiguous())
    return out
