"""Data-parallel sharding by image: weak scaling, no data-path collective.

Each rank processes its own batch of `per_rank` images with global indices
[rank*per_rank, (rank+1)*per_rank) and regenerates them from the per-image seeds, so a
sharded run sees exactly the images a single process would.  The only collectives are the
barrier around the timed region and the max-over-ranks reduction of the measured times.
"""
from __future__ import annotations

import torch


def shard_images(rank: int, world: int, per_rank: int):
    if not (0 <= rank < world) or per_rank <= 0:
        raise ValueError("bad shard")
    return list(range(rank * per_rank, (rank + 1) * per_rank))


def max_over_ranks(dist, values, device):
    """Element-wise max of a list of floats over all ranks (the job's wall time is the
    slowest rank's).  dist=None means single process."""
    t = torch.tensor(values, dtype=torch.float64, device=device)
    if dist is not None:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return [float(v) for v in t.cpu()]
