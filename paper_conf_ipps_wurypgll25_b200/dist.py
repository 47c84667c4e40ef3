"""Multi-GPU host logic (no method arithmetic): one process per GPU, the batch
sharded by sequence, no collective on the hot path.

* ``shard(rank, world, batch_per_rank)``: weak scaling -- rank r owns global
  sequences [r*B, (r+1)*B); the seeded generator is coordinate based, so a
  rank's inputs are exactly the global batch's rows.
* ``max_over_ranks``: timing reduce (the bench reports the slowest rank).
* ``gather_rows``: verification-only all_gather of sampled outputs (C1).
"""
from __future__ import annotations

import os

import torch
import torch.distributed as dist


def env_rank_world():
    return int(os.environ.get("RANK", "0")), int(os.environ.get("WORLD_SIZE", "1")), \
        int(os.environ.get("LOCAL_RANK", "0"))


def shard(rank: int, world: int, batch_per_rank: int):
    """(global batch offset, global batch) under weak scaling."""
    if not (0 <= rank < world) or batch_per_rank <= 0:
        raise ValueError("bad shard")
    return rank * batch_per_rank, world * batch_per_rank


def max_over_ranks(x: float, device=None) -> float:
    if not dist.is_available() or not dist.is_initialized() or dist.get_world_size() == 1:
        return float(x)
    t = torch.tensor([float(x)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def gather_rows(rows: torch.Tensor) -> torch.Tensor:
    """Concatenate every rank's rows (dim 0) on every rank (verification only)."""
    if not dist.is_available() or not dist.is_initialized() or dist.get_world_size() == 1:
        return rows
    out = [torch.empty_like(rows) for _ in range(dist.get_world_size())]
    dist.all_gather(out, rows.contiguous())
    return torch.cat(out, 0)
