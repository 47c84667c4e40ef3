"""Multi-GPU host logic (no method arithmetic): one process per GPU, the batch
sharded by sequence, no collective on the hot path.

The path partitions by sequence: every (sequence, kv head) pair's append and
attention touch only that sequence's cache rows, so rank r of N simply owns a
contiguous range of global batch rows of every layer (cache, q, k_new, v_new,
out).  Two modes:

* ``strong``: the config's global batch B is split -- rank r owns rows
  [r*B//N, (r+1)*B//N) (BASELINE.json north star: "the batch is split across
  1, 2, 4 and 8 GPUs"; c5: batch 128 sharded over 8).
* ``weak``: every rank owns a full config-sized batch B at global offset r*B
  (the paper's own multi-GPU methodology); global batch N*B.

The seeded generator is coordinate based, so a rank's inputs are exactly the
global batch's rows whatever N is.  NCCL is used only for the C1 verification
gather (``gather_rows``) and the C2 timing reduce (``max_over_ranks``).
"""
from __future__ import annotations

import os
from dataclasses import dataclass

import torch
import torch.distributed as dist

MODES = ("strong", "weak")


def env_rank_world():
    return int(os.environ.get("RANK", "0")), int(os.environ.get("WORLD_SIZE", "1")), \
        int(os.environ.get("LOCAL_RANK", "0"))


@dataclass(frozen=True)
class Shard:
    b_off: int          # first global sequence of this rank
    batch: int          # sequences on this rank
    global_batch: int   # sequences over all ranks


def shard(rank: int, world: int, batch: int, mode: str = "strong") -> Shard:
    """This rank's rows of the batch.  strong: `batch` is the GLOBAL batch, split in
    contiguous near-equal ranges (every rank gets >= 1 row); weak: `batch` is the
    per-rank batch."""
    if not (0 <= rank < world) or batch <= 0 or mode not in MODES:
        raise ValueError(f"bad shard: rank {rank} world {world} batch {batch} mode {mode}")
    if mode == "weak":
        return Shard(rank * batch, batch, world * batch)
    if world > batch:
        raise ValueError(f"strong scaling needs batch >= world ({batch} < {world})")
    b0, b1 = rank * batch // world, (rank + 1) * batch // world
    return Shard(b0, b1 - b0, batch)


def max_over_ranks(x: float, device=None) -> float:
    """C2: the slowest rank's value on every rank (bench timing reduce)."""
    if not dist.is_available() or not dist.is_initialized() or dist.get_world_size() == 1:
        return float(x)
    if dist.get_backend() == "gloo":
        device = "cpu"
    t = torch.tensor([float(x)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def gather_rows(rows: torch.Tensor) -> torch.Tensor:
    """C1: concatenate every rank's rows (dim 0, equal shapes on every rank) on
    every rank -- verification only, outside any timed region."""
    if not dist.is_available() or not dist.is_initialized() or dist.get_world_size() == 1:
        return rows
    dev = rows.device
    if dist.get_backend() == "gloo":          # (gloo: host tensors)
        rows = rows.cpu()
    rows = rows.contiguous()
    out = torch.empty((dist.get_world_size() * rows.shape[0], *rows.shape[1:]), dtype=rows.dtype,
                      device=rows.device)
    dist.all_gather_into_tensor(out, rows)
    return out.to(dev)


def sample_pairs(sh: Shard, kv_heads: int, n: int, salt: int = 0):
    """n (local b, kv head) pairs of this rank for the C1 verification: the first
    and last pair of the shard plus seeded picks (same count on every rank, so the
    gathered tensors line up)."""
    import numpy as np
    rng = np.random.default_rng(1009 * sh.b_off + 7919 * salt + sh.batch)
    out = [(0, 0), (sh.batch - 1, kv_heads - 1)]
    while len(out) < n:
        out.append((int(rng.integers(sh.batch)), int(rng.integers(kv_heads))))
    return out[:n]
