"""World-size-2 gloo tests of the sharded (batch-split, collective-free) host logic."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ipps_wurypgll25_b200 import dist as D
from paper_conf_ipps_wurypgll25_b200 import inputs as I


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank),
                      WORLD_SIZE=str(world))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        B = 3
        b_off, gB = D.shard(rank, world, B)
        # a rank's slice of the seeded inputs == the same rows of the global batch
        kv = I.gen_f16(I.seed_for_config(4), I.STREAM_K, 5, b_off, B, 0, 2, 100, 4, 128)
        allk = D.gather_rows(torch.from_numpy(kv.astype(np.float32))).numpy().astype(np.float16)
        ref = I.gen_f16(I.seed_for_config(4), I.STREAM_K, 5, 0, gB, 0, 2, 100, 4, 128)
        ok_gen = np.array_equal(allk, ref)
        # timing reduce returns the slowest rank's time on every rank
        t = D.max_over_ranks(1.5 + rank)
        q.put((rank, ok_gen, t, gB))
    finally:
        dist.destroy_process_group()


def test_two_rank_sharding_and_timing_reduce():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted(q.get(timeout=120) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    assert all(r[1] for r in res)
    assert all(r[2] == 2.5 for r in res)
    assert all(r[3] == 6 for r in res)


def test_shard_bounds():
    assert D.shard(0, 1, 32) == (0, 32)
    assert D.shard(7, 8, 16) == (112, 128)
    with pytest.raises(ValueError):
        D.shard(2, 2, 4)
    assert D.max_over_ranks(3.0) == 3.0
