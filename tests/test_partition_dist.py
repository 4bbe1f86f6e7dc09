"""Multi-process (world_size 2, gloo, CPU) tests of the batch partitioner and the
timing reduction used by the multi-GPU bench; the GPU data path has no
collective, so these cover all of the N > 1 host logic."""
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ppopp_sunggggh14_b200.partition import max_over_ranks, shard


def test_shard_arithmetic():
    for count in [0, 1, 7, 512, 513, 1000]:
        for world in [1, 2, 3, 4, 8]:
            parts = [shard(count, world, r) for r in range(world)]
            assert parts[0][0] == 0 and parts[-1][1] == count
            for (a, b), (c, d) in zip(parts, parts[1:]):
                assert b == c                       # contiguous, disjoint
            sizes = [b - a for a, b in parts]
            assert max(sizes) - min(sizes) <= 1     # balanced
    with pytest.raises(ValueError):
        shard(10, 2, 2)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, count, out):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        lo, hi = shard(count, world, rank)
        owned = torch.zeros(count, dtype=torch.int64)
        owned[lo:hi] = 1
        dist.all_reduce(owned)                      # every matrix owned exactly once
        t = max_over_ranks(10.0 * (rank + 1))       # max over ranks
        dist.barrier()
        out[rank] = (int(owned.min()), int(owned.max()), t, hi - lo)
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("count", [512, 7])
def test_two_rank_gloo_partition(count):
    world = 2
    mgr = mp.Manager()
    out = mgr.dict()
    port = _free_port()
    mp.spawn(_worker, args=(world, port, count, out), nprocs=world, join=True)
    for r in range(world):
        mn, mx, t, n = out[r]
        assert mn == 1 and mx == 1
        assert t == 20.0
    assert out[0][3] + out[1][3] == count
