"""Batch partitioner and the multi-rank bookkeeping that
bench.py runs at N > 1.

A single matrix does not shard: stage 1 (100!) is one global permutation whose cycles span
the whole array, so splitting it would need an out-of-place exchange buffer.  A
batch of independent matrices does (the instances are independent): rank r of G
owns the contiguous block of matrices [floor(r*count/G), floor((r+1)*count/G)) and
transposes it with one ipt_transpose_batched call per step on its own GPU -- no
collective on the data path.  Matrices are generated from their global index t, so the
union over ranks is independent of G.

`torch.distributed` is used only for a start/stop barrier and a max-reduce of the timed
region (device time, max over ranks).  Every function here is exercised by
tests/test_partition_dist.py under world_size-2 gloo, exactly as bench.py calls it.
"""
from __future__ import annotations

from dataclasses import dataclass


def shard(count: int, world: int, rank: int) -> tuple[int, int]:
    """[lo, hi) of the matrices owned by `rank` (balanced to within one matrix)."""
    if world < 1 or not 0 <= rank < world or count < 0:
        raise ValueError("bad shard arguments")
    return count * rank // world, count * (rank + 1) // world


@dataclass(frozen=True)
class BatchShard:
    """This rank's share of a batch of `total` M x N matrices of `elem_bytes` bytes."""
    total: int
    M: int
    N: int
    elem_bytes: int
    world: int
    rank: int

    @property
    def lo(self) -> int:          # global index of the first owned matrix (generator t0)
        return shard(self.total, self.world, self.rank)[0]

    @property
    def hi(self) -> int:
        return shard(self.total, self.world, self.rank)[1]

    @property
    def count(self) -> int:       # matrices owned by this rank
        return self.hi - self.lo

    @property
    def matrix_bytes(self) -> int:
        return self.M * self.N * self.elem_bytes

    def rank_bytes_per_step(self) -> int:
        """Algorithmic bytes of this rank's step (read + write of every owned element)."""
        return 2 * self.matrix_bytes * self.count

    def job_bytes_per_step(self) -> int:
        """Whole-job bytes per step (all ranks): the metric's numerator."""
        return 2 * self.matrix_bytes * self.total


def aggregate_gbs(job_bytes_per_step: int, steps: int, max_elapsed_ms: float) -> float:
    """Whole-job effective GB/s: every rank's bytes over the slowest rank's time."""
    if max_elapsed_ms <= 0:
        raise ValueError("elapsed time must be positive")
    return job_bytes_per_step * steps / (max_elapsed_ms / 1e3) / 1e9


def dist_env() -> tuple[int, int, int]:
    """(world, rank, local_rank) from the torchrun environment (1, 0, 0 when absent)."""
    import os

    return (int(os.environ.get("WORLD_SIZE", "1")), int(os.environ.get("RANK", "0")),
            int(os.environ.get("LOCAL_RANK", "0")))


def init_ranks(backend: str, device=None) -> tuple[int, int]:
    """Initialise the process group when WORLD_SIZE > 1 (NCCL binds `device`); returns
    (world, rank) and logs them so a run's rank count can be checked."""
    import sys

    import torch.distributed as dist

    world, rank, _ = dist_env()
    if world > 1 and not dist.is_initialized():
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=device)
        else:
            dist.init_process_group(backend)
        world, rank = dist.get_world_size(), dist.get_rank()
        print(f"[partition] rank {rank}/{world}: process group up (backend {backend}, "
              f"device {device})", file=sys.stderr, flush=True)
    return world, rank


def barrier():
    import torch.distributed as dist

    if dist.is_available() and dist.is_initialized() and dist.get_world_size() > 1:
        dist.barrier()


def max_over_ranks(value: float, device=None) -> float:
    """Max of a per-rank timing over the process group (identity when not initialised)."""
    import torch
    import torch.distributed as dist

    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        return float(value)
    t = torch.tensor([float(value)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def sum_over_ranks(value: float, device=None) -> float:
    """Sum over the process group (identity when not initialised)."""
    import torch
    import torch.distributed as dist

    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        return float(value)
    t = torch.tensor([float(value)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.SUM)
    return float(t.item())


def all_ok(ok: bool, device=None) -> bool:
    """True iff every rank's verification passed."""
    return max_over_ranks(0.0 if ok else 1.0, device) == 0.0
