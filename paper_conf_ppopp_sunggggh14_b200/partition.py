"""Batch partitioner.

A single matrix does not shard: stage 1 (100!) is one global permutation whose cycles span
the whole array, so splitting it would need an out-of-place exchange buffer.  A
batch of independent matrices does: rank r of G owns the contiguous block of matrices
[floor(r*count/G), floor((r+1)*count/G)) and transposes it with one ipt_transpose_batched
call on its own GPU -- no collective on the data path.  Matrices are generated from their
global index, so the union over ranks is independent of G.

`torch.distributed` is used only for a start/stop barrier and a max-reduce of timings.
"""
from __future__ import annotations


def shard(count: int, world: int, rank: int) -> tuple[int, int]:
    """[lo, hi) of the matrices owned by `rank` (balanced to within one matrix)."""
    if world < 1 or not 0 <= rank < world or count < 0:
        raise ValueError("bad shard arguments")
    return count * rank // world, count * (rank + 1) // world


def run_sharded_batch(buf, count_total: int, M: int, N: int, rank: int, world: int,
                      elem_bytes: int | None = None, stream=None):
    """Transpose this rank's shard (already resident in `buf`, contiguous) in place."""
    from . import transpose_batched_

    lo, hi = shard(count_total, world, rank)
    if hi > lo:
        transpose_batched_(buf, hi - lo, M, N, stream=stream, elem_bytes=elem_bytes)
    return lo, hi


def max_over_ranks(value: float, device=None) -> float:
    """Max of a per-rank timing over the process group (identity when not initialised)."""
    import torch
    import torch.distributed as dist

    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        return float(value)
    t = torch.tensor([float(value)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())
