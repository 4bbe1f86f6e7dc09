"""Multi-process (world_size 2, gloo, CPU) tests of the batch partitioner and of the exact
rank bookkeeping bench.py runs at N > 1: partition.dist_env /
init_ranks / BatchShard (owned block, generator offset, bytes) / barrier / max_over_ranks /
sum_over_ranks / all_ok / aggregate_gbs.  The GPU data path has no collective.  The last
test runs bench.py's own multi-rank path (`--gpus 2` re-launching itself under
torch.distributed.run) far enough to check its rank handling without a GPU."""
import os
import socket
import subprocess
import sys

import numpy as np
import pytest
import torch.multiprocessing as mp

from inputs import seeded
from paper_conf_ppopp_sunggggh14_b200 import partition as part

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_shard_arithmetic():
    for count in [0, 1, 7, 512, 513, 1000]:
        for world in [1, 2, 3, 4, 8]:
            parts = [part.shard(count, world, r) for r in range(world)]
            assert parts[0][0] == 0 and parts[-1][1] == count
            for (a, b), (c, d) in zip(parts, parts[1:]):
                assert b == c                       # contiguous, disjoint
            sizes = [b - a for a, b in parts]
            assert max(sizes) - min(sizes) <= 1     # balanced
    with pytest.raises(ValueError):
        part.shard(10, 2, 2)


def test_batch_shard_bytes_and_aggregate():
    for world in (1, 2, 4, 8):
        shs = [part.BatchShard(512, 4096, 3000, 4, world, r) for r in range(world)]
        assert sum(s.count for s in shs) == 512
        assert sum(s.rank_bytes_per_step() for s in shs) == shs[0].job_bytes_per_step()
        assert shs[0].job_bytes_per_step() == 2 * 4096 * 3000 * 4 * 512
    # 25.17 GB read + written once per step, 20 steps in 10 ms each
    gbs = part.aggregate_gbs(2 * 25_165_824_000, 20, 200.0)
    assert abs(gbs - 2 * 25_165_824_000 * 20 / 0.2 / 1e9) < 1e-6
    with pytest.raises(ValueError):
        part.aggregate_gbs(1, 1, 0.0)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, count, M, N, out):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), WORLD_SIZE=str(world),
                      RANK=str(rank), LOCAL_RANK=str(rank))
    w, r = part.init_ranks("gloo")            # bench.py's call (NCCL on the GPU box)
    try:
        assert (w, r) == (world, rank) and part.dist_env() == (world, rank, rank)
        sh = part.BatchShard(count, M, N, 4, w, r)
        # the rank's block, filled from the GLOBAL matrix index (bench: fill_device_ t0=sh.lo)
        mine = seeded.values_np(np.arange(sh.lo * M * N, sh.hi * M * N, dtype=np.uint64), 4)
        part.barrier()
        t = part.max_over_ranks(10.0 * (rank + 1))           # slowest rank's time
        nb = part.sum_over_ranks(sh.rank_bytes_per_step())   # bytes of all ranks
        ok_all = part.all_ok(True)
        ok_one = part.all_ok(rank == 0)                        # one rank fails -> all fail
        gbs = part.aggregate_gbs(sh.job_bytes_per_step(), 3, t)
        out[rank] = (sh.lo, sh.hi, mine.tobytes(), t, nb, ok_all, ok_one, gbs)
    finally:
        import torch.distributed as dist

        dist.destroy_process_group()


@pytest.mark.parametrize("count", [7, 2])
def test_two_rank_gloo_bench_bookkeeping(count):
    world, M, N = 2, 6, 5
    out = mp.Manager().dict()
    mp.spawn(_worker, args=(world, _free_port(), count, M, N, out), nprocs=world, join=True)
    los = sorted((out[r][0], out[r][1]) for r in range(world))
    assert los[0][0] == 0 and los[-1][1] == count and los[0][1] == los[1][0]
    # the union of the ranks' blocks is the G = 1 batch, bit for bit
    union = b"".join(out[r][2] for r in sorted(range(world), key=lambda r: out[r][0]))
    assert union == seeded.batch_np(count, M, N, 4).tobytes()
    job = 2 * M * N * 4 * count
    for r in range(world):
        _, _, _, t, nb, ok_all, ok_one, gbs = out[r]
        assert t == 20.0 and nb == job and ok_all and not ok_one
        assert abs(gbs - job * 3 / 0.020 / 1e9) < 1e-9


def test_bench_gpus_flag_spawns_ranks(tmp_path):
    """`bench.py --gpus 2` without WORLD_SIZE re-launches itself with 2 ranks; each rank
    checks WORLD_SIZE == --gpus (here under the reference arm, which needs no GPU: rank 0
    prints the line, the other rank exits 0)."""
    env = dict(os.environ)
    env.pop("WORLD_SIZE", None)
    record = os.path.join(str(tmp_path), "runs.jsonl")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--impl",
                        "reference", "--steps", "1", "--warmup", "0", "--record", record],
                       capture_output=True, text=True, timeout=600, env=env, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [x for x in r.stdout.splitlines() if x.startswith("{")]
    assert len(lines) == 1 and '"n_gpus": 2' in lines[0] and '"impl": "reference"' in lines[0]
    # --record: the same line (rank 0 only) appended to a JSONL run record, stamped
    import json
    recs = [json.loads(x) for x in open(record)]
    assert len(recs) == 1 and recs[0]["value"] == json.loads(lines[0])["value"]
    assert recs[0]["recorded_utc"].endswith("Z") and "--record" in recs[0]["argv"]
    # a mismatched rank count is refused
    env.update(WORLD_SIZE="1", RANK="0", LOCAL_RANK="0")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2"],
                       capture_output=True, text=True, timeout=120, env=env, cwd=ROOT)
    assert r.returncode == 2


def test_workloads_lists():
    """The benched shape lists (inputs/workloads.py): the full SURVEY C2 classes, seeded
    random pairs reproducible, in range, no duplicates; C5 = 512 x 4096 x 3000."""
    from inputs import workloads as W

    assert W.C5_SHAPE == (4096, 3000) and W.C5_COUNT == 512
    assert W.sweep_random_pairs() == W.SWEEP_RANDOM and len(W.SWEEP_RANDOM) == 16
    assert all(1000 <= a <= 20000 and 1000 <= b <= 20000 for a, b in W.SWEEP_RANDOM)
    for s in W.TABLE2 + W.SWEEP_POW2 + W.SWEEP_FEW_FACTORS + W.SWEEP_LARGE + W.SWEEP_RANDOM:
        assert s in W.SWEEP_ALL
    assert len(set(W.SWEEP_ALL)) == len(W.SWEEP_ALL)
    assert (9797, 13081) in W.SWEEP_ALL and (10007, 19997) in W.PRIMES


def test_bench_verify_composed_transposes():
    """bench._verify undoes a sequence of transposes (the fixed-orientation headline: the
    M x N result re-read as the next M x N input, plus N x M steps): checked against
    numpy transposes of the generator values on CPU tensors, and a wrong sequence fails."""
    import importlib.util
    import torch

    spec = importlib.util.spec_from_file_location("bench_mod", os.path.join(ROOT, "bench.py"))
    bench = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(bench)
    for eb in (4, 8):
        count, M, N, t0 = 3, 6, 10, 5
        x = seeded.values_np(np.arange(t0 * M * N, (t0 + count) * M * N, dtype=np.uint64), eb)
        x = x.reshape(count, M * N)
        seq = [(M, N), (M, N), (N, M), (M, N), (M, N)]
        for (a, b) in seq:
            x = np.ascontiguousarray(x.reshape(count, a, b).transpose(0, 2, 1)).reshape(count, M * N)
        dt = torch.int32 if eb == 4 else torch.int64
        t = torch.from_numpy(x.reshape(-1).view(np.int32 if eb == 4 else np.int64).copy()).to(dt)
        assert bench._verify(t, M, N, eb, False, t0=t0, count=count, nsamp=256, seq=seq)
        assert not bench._verify(t, M, N, eb, False, t0=t0, count=count, nsamp=256, seq=seq[:-1])
