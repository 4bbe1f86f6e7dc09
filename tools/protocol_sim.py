"""Interleaving simulator of the PTTWAC claim protocol used by cycle_global.cu (SURVEY.md
T3, 8(c) C7).  Host-side model, no GPU: walkers are coroutines that yield at every shared
memory access (data read, data write, flag check, atomic claim); a seeded random scheduler
interleaves them under sequential consistency (the kernel's fences -- acquire claim +
__syncwarp on the writer side, fence.acq_rel.gpu between the start walker's data read and
its flag re-check -- are what make SC the right model).

Protocols:
  "P1"        the kernel's protocol: start x: read A[x], re-check bit x (abort if set);
              chain step: d = next(cur); read backup A[d]; claim bit d (atomic OR); lost
              -> stop; won -> write carried data into d, carry backup.  Closing the cycle
              at the walker's own start still claims it, but skips the backup read.
  "P0"        no start re-check (must fail).
  "HOME_SKIP" the cycle close at the walker's own start writes WITHOUT claiming (the bug
              found on B200 on square matrices: another carrier of A[prev(x)] may claim x
              and read it after the unclaimed write) -- must fail.
"""
from __future__ import annotations

import random


def perm_transpose(A: int, B: int):
    """Eq. (1) on an A x B array: k -> (k mod B) * A + k // B."""
    return [(k % B) * A + k // B for k in range(A * B)]


def walker(x, nxt, mem, flag, protocol, stats):
    data = mem[x]
    stats["reads"] += 1
    yield
    if protocol != "P0":
        if flag[x]:
            return
        yield
    cur = x
    while True:
        d = nxt[cur]
        if d == cur:
            return
        home = d == x
        if protocol == "HOME_SKIP" and home:
            mem[d] = data
            stats["writes"] += 1
            return
        if not home:
            backup = mem[d]
            stats["reads"] += 1
            yield
        old = flag[d]
        flag[d] = 1
        yield
        if old:
            return
        mem[d] = data
        stats["writes"] += 1
        yield
        if home:
            return
        data = backup
        cur = d


def simulate(A: int, B: int, protocol: str, workers: int, seed: int):
    """Returns (correct, stats).  Start positions are handed out in increasing order to
    `workers` concurrent walkers (adjacent work-items start at adjacent elements);
    the flag word pre-check skips positions already claimed."""
    rnd = random.Random(seed)
    nxt = perm_transpose(A, B)
    n = A * B
    mem = list(range(n))
    flag = [0] * n
    stats = {"reads": 0, "writes": 0}
    next_start = 0
    active = []

    def spawn():
        nonlocal next_start
        while next_start < n:
            x = next_start
            next_start += 1
            if flag[x] or nxt[x] == x:      # pre-check from the cached flag word
                continue
            return walker(x, nxt, mem, flag, protocol, stats)
        return None

    for _ in range(workers):
        w = spawn()
        if w is not None:
            active.append(w)
    while active:
        i = rnd.randrange(len(active))
        try:
            next(active[i])
        except StopIteration:
            w = spawn()
            if w is None:
                active.pop(i)
            else:
                active[i] = w
    expect = [0] * n
    for k in range(n):
        expect[nxt[k]] = k
    return mem == expect, stats
