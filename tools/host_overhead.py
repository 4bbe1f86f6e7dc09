"""Host-side cost of one ipt.transpose_ call vs its GPU time, for single matrices.

    python tools/host_overhead.py M N [eb]

Prints: host microseconds per call (Python + ctypes + libipt enqueue), GPU time per
transpose back to back (no flush), with a 512 MB read flush before each (cold L2, events
around the call as bench.py's sub-records), and replayed as a captured CUDA graph."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ppopp_sunggggh14_b200 as ipt  # noqa: E402
from inputs import seeded  # noqa: E402

M, N = int(sys.argv[1]), int(sys.argv[2])
eb = int(sys.argv[3]) if len(sys.argv) > 3 else 4
t = torch.empty(M * N, dtype=torch.int32 if eb == 4 else torch.int64, device="cuda")
seeded.fill_device_(t, M, N, eb)
p, q = ipt.plan_autotune(t, M, N, 8), None
ipt.transpose_(t, M, N, plan_=p)
q = ipt.plan_autotune(t, N, M, 8)
ipt.transpose_(t, N, M, plan_=q)
print("plans", p.as_dict()["variant"], ipt.stage_kernels(p), ipt.stage_kernels(q), flush=True)
torch.cuda.synchronize()
ev = lambda: torch.cuda.Event(enable_timing=True)
# host cost per call (GPU kept busy by a long queue)
reps = 200
h0 = time.perf_counter()
for r in range(reps):
    ipt.transpose_(t, M, N, plan_=p) if r % 2 == 0 else ipt.transpose_(t, N, M, plan_=q)
h1 = time.perf_counter()
torch.cuda.synchronize()
print(f"host us/call {1e6 * (h1 - h0) / reps:.1f}")
# GPU back to back
e0, e1 = ev(), ev()
e0.record()
for r in range(20):
    ipt.transpose_(t, M, N, plan_=p) if r % 2 == 0 else ipt.transpose_(t, N, M, plan_=q)
e1.record()
torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / 20
print(f"back-to-back us/transpose {1e3 * ms:.1f}  eff GB/s {2 * M * N * eb / ms / 1e6:.0f}")
# cold L2, events around each call
flush = torch.zeros(128 << 20, dtype=torch.int32, device="cuda")
tot = 0.0
for r in range(10):
    flush.sum()
    a, b = ev(), ev()
    a.record()
    ipt.transpose_(t, M, N, plan_=p) if r % 2 == 0 else ipt.transpose_(t, N, M, plan_=q)
    b.record()
    torch.cuda.synchronize()
    tot += a.elapsed_time(b)
print(f"cold us/transpose {1e3 * tot / 10:.1f}  eff GB/s {2 * M * N * eb * 10 / tot / 1e6:.0f}")
# cold L2 by a large-shared-memory kernel instead (a 256 MB in-place transpose of another
# buffer): no shared-memory carveout change before the timed launch
big = torch.empty(64 << 20, dtype=torch.int32, device="cuda")
bp = ipt.plan(4096, 16384, 4, 0)
ipt.transpose_(big, 4096, 16384, plan_=bp)
ipt.transpose_(big, 16384, 4096)
tot = 0.0
for r in range(10):
    ipt.transpose_(big, 4096, 16384, plan_=bp) if r % 2 == 0 else ipt.transpose_(big, 16384, 4096)
    a, b = ev(), ev()
    a.record()
    ipt.transpose_(t, M, N, plan_=p) if r % 2 == 0 else ipt.transpose_(t, N, M, plan_=q)
    b.record()
    torch.cuda.synchronize()
    tot += a.elapsed_time(b)
print(f"cold (smem-kernel flush) us/transpose {1e3 * tot / 10:.1f}  eff GB/s {2 * M * N * eb * 10 / tot / 1e6:.0f}",
      ipt.stage_kernels(bp))
del big
# graphs
gA, gB = ipt.Graph(t, M, N, p), ipt.Graph(t, N, M, q)
tot = 0.0
for r in range(10):
    flush.sum()
    a, b = ev(), ev()
    a.record()
    (gA if r % 2 == 0 else gB).launch()
    b.record()
    torch.cuda.synchronize()
    tot += a.elapsed_time(b)
print(f"cold graph us/transpose {1e3 * tot / 10:.1f}  eff GB/s {2 * M * N * eb * 10 / tot / 1e6:.0f}")
# stage events
for r in range(2):
    flush.sum()
    evs = [ev() for _ in range(4)]
    ipt.transpose_(t, M, N, plan_=p, events=evs) if r % 2 == 0 else ipt.transpose_(t, N, M, plan_=q, events=evs)
    torch.cuda.synchronize()
    print("stage us", [round(1e3 * evs[i].elapsed_time(evs[i + 1]), 1) for i in range(3)])
