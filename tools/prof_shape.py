"""Transpose one workload matrix (or batch) a few times, for ncu captures.

    python tools/prof_shape.py M N [--eb 4] [--m m --n n] [--count c] [--reps r] [--autotune k]

Both orientations are run each repetition (M x N -> N x M -> M x N), with the planner's
plans, forced tiles (--m/--n), or measured plans (--autotune k, as bench.py).  Prints the
plans and the kernel each stage launches (ipt__stage_kernel)."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ppopp_sunggggh14_b200 as ipt  # noqa: E402
from inputs import seeded  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("M", type=int)
ap.add_argument("N", type=int)
ap.add_argument("--eb", type=int, default=4)
ap.add_argument("--m", type=int, default=0)
ap.add_argument("--n", type=int, default=0)
ap.add_argument("--count", type=int, default=1)
ap.add_argument("--reps", type=int, default=2)
ap.add_argument("--autotune", type=int, default=0)
a = ap.parse_args()
M, N, eb, cnt = a.M, a.N, a.eb, a.count
t = torch.empty(cnt * M * N, dtype=torch.int32 if eb == 4 else torch.int64, device="cuda")
seeded.fill_device_(t, M, N, eb, count=cnt)
if a.m:
    p1, p2 = ipt.plan(M, N, eb, 0, m=a.m, n=a.n), ipt.plan(N, M, eb, 0, m=a.n, n=a.m)
elif a.autotune > 1:
    tune = (lambda x, y: ipt.plan_autotune_batched(t, cnt, x, y, a.autotune)) if cnt > 1 else \
           (lambda x, y: ipt.plan_autotune(t, x, y, a.autotune))
    p1 = tune(M, N)
    ipt.transpose_batched_(t, cnt, M, N, plan_=p1)
    p2 = tune(N, M)
    ipt.transpose_batched_(t, cnt, N, M, plan_=p2)
else:
    p1, p2 = ipt.plan(M, N, eb, 0), ipt.plan(N, M, eb, 0)
for p in (p1, p2):
    print(p.as_dict(), ipt.stage_kernels(p, cnt, t), flush=True)
torch.cuda.synchronize()
for _ in range(a.reps):
    ipt.transpose_batched_(t, cnt, M, N, plan_=p1)
    ipt.transpose_batched_(t, cnt, N, M, plan_=p2)
torch.cuda.synchronize()
print("done", flush=True)
