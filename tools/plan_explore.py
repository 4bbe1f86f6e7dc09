"""Time every divisor-pair plan (m | M, n | N) of a shape whose stage-2 tile is at most
MAXMB, next to the planner's and the autotuned plan, to check the cost model:
    SHAPES='[(16636,19025)]' python tools/plan_explore.py
Timing only (each plan run 3x on the same buffer, the data is permuted, not checked)."""
import ast
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import paper_conf_ppopp_sunggggh14_b200 as ipt


def divisors(x):
    return [d for d in range(1, x + 1) if x % d == 0]


def timed(t, M, N, p, reps=3):
    ipt.transpose_(t, M, N, plan_=p)
    best = 1e9
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        ipt.transpose_(t, M, N, plan_=p)
        e1.record()
        torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1))
    return best


eb = int(os.environ.get("EB", "4"))
maxmb = float(os.environ.get("MAXMB", "80"))
for (M, N) in ast.literal_eval(os.environ["SHAPES"]):
    t = torch.zeros(M * N, dtype=torch.int32 if eb == 4 else torch.int64, device="cuda")
    res = []
    p0 = ipt.plan(M, N, eb, 0)
    pa = ipt.plan_autotune(t, M, N, 8)
    for m in divisors(M):
        for n in divisors(N):
            if m * n * eb > maxmb * 1e6 or (n < N and n * eb < 64) or (m < M and m * eb < 64):
                continue   # tiles beyond on-chip paths; tiny units (host cycle walks of 1e8 units)
            try:
                p = ipt.plan(M, N, eb, 0, m=m, n=n)
            except Exception:
                continue
            ms = timed(t, M, N, p)
            res.append((ms, m, n, p.n_stages, ipt.stage_kernels(p, 1, t)))
    res.sort()
    gb = 2 * M * N * eb / 1e9
    out = {"shape": f"{M}x{N}", "planner": [p0.m, p0.n, round(timed(t, M, N, p0), 4)],
           "autotune": [pa.m, pa.n, round(timed(t, M, N, pa), 4)],
           "best": [(round(ms, 4), m, n, s, round(gb / ms * 1e3), k) for ms, m, n, s, k in res[:8]]}
    print(json.dumps(out), flush=True)
    del t
    torch.cuda.empty_cache()
