"""3-stage vs the 4-stage Gustavson/Karlsson baseline (Table 2) with the SAME
tiles: for every shape the cost model's best full 3-stage tiling (m < M, n < N, so no stage
is elided); both algorithms transpose forth and back, L2 cleared (512 MB read) before each
timed call.  Prints effective GB/s and the 3-stage / 4-stage speed-up (paper, K20: ~2.7-3x)."""
import ctypes, json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ppopp_sunggggh14_b200 as ipt

SHAPES = [(7200, 1800), (5100, 2500), (4000, 3200), (3300, 3900), (2500, 5100), (1800, 7200),
          (7200, 18000), (12800, 15000)]
L = ipt.lib()
cost = L.ipt__plan_cost
cost.restype = ctypes.c_double
cost.argtypes = [ctypes.c_int64] * 4 + [ctypes.c_int, ctypes.c_int]
flush = torch.empty(128 << 20, dtype=torch.int32, device="cuda")


def divs(x):
    return [d for d in range(2, x) if x % d == 0]


def timed(fn, reps=6):
    best = None
    for _ in range(reps):
        flush.sum()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); fn(); e1.record(); torch.cuda.synchronize()
        ms = e0.elapsed_time(e1)
        best = ms if best is None else min(best, ms)
    return best


for (M, N) in SHAPES:
    m, n = min(((cost(M, N, a, b, 4, 0), a, b) for a in divs(M) for b in divs(N)))[1:]
    t = torch.randint(0, 1 << 30, (M * N,), dtype=torch.int32, device="cuda")
    ref = t.view(M, N).t().contiguous().view(-1)
    p3, q3 = ipt.plan(M, N, 4, 0, m=m, n=n), ipt.plan(N, M, 4, 0, m=n, n=m)
    st = {"3": 0.0, "4": 0.0}
    ipt.transpose_(t, M, N, plan_=p3); ok3 = torch.equal(t, ref); ipt.transpose_(t, N, M, plan_=q3)
    ipt.transpose_4stage_(t, M, N, m, n); ok4 = torch.equal(t, ref); ipt.transpose_4stage_(t, N, M, n, m)
    t3 = timed(lambda: (ipt.transpose_(t, M, N, plan_=p3), ipt.transpose_(t, N, M, plan_=q3))) / 2
    t4 = timed(lambda: (ipt.transpose_4stage_(t, M, N, m, n), ipt.transpose_4stage_(t, N, M, n, m))) / 2
    g = lambda ms: round(2 * M * N * 4 / (ms / 1e3) / 1e9)
    print(json.dumps({"shape": f"{M}x{N}", "m": m, "n": n, "ok": ok3 and ok4, "3stage_gbs": g(t3),
                      "4stage_gbs": g(t4), "speedup": round(t4 / t3, 2)}), flush=True)
