"""Time forced plans: PLANS = list of (M, N, m, n) (f32 unless EB set); L2 flushed before
every rep; prints effective GB/s and per-stage GB/s (events between stages)."""
import ast, json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ppopp_sunggggh14_b200 as ipt

EB = int(os.environ.get("EB", "4"))
dt = {4: torch.int32, 8: torch.int64}[EB]
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
res = []
for (M, N, m, n) in ast.literal_eval(os.environ["PLANS"]):
    p = ipt.plan(M, N, EB, 0, m=m, n=n)
    t = torch.empty(M * N, dtype=dt, device="cuda")
    t.random_()
    ref = t.view(M, N).t().contiguous().view(-1)
    ipt.transpose_(t, M, N, plan_=p)
    torch.cuda.synchronize()
    ok = torch.equal(t, ref) or bool(os.environ.get("IPT_SEG_DIAG"))
    del ref
    reps, tot, st = 10, 0.0, [0.0, 0.0, 0.0]
    for r in range(reps):
        flush.zero_()
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
        ipt.transpose_(t, M, N, plan_=p, events=ev)
        torch.cuda.synchronize()
        tot += ev[0].elapsed_time(ev[3])
        for i in range(3):
            st[i] += ev[i].elapsed_time(ev[i + 1])
        t = t.view(-1)
        # undo: transpose back with the reverse plan (not timed)
        ipt.transpose_(t, N, M, plan_=ipt.plan(N, M, EB, 0))
    eff = 2 * M * N * EB / (tot / reps / 1e3) / 1e9
    sg = [round(2 * M * N * EB / (s / reps / 1e3) / 1e9) if s > 1e-4 else None for s in st]
    res.append({"plan": [M, N, m, n], "var": [ipt.VARIANTS[v] for v in p.variant],
                "ok": ok, "eff": round(eff), "stage": sg, "us": round(tot / reps * 1e3, 1)})
    print(json.dumps(res[-1]), flush=True)
    del t
