"""Planner plans of whole shapes timed under env variants (A/B of a kernel knob on the
shapes the bench runs):
    SHAPES='[(16534,7265)]' VARIANTS='[{}, {"IPT_TILE_GROUP_2D": 0}]' python tools/variant_time.py
prints, per variant, ms per transpose (best of 3, M x N and N x M averaged) and the stage
kernels; results checked on samples after an even number of transposes."""
import ast
import json
import os
import subprocess
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
if os.environ.get("_CHILD"):
    import torch

    import paper_conf_ppopp_sunggggh14_b200 as ipt
    eb = int(os.environ.get("EB", "4"))
    res = {}
    for (M, N) in ast.literal_eval(os.environ["SHAPES"]):
        t = torch.randint(-2**31, 2**31 - 1, (M * N,), dtype=torch.int32, device="cuda") if eb == 4 else \
            torch.randint(-2**62, 2**62, (M * N,), dtype=torch.int64, device="cuda")
        ref = t[:: max(1, M * N // 4096)].clone()
        if os.environ.get("AUTOTUNE"):   # the bench's choice: 8 model candidates timed
            p, q = ipt.plan_autotune(t, M, N, 8), ipt.plan_autotune(t, N, M, 8)
        else:
            p, q = ipt.plan(M, N, eb, 0), ipt.plan(N, M, eb, 0)
        ks = [ipt.stage_kernels(p, 1, t), ipt.stage_kernels(q, 1, t)]
        ipt.transpose_(t, M, N, plan_=p)
        ipt.transpose_(t, N, M, plan_=q)
        best = [1e9, 1e9]
        for r in range(6):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            if r % 2 == 0:
                ipt.transpose_(t, M, N, plan_=p)
            else:
                ipt.transpose_(t, N, M, plan_=q)
            e1.record()
            torch.cuda.synchronize()
            best[r % 2] = min(best[r % 2], e0.elapsed_time(e1))
        ok = torch.equal(t[:: max(1, M * N // 4096)], ref)
        ms = (best[0] + best[1]) / 2
        res[f"{M}x{N}"] = [round(ms, 4), round(2 * M * N * eb / ms / 1e6), [round(b, 4) for b in best], ks] if ok else "WRONG"
        del t
        torch.cuda.empty_cache()
    print(json.dumps(res), flush=True)
else:
    for v in json.loads(os.environ.get("VARIANTS", "[{}]")):
        env = dict(os.environ, _CHILD="1", **{k: str(x) for k, x in v.items()})
        out = subprocess.run([sys.executable, __file__], env=env, capture_output=True, text=True)
        print(json.dumps(v), out.stdout.strip(), out.stderr.strip()[-300:] if out.returncode else "", flush=True)
