"""Whole-matrix 1-stage plans (m = M, n = N) on batches, timed under env variants:
    SHAPES='[(4096,3000,4,64),(1800,7200,4,1)]' VARIANTS='[{}, {"IPT_TILE_RF_OVERLAP": 0}]' python tools/rf_sweep.py
prints effective GB/s (2*M*N*b*count / time) per variant and shape -- both orientations
together, then M x N and N x M alone -- checked against the definition on samples."""
import ast
import json
import os
import subprocess
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
if os.environ.get("_CHILD"):
    import torch

    import paper_conf_ppopp_sunggggh14_b200 as ipt
    from inputs import seeded
    res = {}
    for (M, N, eb, cnt) in ast.literal_eval(os.environ["SHAPES"]):
        # OOP=1: twice the storage, for IPT_TILE_DIAG=32 (stores to a second buffer after the data)
        t = torch.empty(cnt * M * N * (2 if os.environ.get("OOP") else 1), dtype=torch.int32 if eb == 4 else torch.int64,
                        device="cuda")[:cnt * M * N]
        seeded.fill_device_(t, M, N, eb, count=cnt)
        p, q = ipt.plan(M, N, eb, 0, m=M, n=N), ipt.plan(N, M, eb, 0, m=N, n=M)
        kn = ipt.stage_kernels(p, cnt, t)[1]
        for _ in range(2):
            ipt.transpose_batched_(t, cnt, M, N, plan_=p)
            ipt.transpose_batched_(t, cnt, N, M, plan_=q)
        flush = torch.zeros(128 << 20, dtype=torch.int32, device="cuda") if M * N * eb * cnt < (200 << 20) else None
        tot = 0.0
        per = [0.0, 0.0]
        for r in range(6):
            if flush is not None:
                flush.sum()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            ipt.transpose_batched_(t, cnt, M, N, plan_=p) if r % 2 == 0 else ipt.transpose_batched_(t, cnt, N, M, plan_=q)
            e1.record()
            torch.cuda.synchronize()
            tot += e0.elapsed_time(e1)
            per[r % 2] += e0.elapsed_time(e1)
        idx = torch.randint(0, cnt * M * N, (4096,), device="cuda")
        ok = torch.equal(t[idx], seeded.values_torch_sample(idx, eb).to(t.dtype))
        gbs = round(2 * M * N * eb * cnt * 6 / (tot / 1e3) / 1e9)
        fw, bw = (round(2 * M * N * eb * cnt * 3 / (x / 1e3) / 1e9) for x in per)   # M x N, N x M
        res[f"{M}x{N}x{eb}b{cnt}"] = (gbs, fw, bw, kn) if ok else f"WRONG {gbs}"
        del t
        torch.cuda.empty_cache()
    print(json.dumps(res), flush=True)
else:
    for v in json.loads(os.environ.get("VARIANTS", "[{}]")):
        env = dict(os.environ, _CHILD="1", **{k: str(x) for k, x in v.items()})
        out = subprocess.run([sys.executable, __file__], env=env, capture_output=True, text=True)
        print(json.dumps(v), out.stdout.strip(), out.stderr.strip()[-300:] if out.returncode else "", flush=True)
