"""Square swap kernel (square_swap.cu) on batches of g x g items, under env variants.
SHAPES = list of (g, eb); each fills a ~800 MB buffer with as many items as fit.
VARIANTS = JSON list of env dicts (e.g. {"IPT_SQ_TB": 512})."""
import os, sys, json, ast, subprocess
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
if os.environ.get("_CHILD"):
    import torch
    import paper_conf_ppopp_sunggggh14_b200 as ipt
    TOT_BYTES = 800 << 20
    dt = {2: torch.int16, 4: torch.int32, 8: torch.int64, 16: torch.int64}
    res = {}
    for (g, eb) in ast.literal_eval(os.environ["SHAPES"]):
        cnt = max(1, TOT_BYTES // (g * g * eb))
        w = 2 if eb == 16 else 1
        buf = torch.empty(cnt * g * g * w, dtype=dt[eb], device="cuda")
        buf.random_()
        ref = buf.view(cnt, g, g, w).transpose(1, 2).contiguous().view(-1)
        ipt.ipt_010_(buf, cnt, g, g, elem_bytes=eb)
        torch.cuda.synchronize()
        ok = torch.equal(buf, ref)
        del ref
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for r in range(5):
            ipt.ipt_010_(buf, cnt, g, g, elem_bytes=eb)
        e1.record(); torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / 5
        rate = round(2 * cnt * g * g * eb / (ms / 1e3) / 1e9)
        res[f"{g}^2x{cnt}/{eb}"] = rate if ok else "WRONG"
        del buf
    print(json.dumps(res), flush=True)
else:
    variants = json.loads(os.environ.get("VARIANTS", "[{}]"))
    for v in variants:
        env = dict(os.environ, _CHILD="1", IPT_SQ_FORCE="1", **{k: str(x) for k, x in v.items()})
        out = subprocess.run([sys.executable, __file__], env=env, capture_output=True, text=True)
        dbg = sorted(set(l for l in out.stderr.splitlines() if l.startswith("[ipt]")))
        print(json.dumps(v), out.stdout.strip(), out.stderr.strip()[-300:] if out.returncode else "", flush=True)
        for l in dbg[:6]:
            print("   ", l)
