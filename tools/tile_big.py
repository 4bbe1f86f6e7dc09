"""Tile stage (0010!) on the large tiles of 2-stage plans, under env variants.
VARIANTS = JSON list of env dicts; SHAPES = list of (m, n) tiles (f32)."""
import os, sys, json, ast, subprocess
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
if os.environ.get("_CHILD"):
    import torch
    import paper_conf_ppopp_sunggggh14_b200 as ipt
    TOT = 12800 * 15000
    oop = int(os.environ.get("IPT_TILE_DIAG", "0")) & 32
    buf = torch.empty(2 * TOT if oop else TOT, dtype=torch.int32, device="cuda")
    buf.random_()
    res = {}
    for (m, n) in ast.literal_eval(os.environ["SHAPES"]):
        cnt = TOT // (m * n)
        ref = buf[:cnt * m * n].view(cnt, m, n).transpose(1, 2).contiguous().view(-1)
        ipt.ipt_010_(buf, cnt, m, n)
        torch.cuda.synchronize()
        ok = torch.equal(buf[:cnt * m * n], ref)
        del ref
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for r in range(5):
            ipt.ipt_010_(buf, cnt, m, n)
        e1.record(); torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / 5
        rate = round(2 * cnt * m * n * 4 / (ms / 1e3) / 1e9)
        res[f"{m}x{n}"] = rate if ok else (f"{rate}?" if os.environ.get("IPT_TILE_DIAG") else "WRONG")
    if os.environ.get("COPY_REF"):   # device copy of the same bytes: the practical ceiling
        dst = torch.empty_like(buf)
        dst.copy_(buf)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for r in range(5):
            dst.copy_(buf)
        e1.record(); torch.cuda.synchronize()
        res["copy"] = round(2 * TOT * 4 / (e0.elapsed_time(e1) / 5 / 1e3) / 1e9)
    print(json.dumps(res), flush=True)
else:
    vf = os.environ.get("VARIANTS_FILE")
    variants = json.load(open(vf)) if vf else json.loads(os.environ.get("VARIANTS", "[{}]"))
    for v in variants:
        env = dict(os.environ, _CHILD="1", **{k: str(x) for k, x in v.items()})
        out = subprocess.run([sys.executable, __file__], env=env, capture_output=True, text=True)
        dbg = sorted(set(l for l in out.stderr.splitlines() if l.startswith("[ipt]")))
        print(json.dumps(v), out.stdout.strip(), out.stderr.strip()[-300:] if out.returncode else "", flush=True)
        for l in dbg:
            print("   ", l)
