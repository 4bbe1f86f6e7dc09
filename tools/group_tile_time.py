"""Stage-2 tiles (ipt_010: batch x (A x B) -> (B x A)) timed under env variants, with the
group configuration each variant launched (IPT_DEBUG line):
    TILES='[(1181,1453,70)]' VARIANTS='[{}, {"IPT_TILE_GROUP_COLSPLIT": 2}]' python tools/group_tile_time.py
GB/s = 2 * batch * A * B * 4 / time (best of 5, float32); results checked against torch."""
import ast
import json
import os
import subprocess
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
if os.environ.get("_CHILD"):
    import torch

    import paper_conf_ppopp_sunggggh14_b200 as ipt
    res = {}
    for (A, B, batch) in ast.literal_eval(os.environ["TILES"]):
        t = torch.randint(-2**31, 2**31 - 1, (batch * A * B,), dtype=torch.int32, device="cuda")
        ref = t.view(batch, A, B).transpose(1, 2).contiguous().view(-1)
        ipt.ipt_010_(t, batch, A, B)
        torch.cuda.synchronize()
        ok = torch.equal(t, ref)
        del ref
        best = 1e9
        for r in range(6):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            ipt.ipt_010_(t, batch, B, A) if r % 2 == 0 else ipt.ipt_010_(t, batch, A, B)
            e1.record()
            torch.cuda.synchronize()
            if r % 2 == 1:
                best = min(best, e0.elapsed_time(e1))
        res[f"{A}x{B}b{batch}"] = round(2 * batch * A * B * 4 / best / 1e6) if ok else "WRONG"
        del t
        torch.cuda.empty_cache()
    print(json.dumps(res), flush=True)
else:
    for v in json.loads(os.environ.get("VARIANTS", "[{}]")):
        env = dict(os.environ, _CHILD="1", IPT_DEBUG="1", **{k: str(x) for k, x in v.items()})
        out = subprocess.run([sys.executable, __file__], env=env, capture_output=True, text=True)
        cfgs = sorted({l.split("] ", 1)[1] for l in out.stderr.splitlines() if "tile_group" in l})
        print(json.dumps(v), out.stdout.strip(), out.stderr.strip()[-300:] if out.returncode else "", flush=True)
        for c in cfgs:
            print("    ", c, flush=True)
