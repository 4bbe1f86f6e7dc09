"""cycle stage rate vs super-element bytes: ipt_100_ on P(1, A, B, s) (~1 GB, f32) with the
flag kernel (IPT_CYC_SEG=0) and the segmented kernel (IPT_CYC_SEG=2); prints TB/s."""
import json, os, subprocess, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
SIZES = json.loads(os.environ.get("SIZES", "[64, 128, 192, 256, 320, 384, 512, 640, 768, 960, 1024, 1536, 2000, 2048, 3200, 4096]"))
if os.environ.get("_CHILD"):
    import torch
    import paper_conf_ppopp_sunggggh14_b200 as ipt
    TOT = 1 << 30
    buf = torch.empty(TOT // 4, dtype=torch.int32, device="cuda")
    buf.random_()
    res = {}
    for S in SIZES:
        s = S // 4
        units = TOT // S
        A = 1
        while A * A < units: A *= 2
        A = A // 2 + 3          # not a power of two: no trivial cycle structure
        B = units // A
        n = A * B * s
        t = buf[:n]
        ref = t.view(A, B, s).transpose(0, 1).contiguous().view(-1)
        ipt.ipt_100_(t, 1, A, B, s)
        torch.cuda.synchronize()
        ok = torch.equal(t, ref)
        del ref
        ipt.ipt_100_(t, 1, B, A, s)          # back (and builds the reverse segment plan)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for r in range(4):
            ipt.ipt_100_(t, 1, A if r % 2 == 0 else B, B if r % 2 == 0 else A, s)
        e1.record(); torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / 4
        res[S] = round(2 * n * 4 / (ms / 1e3) / 1e12, 2) if ok else "WRONG"
    print(json.dumps(res), flush=True)
else:
    extra = json.loads(os.environ.get("VARIANTS", "[{}]"))
    for mode in json.loads(os.environ.get("MODES", "[\"0\", \"2\"]")):
        for v in extra:
            env = dict(os.environ, _CHILD="1", IPT_CYC_SEG=mode, **{k: str(x) for k, x in v.items()})
            out = subprocess.run([sys.executable, __file__], env=env, capture_output=True, text=True)
            print("IPT_CYC_SEG=" + mode, json.dumps(v), out.stdout.strip(), out.stderr.strip()[-400:] if out.returncode else "", flush=True)
