"""cycle_global throughput for a few super-element sizes under knob settings (env)."""
import os, sys, json, itertools
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ppopp_sunggggh14_b200 as ipt
dev = torch.device("cuda", 0)
TOT = 16384 * 16384
buf = torch.empty(TOT, dtype=torch.int32, device=dev)
buf.random_()
def bench(batch, A, B, s, reps=3):
    ipt.ipt_100_(buf, batch, A, B, s); ipt.ipt_100_(buf, batch, B, A, s)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for r in range(reps):
        ipt.ipt_100_(buf, batch, A, B, s); ipt.ipt_100_(buf, batch, B, A, s)
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / (2 * reps)
    return round(2 * batch * A * B * s * 4 / (ms / 1e3) / 1e9)
import ast
knobs = ast.literal_eval(open(os.environ["KNOBS_FILE"]).read() if os.environ.get("KNOBS_FILE") else os.environ.get("KNOBS", "[{}]"))
CASES = ast.literal_eval(open(os.environ["CASES_FILE"]).read() if os.environ.get("CASES_FILE") else os.environ.get("CASES", "[('S512_st1', (1, 12800, 117, 128))]"))
for kn in knobs:
    for k in list(os.environ):
        if k.startswith("IPT_CYC"): del os.environ[k]
    os.environ.update(kn)
    res = {}
    for name, args in CASES:
        try:
            res[name] = bench(*args)
        except Exception as e:
            res[name] = str(e)[:30]
    print(json.dumps(kn), json.dumps(res), flush=True)
