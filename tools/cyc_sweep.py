"""Microbenchmark of cycle_global (100! / 0100!) alone vs super-element size and knobs."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ppopp_sunggggh14_b200 as ipt
dev = torch.device("cuda", 0)
TOT = 12800 * 15000
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
cfg = os.environ.get("CFG", "")
print("knobs", cfg, flush=True)
st1 = {}
for s in [8, 24, 40, 60, 100, 120, 200, 300, 500, 1000]:
    st1[s * 4] = bench(1, 12800, 15000 // s, s)
print("stage1-like P(1,12800,15000/s,s) S bytes->GB/s", json.dumps(st1), flush=True)
st3 = {}
for m in [32, 64, 100, 128, 160, 200, 256, 320, 400, 640]:
    st3[m * 4] = bench(75, 12800 // m, 200, m)
print("stage3-like P(75,12800/m,200,m) S bytes->GB/s", json.dumps(st3), flush=True)
