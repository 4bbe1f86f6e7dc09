"""Microbenchmark of the tile stage (0010!) alone across tile shapes (THREADS=256|512)."""
import os, sys, itertools, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ppopp_sunggggh14_b200 as ipt
dev = torch.device("cuda", 0)
TOT = 12800 * 15000  # elements (768 MB f32)
buf = torch.empty(TOT, dtype=torch.int32, device=dev)
buf.random_()
def bench(m, n, reps=5):
    cnt = TOT // (m * n)
    ipt.ipt_010_(buf, cnt, m, n)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for r in range(reps):
        ipt.ipt_010_(buf, cnt, m, n)
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / reps
    return 2 * cnt * m * n * 4 / (ms / 1e3) / 1e9
import ast
shapes = ast.literal_eval(os.environ.get("SHAPES", "[(128, 200)]"))
thr = os.environ.get("THREADS", "512")
os.environ["IPT_TILE_THREADS"] = thr
res = {}
for (m, n) in shapes:
    try:
        res[f"{m}x{n}"] = round(bench(m, n), 0)
    except Exception as e:
        res[f"{m}x{n}"] = str(e)[:40]
print(f"threads={thr}", json.dumps(res), flush=True)
