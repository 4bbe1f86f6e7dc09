"""Tile stage (0010!) on one shape, for ncu captures:  tile_one.py m n [reps] [eb]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ppopp_sunggggh14_b200 as ipt
m, n = int(sys.argv[1]), int(sys.argv[2])
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 2
eb = int(sys.argv[4]) if len(sys.argv) > 4 else 4
TOT = 12800 * 15000 * 4 // eb
buf = torch.empty(TOT, dtype=torch.int32 if eb == 4 else torch.int64, device="cuda")
cnt = TOT // (m * n)
for r in range(reps):
    ipt.ipt_010_(buf, cnt, m, n)
torch.cuda.synchronize()
print("done", cnt, flush=True)
