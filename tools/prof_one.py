"""Run one workload matrix a few times (for ncu captures):  prof_one.py M N [reps] [eb]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ppopp_sunggggh14_b200 as ipt
from inputs import seeded
M, N = int(sys.argv[1]), int(sys.argv[2])
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 2
eb = int(sys.argv[4]) if len(sys.argv) > 4 else 4
t = torch.empty(M * N, dtype=torch.int32 if eb == 4 else torch.int64, device="cuda")
seeded.fill_device_(t, M, N, eb)
p1, p2 = ipt.plan(M, N, eb, 0), ipt.plan(N, M, eb, 0)
print(p1.as_dict(), p2.as_dict(), flush=True)
for r in range(reps):
    ipt.transpose_(t, M, N, plan_=p1)
    ipt.transpose_(t, N, M, plan_=p2)
torch.cuda.synchronize()
print("done", flush=True)
