"""cycle_global alone on one P(batch, A, B, s) (for ncu):  cyc_one.py batch A B s [reps]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ppopp_sunggggh14_b200 as ipt
b, A, B, s = (int(x) for x in sys.argv[1:5])
reps = int(sys.argv[5]) if len(sys.argv) > 5 else 2
buf = torch.empty(b * A * B * s, dtype=torch.int32, device="cuda")
buf.random_()
for r in range(reps):
    ipt.ipt_100_(buf, b, A, B, s)
    ipt.ipt_100_(buf, b, B, A, s)
torch.cuda.synchronize()
print("done")
