import os, sys, itertools
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ppopp_sunggggh14_b200 as ipt
from inputs import seeded
dev = torch.device("cuda", 0)

def runP(batch, A, B, s, reps=2):
    out = []
    for r in range(reps):
        n = batch * A * B * s
        t = torch.empty(n, dtype=torch.int32, device=dev)
        seeded.fill_device_(t, n, 1, 4)
        ref = t.view(batch, A, B, s).permute(0, 2, 1, 3).contiguous().view(-1)
        ipt.ipt_100_(t, batch, A, B, s)
        torch.cuda.synchronize()
        out.append(int((t != ref).sum()))
    print(f"P({batch},{A},{B},{s}) env={os.environ.get('IPT_CYC_REFRESH')},{os.environ.get('IPT_CYC_G')} mism={out}", flush=True)

cases = [(1,128,128,128),(128,128,128,128),(2,64,32,128),(128,128,127,128),(128,127,128,128),(16,128,128,128),(128,64,64,128),(128,128,128,4),(128,128,128,1),(1,1024,1024,4),(1,2048,2048,1),(64,200,200,32)]
for refresh in ["1","0"]:
    os.environ["IPT_CYC_REFRESH"] = refresh
    for c in cases:
        runP(*c)
os.environ["IPT_CYC_REFRESH"] = "1"
for G,R in [(16,2),(8,4)]:
    os.environ["IPT_CYC_G"]=str(G); os.environ["IPT_CYC_R"]=str(R)
    for c in [(128,128,128,128),(1,1024,1024,4)]:
        runP(*c)
