"""Stage isolation: run each stage of a plan through the elementary ABI and compare with
torch reshape/permute on the device (debug only)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ppopp_sunggggh14_b200 as ipt
from inputs import seeded
dev = torch.device("cuda", 0)

def stages(M, N, m, n, reps=3):
    Mp, Np = M // m, N // n
    for r in range(reps):
        t = torch.empty(M * N, dtype=torch.int32, device=dev)
        seeded.fill_device_(t, M, N, 4)
        ref = t.clone()
        res = []
        # stage 1
        ipt.ipt_100_(t, 1, M, Np, n); ref = ref.view(M, Np, n).permute(1, 0, 2).contiguous().view(-1)
        res.append(int((t != ref).sum()))
        t.copy_(ref)
        ipt.ipt_0010_(t, Np, Mp, m, n); ref = ref.view(Np, Mp, m, n).permute(0, 1, 3, 2).contiguous().view(-1)
        res.append(int((t != ref).sum()))
        t.copy_(ref)
        ipt.ipt_0100_(t, Np, Mp, n, m); ref = ref.view(Np, Mp, n, m).permute(0, 2, 1, 3).contiguous().view(-1)
        res.append(int((t != ref).sum()))
        torch.cuda.synchronize()
        print(f"{M}x{N} m={m} n={n} rep{r} mismatches per stage {res}", flush=True)

for env in ["1", "0"]:
    os.environ["IPT_CYC_FENCE"] = env
    print("IPT_CYC_FENCE", env)
    for (M, N, m, n) in [(16384, 16384, 128, 128), (7200, 18000, 120, 120), (7200, 18000, 160, 180), (4000, 3200, 160, 160)]:
        stages(M, N, m, n)
    # scalar single stage
    for r in range(3):
        M, N = 1021, 4093
        t = torch.empty(M * N, dtype=torch.int32, device=dev)
        seeded.fill_device_(t, M, N, 4)
        ref = t.view(M, N).t().contiguous().view(-1)
        ipt.ipt_100_(t, 1, M, N, 1)
        print("scalar 1021x4093 mismatches", int((t != ref).sum()), flush=True)
