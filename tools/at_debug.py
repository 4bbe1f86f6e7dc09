import os, sys
sys.path.insert(0, os.getcwd())
import torch, paper_conf_ppopp_sunggggh14_b200 as ipt
for (M, N) in [(18000, 7200), (7200, 18000)]:
    t = torch.empty(M * N, dtype=torch.int32, device="cuda"); t.random_()
    p = ipt.plan_autotune(t, M, N, 24)
    print("chosen", M, N, p.m, p.n, flush=True)
