import os, sys, traceback
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ppopp_sunggggh14_b200 as ipt
from inputs import seeded
from oracle import oracle
dev = torch.device("cuda", 0)
print(ipt.lib().ipt_version())
props = torch.cuda.get_device_properties(0)
print(props)
def run010(batch, A, B, eb=4):
    a = seeded.values_np(np.arange(batch*A*B), eb)
    t = torch.from_numpy(a.view(np.int32 if eb==4 else np.int64).copy()).cuda()
    try:
        ipt.ipt_010_(t, batch, A, B); torch.cuda.synchronize()
    except Exception as e:
        print("010", batch, A, B, eb, "ERR", e); return
    ref = oracle.permute_inplace(a.copy(), batch, A, B, 1)
    got = t.cpu().numpy().view(a.dtype)
    print("010", batch, A, B, eb, "ok" if np.array_equal(got, ref) else f"MISMATCH {np.sum(got!=ref)}")
for (b, A, B, eb) in [(3, 8, 8, 4), (3, 64, 48, 4), (5, 60, 44, 4), (3, 8, 8, 8), (3, 60, 44, 8), (300, 20, 40, 8), (2, 61, 59, 4), (2, 160,160,4), (2,160,180,4), (2,180,144,4), (2, 200, 288, 4)]:
    run010(b, A, B, eb)
def runT(M, N, m=None, n=None):
    t = torch.empty(M*N, dtype=torch.int32, device=dev)
    seeded.fill_device_(t, M, N, 4)
    p = ipt.plan(M, N, 4, 0) if m is None else ipt.plan(M, N, 4, 0, m=m, n=n)
    try:
        ipt.transpose_(t, M, N, plan_=p); torch.cuda.synchronize()
    except Exception as e:
        print("T", M, N, p.as_dict(), "ERR", e); return
    pos = torch.arange(M*N, device=dev)
    exp = seeded.values_torch_sample((pos % M) * N + pos // M, 4)
    bad = (t != exp).sum().item()
    print("T", M, N, (p.m, p.n, [ipt.VARIANTS[v] for v in p.variant]), "ok" if bad == 0 else f"MISMATCH {bad}")
for shp in [(1800,7200),(7200,18000),(18000,7200),(4000,3200),(16384,16384),(1021,4093)]:
    runT(*shp)
# isolate stages for 7200x18000
for (m, n) in [(160,180),(144,180),(120,120),(160,160)]:
    runT(7200, 18000, m, n)
