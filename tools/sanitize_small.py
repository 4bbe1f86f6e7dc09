"""Small end-to-end runs for compute-sanitizer (memcheck / racecheck / synccheck)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ppopp_sunggggh14_b200 as ipt
from inputs import seeded
from oracle import oracle
ok = True
for (M, N, m, n) in [(120, 72, 12, 8), (97, 89, 97, 89), (360, 1000, 40, 25), (64, 64, 64, 64), (131, 256, 131, 128)]:
    for eb in (4, 8):
        a = seeded.matrix_np(M, N, eb)
        t = torch.from_numpy(a.view(np.int32 if eb == 4 else np.int64).copy()).cuda()
        ipt.transpose_(t, M, N, plan_=ipt.plan(M, N, eb, 0, m=m, n=n))
        got = t.cpu().numpy().view(a.dtype)
        ok &= np.array_equal(got, oracle.transpose_inplace(a.copy(), M, N))
# cluster tile, element path, realigning walker
for (b, A, B, s) in [(2, 64, 20, 1), (1, 40, 30, 131)]:
    a = seeded.values_np(np.arange(b * A * B * s), 4)
    t = torch.from_numpy(a.view(np.int32).copy()).cuda()
    ipt.ipt_100_(t, b, A, B, s)
    ok &= np.array_equal(t.cpu().numpy().view(np.uint32), oracle.permute_inplace(a.copy(), b, A, B, s))
a = seeded.values_np(np.arange(2 * 512 * 512), 4)
t = torch.from_numpy(a.view(np.int32).copy()).cuda()
ipt.ipt_010_(t, 2, 512, 512)
ok &= np.array_equal(t.cpu().numpy().view(np.uint32), oracle.permute_inplace(a.copy(), 2, 512, 512, 1))
# square swaps: register-staged 256/512-byte blocks, 1024-thread CTAs, element path,
# TMA ring; ragged sides and batches
def sq(g, batch, eb, env):
    global ok
    for k, v in env.items():
        os.environ[k] = v
    a = seeded.values_np(np.arange(batch * g * g), eb)
    t = torch.from_numpy(a.view(np.int32 if eb == 4 else np.int64).copy()).cuda()
    ipt.ipt_010_(t, batch, g, g, elem_bytes=eb)
    ok &= np.array_equal(t.cpu().numpy().view(a.dtype), oracle.permute_inplace(a.copy(), batch, g, g, 1))
    for k in env:
        del os.environ[k]
for env in [{"IPT_SQ_FORCE": "1", "IPT_SQ_TB": "256"}, {"IPT_SQ_FORCE": "1", "IPT_SQ_TB": "512"},
            {"IPT_SQ_FORCE": "1", "IPT_SQ_TB": "512", "IPT_SQ_NT": "512"},
            {"IPT_SQ_FORCE": "1", "IPT_SQ_ELEM": "1"}]:
    sq(300, 2, 4, env)
    sq(129, 3, 8, env)
# element-path group tiles: TMA slices (aligned input rows) and cp.async slices
for (b, A, B) in [(2, 999, 96), (2, 96, 999)]:
    a = seeded.values_np(np.arange(b * A * B), 4)
    t = torch.from_numpy(a.view(np.int32).copy()).cuda()
    ipt.ipt_010_(t, b, A, B)
    ok &= np.array_equal(t.cpu().numpy().view(np.uint32), oracle.permute_inplace(a.copy(), b, A, B, 1))
# segmented cycle following (one grid barrier, no flags)
os.environ["IPT_CYC_SEG"] = "2"
for (b, A, B, s) in [(1, 180, 40, 36), (3, 17, 31, 8), (2, 40, 56, 600)]:
    a = seeded.values_np(np.arange(b * A * B * s), 4)
    t = torch.from_numpy(a.view(np.int32).copy()).cuda()
    ipt.ipt_100_(t, b, A, B, s)
    ok &= np.array_equal(t.cpu().numpy().view(np.uint32), oracle.permute_inplace(a.copy(), b, A, B, s))
del os.environ["IPT_CYC_SEG"]
torch.cuda.synchronize()
print("sanitize run ok" if ok else "MISMATCH")
