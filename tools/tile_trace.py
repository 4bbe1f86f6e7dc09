"""Timeline of the group-split tile kernel (IPT_TILE_DIAG=16): per iteration, the spread
of start / own-slice-landed / group-complete / write-done times across the CTAs.
    tile_trace.py m n [count]"""
import os, sys, ctypes
os.environ["IPT_TILE_DIAG"] = "16"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ppopp_sunggggh14_b200 as ipt
m, n = int(sys.argv[1]), int(sys.argv[2])
TOT = 12800 * 15000
cnt = int(sys.argv[3]) if len(sys.argv) > 3 else TOT // (m * n)
buf = torch.empty(cnt * m * n, dtype=torch.int32, device="cuda").random_()
for _ in range(3):
    ipt.ipt_010_(buf, cnt, m, n)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record(); ipt.ipt_010_(buf, cnt, m, n); e1.record(); torch.cuda.synchronize()
ms = e0.elapsed_time(e1)
tr = np.zeros(1024 * 64 * 4, dtype=np.uint64)
lib = ipt.lib()
lib.ipt__tile_trace.argtypes = [ctypes.c_void_p, ctypes.c_size_t]
assert lib.ipt__tile_trace(tr.ctypes.data, tr.nbytes) == 0
tr = tr.reshape(1024, 64, 4).astype(np.int64)
ctas = np.nonzero(tr[:, 0, 0])[0]
tr = tr[ctas]
smid = tr[:, 63, 0].copy()
tr = tr[:, :63]
os.makedirs("gpurun_out", exist_ok=True)
np.savez(f"gpurun_out/trace_{m}x{n}.npz", tr=tr, smid=smid, ctas=ctas)
t0 = tr[:, 0, 0].min()
tr = np.where(tr > 0, tr - t0, -1)
print(f"{m}x{n} x{cnt}: {ms*1e3:.1f} us, {2*cnt*m*n*4/ms/1e6:.0f} GB/s, {len(ctas)} CTAs")
print("iter  start(min/max)  landed(min/med/max)  group(min/max)  wdone(min/med/max)   [us]")
for i in range(min(64, tr.shape[1])):
    c = tr[:, i, :]
    ok = c[:, 0] >= 0
    if not ok.any():
        break
    c = c[ok] / 1e3
    print(f"{i:3d}  {c[:,0].min():7.2f} {c[:,0].max():7.2f}   {c[:,1].min():7.2f} {np.median(c[:,1]):7.2f} {c[:,1].max():7.2f}"
          f"   {c[:,2].min():7.2f} {c[:,2].max():7.2f}   {c[:,3].min():7.2f} {np.median(c[:,3]):7.2f} {c[:,3].max():7.2f}")
