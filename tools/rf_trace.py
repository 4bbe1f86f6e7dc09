"""Timeline of tile_group_rf (IPT_TILE_DIAG=16): per tile, the spread over the CTAs of the
phase end times (us from the first CTA's start):
    rf_trace.py M N count"""
import ctypes
import os
import sys

os.environ["IPT_TILE_DIAG"] = "16"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ppopp_sunggggh14_b200 as ipt  # noqa: E402

M, N, cnt = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
t = torch.empty(cnt * M * N, dtype=torch.int32, device="cuda").random_()
p = ipt.plan(M, N, 4, 0, m=M, n=N)
q = ipt.plan(N, M, 4, 0, m=N, n=M)
for _ in range(2):
    ipt.transpose_batched_(t, cnt, M, N, plan_=p)
    ipt.transpose_batched_(t, cnt, N, M, plan_=q)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
ipt.transpose_batched_(t, cnt, M, N, plan_=p)
e1.record()
torch.cuda.synchronize()
ms = e0.elapsed_time(e1)
tr = np.zeros(1024 * 64 * 4, dtype=np.uint64)
lib = ipt.lib()
lib.ipt__tile_trace.argtypes = [ctypes.c_void_p, ctypes.c_size_t]
assert lib.ipt__tile_trace(tr.ctypes.data, tr.nbytes) == 0
tr = tr.reshape(1024, 32, 8)[:148].astype(np.int64)
t0 = tr[:, 0, 0].min()
tr = np.where(tr > 0, tr - t0, -1) / 1e3
names = ["start", "B parked", "A landed", "group", "A written", "B staged", "B written"]
print(f"{M}x{N} x{cnt}: {ms * 1e3:.1f} us, {2 * cnt * M * N * 4 / ms / 1e6:.0f} GB/s")
print("tile " + "".join(f"{n:>22s}" for n in names))
for i in range(min(cnt, 31)):
    c = tr[:, i, :]
    if (c[:, 0] < 0).all():
        break
    print(f"{i:4d} " + "".join(f"   {c[:, k].min():6.1f}/{np.median(c[:, k]):6.1f}/{c[:, k].max():6.1f}" for k in range(7)))
# per-CTA phase durations, averaged over tiles 1..: which CTAs (SMs) are slow?
raw = np.zeros(1024 * 64 * 4, dtype=np.uint64)
lib.ipt__tile_trace(raw.ctypes.data, raw.nbytes)
raw = raw.reshape(1024, 32, 8)[:148].astype(np.int64)
smid = raw[:, 31, 0]
nt = min(cnt, 31)
if nt > 2:
    d = raw[:, 1:nt, :].astype(np.float64) / 1e3
    load = (d[:, :, 1] - d[:, :, 0]).mean(1)
    wa = (d[:, :, 4] - d[:, :, 3]).mean(1)
    sb = (d[:, :, 5] - d[:, :, 4]).mean(1)
    wb = (d[:, :, 6] - d[:, :, 5]).mean(1)
    tot = wa + sb + wb
    order = np.argsort(tot)
    print("slowest CTAs (cta, sm, load, writeA, stageB, writeB us):")
    for c in order[-8:]:
        print(f"  cta {c:3d} sm {smid[c]:3d}  {load[c]:5.1f} {wa[c]:5.1f} {sb[c]:5.1f} {wb[c]:5.1f}")
    print("fastest:")
    for c in order[:4]:
        print(f"  cta {c:3d} sm {smid[c]:3d}  {load[c]:5.1f} {wa[c]:5.1f} {sb[c]:5.1f} {wb[c]:5.1f}")
    print(f"median load {np.median(load):.1f} writeA {np.median(wa):.1f} stageB {np.median(sb):.1f} writeB {np.median(wb):.1f}")
    rows = np.array([((c + 1) * (M // 4) // 148 - c * (M // 4) // 148) for c in range(148)])
    print("rows(V-blocks) of the slowest:", rows[order[-8:]], " fastest:", rows[order[:4]])
if nt > 2 and os.environ.get("RF_TRACE_ALL"):
    wt = wa + sb + wb
    print("per SM (sm: write us):")
    by = sorted(zip(smid, wt, load))
    print(" ".join(f"{int(s)}:{w:.1f}" for s, w, _ in by))
    np.save("gpurun_out/rf_sm_write.npy", np.array([[s, w, l] for s, w, l in by]))
