"""cycle_global rate vs the random-RMW probe ceiling at the same block size S."""
import os, sys, json, ctypes
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ppopp_sunggggh14_b200 as ipt
HERE = os.path.dirname(os.path.abspath(__file__))
L = ctypes.CDLL(os.path.join(HERE, "probe", "libprobe.so"))
L.probe_rmw.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_int, ctypes.c_int, ctypes.c_void_p]
TOT = 16384 * 16384
buf = torch.empty(TOT, dtype=torch.int32, device="cuda")
buf.random_()
st = torch.cuda.current_stream().cuda_stream
def timeit(f, reps=4):
    f(); torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps): f()
    e1.record(); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps
res = {}
for S in [int(x) for x in os.environ.get("SIZES", "128,256,384,512,768,960,1024,1536,2048").split(",")]:
    s = S // 4
    nblk = TOT // s
    perm = torch.randperm(nblk, device="cuda", dtype=torch.int64).to(torch.int32)
    pr = max(round(2 * nblk * S / timeit(lambda: L.probe_rmw(buf.data_ptr(), perm.data_ptr(), nblk, S, U, 148, st)) / 1e6) for U in (1, 2))
    del perm
    # stage-3-like: P(Np, Mp, n, m) with m = s, n = 128 (like 16384^2 m=64 plans)
    Mp = 16384 // s if 16384 % s == 0 else 16384 // s
    A, B = Mp, 128
    batch = TOT // (A * B * s)
    ms = timeit(lambda: (ipt.ipt_100_(buf, batch, A, B, s), ipt.ipt_100_(buf, batch, B, A, s)))
    cyc3 = round(2 * 2 * batch * A * B * s * 4 / ms / 1e6)
    # stage-1-like: P(1, M, N', n)
    M = 16384
    Np = TOT // (M * s)
    ms = timeit(lambda: (ipt.ipt_100_(buf, 1, M, Np, s), ipt.ipt_100_(buf, 1, Np, M, s)))
    cyc1 = round(2 * 2 * M * Np * s * 4 / ms / 1e6)
    res[S] = {"probe": pr, "cyc_stage3": cyc3, "cyc_stage1": cyc1}
    print(S, res[S], flush=True)
