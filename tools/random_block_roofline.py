"""Practical roofline probe: out-of-place moves of S-byte blocks with a random permutation
(torch gather / scatter kernels), plus a contiguous copy, on the same 768 MB buffer."""
import torch, json
dev = torch.device("cuda", 0)
TOT = 12800 * 15000
x = torch.empty(TOT, dtype=torch.int32, device=dev).random_()
y = torch.empty_like(x)
def t(fn, reps=5):
    fn(); torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps): fn()
    e1.record(); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps
ms = t(lambda: y.copy_(x)); print("copy GB/s", round(2 * TOT * 4 / ms / 1e6))
res = {}
for S in [128, 256, 512, 800, 1024, 2048]:
    s = S // 4
    rows = TOT // s
    xv = x[:rows * s].view(rows, s); yv = y[:rows * s].view(rows, s)
    perm = torch.randperm(rows, device=dev)
    g = t(lambda: torch.index_select(xv, 0, perm, out=yv))
    sc = t(lambda: yv.index_copy_(0, perm, xv))
    res[S] = (round(2 * rows * S / g / 1e6), round(2 * rows * S / sc / 1e6))
print("random block gather/scatter GB/s by S bytes", json.dumps(res))
