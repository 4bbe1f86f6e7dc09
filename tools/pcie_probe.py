"""PCIe ceiling for the e2e number: pinned H2D, D2H, and both at once (GB/s)."""
import torch, json
n = 1 << 30
h1 = torch.empty(n, dtype=torch.uint8, pin_memory=True); h2 = torch.empty(n, dtype=torch.uint8, pin_memory=True)
d1 = torch.empty(n, dtype=torch.uint8, device="cuda"); d2 = torch.empty(n, dtype=torch.uint8, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
def t(fn):
    fn(); torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(); fn(); e1.record(); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / 1e3
res = {}
res["h2d"] = n / t(lambda: d1.copy_(h1, non_blocking=True)) / 1e9
res["d2h"] = n / t(lambda: h2.copy_(d2, non_blocking=True)) / 1e9
def both():
    cur = torch.cuda.current_stream()
    s1.wait_stream(cur); s2.wait_stream(cur)
    with torch.cuda.stream(s1): d1.copy_(h1, non_blocking=True)
    with torch.cuda.stream(s2): h2.copy_(d2, non_blocking=True)
    cur.wait_stream(s1); cur.wait_stream(s2)
res["both_each_dir"] = n / t(both) / 1e9
print(json.dumps({k: round(v, 1) for k, v in res.items()}))
