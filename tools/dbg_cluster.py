import os, sys
sys.path.insert(0, os.getcwd())
os.environ["IPT_DEBUG"] = "1"
import torch, paper_conf_ppopp_sunggggh14_b200 as ipt
buf = torch.empty(12800 * 15000, dtype=torch.int32, device="cuda")
for (m, n) in [(800, 400), (400, 400), (1800, 60), (1600, 256), (512, 512)]:
    cnt = buf.numel() // (m * n)
    ipt.ipt_010_(buf, cnt, m, n); torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(); ipt.ipt_010_(buf, cnt, m, n); e1.record(); torch.cuda.synchronize()
    print(m, n, e0.elapsed_time(e1), "ms", flush=True)
