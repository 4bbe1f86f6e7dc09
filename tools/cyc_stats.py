"""Round statistics of cycle_global for stage-like shapes.  Needs a diagnostic build:
    IPT_NVCC_EXTRA=-DIPT_CYC_STATS python -m paper_conf_ppopp_sunggggh14_b200.build --force
and IPT_CYC_STATS=1 at run time."""
import os, sys, ctypes, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["IPT_CYC_STATS"] = "1"
import torch
import paper_conf_ppopp_sunggggh14_b200 as ipt
dev = torch.device("cuda", 0)
L = ipt.lib()
TOT = 12800 * 15000
buf = torch.empty(TOT, dtype=torch.int32, device=dev).random_()
def run(batch, A, B, s):
    wsb = L.ipt_stage_workspace_bytes(batch, A, B, s, 4)
    ws = torch.zeros(wsb, dtype=torch.uint8, device=dev)
    st = ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    rc = L.ipt_100(ctypes.c_void_p(buf.data_ptr()), batch, A, B, s, 4, ctypes.c_void_p(ws.data_ptr()), wsb, st)
    e1.record(); torch.cuda.synchronize()
    assert rc == 0
    ms = e0.elapsed_time(e1)
    v = ws[64:112].view(torch.int64).tolist()
    units = batch * A * B
    names = ["start", "abort", "step", "lost", "refresh", "iters_per_warp_sum"]
    d = dict(zip(names, v))
    out = {k: round(val / units, 3) for k, val in d.items()}
    out["GBps"] = round(2 * units * s * 4 / ms / 1e6)
    print(f"P({batch},{A},{B},{s}) S={s*4}", json.dumps(out), flush=True)
for (b, A, B, s) in [(1, 12800, 117, 128), (75, 100, 200, 128), (1, 16384, 128, 128), (1, 12800, 250, 60), (75, 64, 200, 200), (1, 12800, 15, 1000)]:
    run(b, A, B, s); run(b, B, A, s)
