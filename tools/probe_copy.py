"""Copy through shared memory with the group kernel's pipeline shape (tools/probe/probe_copy.cu)."""
import ctypes, os, json, subprocess, torch
HERE = os.path.dirname(os.path.abspath(__file__))
so = os.path.join(HERE, "probe", "libprobe_copy.so")
subprocess.check_call(["nvcc", "-O3", "-gencode", "arch=compute_100a,code=sm_100a", "-shared",
                       "-Xcompiler", "-fPIC", os.path.join(HERE, "probe", "probe_copy.cu"), "-o", so])
L = ctypes.CDLL(so)
L.probe_copy.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int,
                         ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p]
TOT = 768 * 1024 * 1024
a = torch.ones(TOT, dtype=torch.uint8, device="cuda")
b = torch.ones(TOT, dtype=torch.uint8, device="cuda")
ctr = torch.zeros(4, dtype=torch.int32, device="cuda")
st = torch.cuda.current_stream().cuda_stream
def run(ch, grid=148, sync=0, inplace=1):
    dst = a if inplace else b
    f = lambda: L.probe_copy(a.data_ptr(), dst.data_ptr(), TOT, ch, grid, sync, ctr.data_ptr(), st)
    assert f() == 0; torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(5): f()
    e1.record(); torch.cuda.synchronize()
    return round(2 * (TOT // ch) * ch / (e0.elapsed_time(e1) / 5) / 1e6)
res = {}
b.copy_(a); torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(5): b.copy_(a)
e1.record(); torch.cuda.synchronize()
res["torch_copy"] = round(2 * TOT / (e0.elapsed_time(e1) / 5) / 1e6)
for ch in (98304, 110592):
    for inplace in (1,):
        for sync in (0, 1, 2, 3):
            res[f"ch{ch}_ip{inplace}_sync{sync}"] = run(ch, 148, sync, inplace)
print(json.dumps(res, indent=0), flush=True)
