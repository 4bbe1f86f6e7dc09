"""Read bandwidth of shared-memory fill mechanisms (tools/probe/probe_read.cu)."""
import ctypes, os, json, subprocess, torch
HERE = os.path.dirname(os.path.abspath(__file__))
so = os.path.join(HERE, "probe", "libprobe_read.so")
subprocess.check_call(["nvcc", "-O3", "-gencode", "arch=compute_100a,code=sm_100a", "-shared",
                       "-Xcompiler", "-fPIC", os.path.join(HERE, "probe", "probe_read.cu"), "-o", so])
L = ctypes.CDLL(so)
L.probe_read.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int, ctypes.c_uint32, ctypes.c_uint32,
                         ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32]
TOT = 1536 * 1024 * 1024
a = torch.ones(TOT, dtype=torch.uint8, device="cuda")
sink = torch.zeros(4, dtype=torch.int32, device="cuda")
st = torch.cuda.current_stream().cuda_stream
def run(mode, ch=0, piece=0, grid=148, off=0, rowv=0, pitchv=0):
    f = lambda: L.probe_read(a.data_ptr(), TOT, mode, ch, piece, grid, sink.data_ptr(), st, off, rowv, pitchv)
    assert f() == 0; torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(5): f()
    e1.record(); torch.cuda.synchronize()
    return round(TOT / (e0.elapsed_time(e1) / 5) / 1e6)
res = {}
for off in (0, 16, 64):
    res[f"cp2_96000_off{off}"] = run(1, 96000, off=off)
    res[f"cp2_96000_off{off}_rows60p61"] = run(1, 96000, off=off, rowv=60, pitchv=61)
    res[f"cp2_96000_off{off}_rows60p60"] = run(1, 96000, off=off, rowv=60, pitchv=60)
print(json.dumps(res, indent=0), flush=True)
