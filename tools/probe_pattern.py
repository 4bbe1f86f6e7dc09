"""DRAM rate of tile-stage-like patterns (tools/probe/probe_pattern.cu)."""
import ctypes, os, json, subprocess, torch
HERE = os.path.dirname(os.path.abspath(__file__))
so = os.path.join(HERE, "probe", "libprobe_pattern.so")
if not os.path.exists(so):
    subprocess.check_call(["nvcc", "-O3", "-gencode", "arch=compute_100a,code=sm_100a", "-shared",
                           "-Xcompiler", "-fPIC", os.path.join(HERE, "probe", "probe_pattern.cu"), "-o", so])
L = ctypes.CDLL(so)
L.probe_pattern.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint64,
                            ctypes.c_uint32, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_void_p]
TOT = 768 * 1024 * 1024
a = torch.zeros(TOT, dtype=torch.uint8, device="cuda")
b = torch.zeros(TOT, dtype=torch.uint8, device="cuda")
st = torch.cuda.current_stream().cuda_stream
def run(rows, X, C, K, inplace, grid, H=0, mode=0):
    T = rows * X
    nt = TOT // T
    nunits = nt * K
    dst = a if inplace else b
    f = lambda: L.probe_pattern(a.data_ptr(), dst.data_ptr(), nunits, K, T, rows, X, C, grid, H, mode, st)
    assert f() == 0; torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(5): f()
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 5
    return round(2 * nunits * rows * C / ms / 1e6)
# (rows, X, C, K): colsplit slice of a 120 x 7200 f32 tile; contiguous equivalents
cases = {"colsplit120x7200": (120, 28800, 1808, 16), "rows64x40000_K16": (64, 40000, 2496, 16),
         "chunks_512": (256, 28672, 512, 56), "chunks_4096": (64, 65536, 4096, 16)}
for name, (rows, X, C, K) in cases.items():
    res = {}
    for inplace in (0, 1):
        for mode in (0, 1, 2):
            res[f"ip{inplace}_m{mode}"] = run(rows, X, C, K, inplace, 148, 0, mode)
    print(name, json.dumps(res), flush=True)
