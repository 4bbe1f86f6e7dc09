import ctypes, os, json, torch
L = ctypes.CDLL(os.path.join(os.path.dirname(os.path.abspath(__file__)), "probe", "libprobe.so"))
L.probe_rmw.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_int, ctypes.c_int, ctypes.c_void_p]
dev = torch.device("cuda", 0)
TOT = 12800 * 15000 * 4
x = torch.zeros(TOT, dtype=torch.uint8, device=dev)
st = torch.cuda.current_stream().cuda_stream
for S in [int(v) for v in os.environ.get("SIZES", "256,512,800,1024,2048").split(",")]:
    nblk = TOT // S
    perm = torch.randperm(nblk, device=dev, dtype=torch.int64).to(torch.int32)
    res = {}
    for U in [1, 2]:
        f = lambda: L.probe_rmw(x.data_ptr(), perm.data_ptr(), nblk, S, U, 148, st)
        assert f() == 0; torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(5): f()
        e1.record(); torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / 5
        res[U] = round(2 * nblk * S / ms / 1e6)
    print("S", S, "random RMW GB/s by blocks-in-flight/warp", json.dumps(res), flush=True)
