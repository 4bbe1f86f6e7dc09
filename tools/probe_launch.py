"""Launch floor of a tile_group_rf-shaped kernel (tools/probe/probe_launch.cu): us per
back-to-back launch by dynamic shared memory, cooperative attribute and TMEM allocation."""
import ctypes, os, subprocess
HERE = os.path.dirname(os.path.abspath(__file__))
so = os.path.join(HERE, "probe", "libprobe_launch.so")
subprocess.check_call(["nvcc", "-O3", "-gencode", "arch=compute_100a,code=sm_100a", "-shared", "-Xcompiler", "-fPIC",
                       os.path.join(HERE, "probe", "probe_launch.cu"), "-o", so])
L = ctypes.CDLL(so)
L.probe_launch.restype = ctypes.c_float
for smem in (0, 100 * 1024, 227 * 1024):
    for coop in (0, 1):
        for tmem in (0, 1):
            print(f"smem {smem >> 10:3d} KB coop {coop} tmem {tmem}: {L.probe_launch(smem, coop, tmem, 200):.2f} us", flush=True)
