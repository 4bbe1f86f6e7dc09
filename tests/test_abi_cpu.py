"""CPU-only tests of the C ABI library (no GPU needed): it loads, exports every symbol
include/ipt.h declares, validates arguments before touching a device, and the planner
(Sec. 7.4) produces valid plans whose stage sequence (simulated with numpy) is the
transpose.  No compute call is made here."""
import ctypes
import math
import os
import random
import re

import numpy as np
import pytest

import paper_conf_ppopp_sunggggh14_b200 as ipt
from paper_conf_ppopp_sunggggh14_b200 import build as ipt_build

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module", autouse=True)
def _built():
    ipt_build.build()


def header_symbols():
    txt = open(os.path.join(ROOT, "include", "ipt.h")).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(ipt_[a-z0-9_]+)\s*\(", txt)))


def test_exports_every_header_symbol():
    syms = header_symbols()
    assert len(syms) >= 17
    L = ctypes.CDLL(ipt.LIB_PATH)
    for s in syms:
        assert hasattr(L, s), s
    # and the Python binding types every one of them
    assert sorted(n for n, _, _ in ipt.ABI) == syms


def test_library_is_sm100a():
    out = os.popen(f"/usr/local/cuda/bin/cuobjdump --list-elf {ipt.LIB_PATH} 2>&1").read()
    assert "sm_100a" in out, out


def test_status_strings_and_version():
    L = ipt.lib()
    for code in range(7):
        assert L.ipt_status_string(code).decode().startswith("IPT_")
    assert "sm_100a" in ipt.version()


def test_validation_before_device():
    """Errors are returned before any launch (and without a GPU)."""
    L = ipt.lib()
    null = ctypes.c_void_p(0)
    assert L.ipt_transpose(null, 4, 4, 4, null) == 1                       # NULL data
    assert L.ipt_transpose(ctypes.c_void_p(256), 4, 4, 3, null) == 2        # elem 3
    assert L.ipt_transpose(ctypes.c_void_p(258), 4, 4, 4, null) == 3        # misaligned
    assert L.ipt_transpose(ctypes.c_void_p(256), 0, 4, 4, null) == 1        # M < 1
    assert L.ipt_transpose(ctypes.c_void_p(256), 2**40, 2**40, 4, null) == 1  # overflow
    assert L.ipt_transpose(ctypes.c_void_p(256), 1, 77, 4, null) == 0       # 1 x N: no-op
    assert L.ipt_transpose(ctypes.c_void_p(256), 77, 1, 8, null) == 0       # M x 1: no-op
    assert L.ipt_100(ctypes.c_void_p(256), 1, 0, 3, 1, 4, null, 0, null) == 1
    assert L.ipt_100(ctypes.c_void_p(256), 0, 3, 3, 1, 4, null, 0, null) == 0  # empty batch
    assert L.ipt_transpose_batched(ctypes.c_void_p(256), 2, 4, 4, 4, 4, null) == 1  # stride too small
    p = ipt.Plan()
    assert L.ipt_plan_with_tiles(12, 10, 5, 5, 4, -1, ctypes.byref(p)) == 1   # 5 does not divide 12
    # host pipeline: arguments checked before the device is touched
    f = L.ipt_transpose_host_pipeline
    P = (ctypes.c_void_p * 2)(256, 512)
    Ms, Ns = (ctypes.c_int64 * 2)(4, 8), (ctypes.c_int64 * 2)(4, 8)
    assert f(P, Ms, Ns, 0, 4, null, 0, null) == 0                             # nothing to do
    assert f(P, Ms, Ns, -1, 4, null, 0, null) == 1                            # count < 0
    assert f(None, Ms, Ns, 2, 4, null, 0, null) == 1                          # NULL arrays
    assert f(P, Ms, Ns, 2, 3, null, 0, null) == 2                             # elem 3
    bad = (ctypes.c_int64 * 2)(4, 0)
    assert f(P, bad, Ns, 2, 4, null, 0, null) == 1                            # M < 1
    Pm = (ctypes.c_void_p * 2)(256, 514)
    assert f(Pm, Ms, Ns, 2, 4, null, 0, null) == 3                            # misaligned host pointer


def test_fastdiv_exact():
    """The multiply-high division used by every kernel's index map (host evaluation)."""
    L = ipt.lib()
    rnd = random.Random(3)
    ds = [1, 2, 3, 7, 25, 127, 128, 129, 1800, 7200, 12345678, 2**31 - 1, 2**32 + 15,
          2**63 - 25, 2**63, 2**64 - 1]
    ns = [0, 1, 2, 3, 2**32 - 1, 2**32, 2**63 - 1, 2**63, 2**64 - 1, 2**64 - 2]
    for d in ds:
        for n in ns + [rnd.randrange(2**64) for _ in range(200)] + [rnd.randrange(10**7) for _ in range(50)]:
            assert L.ipt__fastdiv(n, d) == n // d, (n, d)


def test_fastdiv32_exact():
    L = ipt.lib()
    rnd = random.Random(4)
    ds = [1, 2, 3, 7, 131, 4999, 14803, 65536, 2**31 - 1, 2**31, 2**32 - 1]
    for d in ds:
        for n in [0, 1, d - 1, d, d + 1, 2**32 - 1, 2**31] + [rnd.randrange(2**32) for _ in range(300)]:
            n &= 0xFFFFFFFF
            assert L.ipt__fastdiv32(n, d) == n // d, (n, d)


# ----------------------------------------------------------------------------- planner
def _np_stages(a, M, N, m, n):
    Mp, Np = M // m, N // n
    a = a.reshape(M, Np, n).transpose(1, 0, 2).reshape(-1)            # 100!
    a = a.reshape(Np, Mp, m, n).transpose(0, 1, 3, 2).reshape(-1)     # 0010!
    a = a.reshape(Np, Mp, n, m).transpose(0, 2, 1, 3).reshape(-1)     # 0100!
    return a


SWEEP = [(1800, 7200), (7200, 1800), (5100, 2500), (4000, 3200), (3300, 3900), (2500, 5100),
         (1024, 16384), (4096, 4096), (8192, 2048), (9998, 4096), (9797, 13081), (14803, 1024),
         (19997, 1024), (1021, 4093), (1009, 7001), (10007, 19997), (1_000_000, 256),
         (20000, 30000), (4096, 3000), (5, 3), (64, 64), (2, 2)]


@pytest.mark.parametrize("eb", [4, 8])
def test_plan_valid(eb):
    for (M, N) in SWEEP:
        p = ipt.plan(M, N, eb)
        assert p.M == M and p.N == N and M % p.m == 0 and N % p.n == 0
        assert p.Mp * p.m == M and p.Np * p.n == N
        v = [ipt.VARIANTS[x] for x in p.variant]
        # identity stages exactly when a swapped dimension is 1
        assert (v[0] == "identity") == (p.Np == 1)
        assert (v[1] == "identity") == (p.m == 1 or p.n == 1)
        assert (v[2] == "identity") == (p.Mp == 1 or p.n == 1)
        assert p.n_stages == sum(x != "identity" for x in v)
        # deterministic
        q = ipt.plan(M, N, eb)
        assert (q.m, q.n, list(q.variant)) == (p.m, p.n, list(p.variant))


def test_plan_stage_simulation_is_transpose():
    rnd = random.Random(5)
    shapes = [(rnd.randint(1, 90), rnd.randint(1, 90)) for _ in range(40)] + [(5, 3), (97, 89)]
    for (M, N) in shapes:
        p = ipt.plan(M, N, 4)
        a = np.arange(M * N, dtype=np.uint32)
        assert np.array_equal(_np_stages(a, M, N, p.m, p.n), a.reshape(M, N).T.reshape(-1))


def test_plan_overhead_below_paper_bound():
    """flag bits ~ one per super-element; < 0.1% with m, n in [50, 100]."""
    for (M, N) in [(7200, 1800), (1800, 7200), (4000, 3200), (20000, 20000)]:
        p = ipt.plan(M, N, 4, m=None, n=None)
        data = M * N * 4
        assert p.workspace_bytes < 0.001 * data, (M, N, p.workspace_bytes)
    p = ipt.plan(7200, 1800, 4, m=60, n=60)
    assert p.workspace_bytes < 0.001 * 7200 * 1800 * 4


def test_plan_prefers_vector_tiles_on_large_f32():
    """Sec. 7.4 pruning: big super-elements for stages 1/3, tile on chip for stage 2."""
    for (M, N) in [(12800, 15000), (15000, 12800), (19200, 10000)]:
        p = ipt.plan(M, N, 4)
        assert p.n * 4 >= 256 and p.m * 4 >= 256
        assert p.n * 4 % 16 == 0 and p.m * 4 % 16 == 0     # 16-byte vector super-elements
        assert ipt.VARIANTS[p.variant[1]] == "tile_onchip"
        # 3 stages, or 2 when a whole M x n (m x N) panel fits a group of CTAs on chip
        assert p.n_stages == 3 or (p.n_stages == 2 and (p.m == M or p.n == N))
    # panel plans (one of stages 1/3 elided: m = M or n = N) where the whole panel fits a
    # group of CTAs on chip
    p = ipt.plan(7200, 18000, 4)
    assert p.n_stages >= 2 and ipt.VARIANTS[p.variant[1]] == "tile_onchip"
    if p.n_stages == 2:
        assert (p.m == 7200 and p.n * 4 >= 256) or (p.n == 18000 and p.m * 4 >= 256)


def test_workspace_batch_scales():
    # flag bits scale with the batch (one per unit and matrix) ...
    p = ipt.plan(4096, 3000, 4, m=256, n=3000)          # tile stage + cycle stage
    w1, w8 = ipt.workspace_bytes(p, 1), ipt.workspace_bytes(p, 8)
    assert w8 > w1 and w8 <= 8 * w1 + 256
    # ... a one-stage whole-matrix plan (the tile on chip) needs only the group counters
    p = ipt.plan(4096, 3000, 4)
    assert p.n_stages == 1 and ipt.workspace_bytes(p, 512) == ipt.workspace_bytes(p, 1) == 8192


def test_group_split_extends_on_chip_tiles():
    """Tiles beyond 16 x 227 KB clusters run on chip over co-resident CTA groups (up to
    ~148 x 113 KB double-buffered, ~148 x 227 KB single-buffered); larger tiles fall back to
    cycle following.  A tile
    stage reserves 8 KB of workspace for the group counters (nominal B200, no GPU)."""
    V = ipt.VARIANTS
    for (M, N, m, n) in [(4096, 8192, 1024, 1024 + 1024),  # 8 MB 16-byte-path tiles
                         (16384, 16384, 128, 16384),   # 8 MB panels (n = N)
                         (14803, 8192, 14803, 128),    # 7.6 MB element-path panels (m = M)
                         (12288, 9998, 192, 9998)]:
        p = ipt.plan(M, N, 4, m=m, n=n)
        assert V[p.variant[1]] == "tile_onchip", (M, N, m, n)
        assert p.workspace_bytes >= 8192
    # up to ~148 x 227 KB with ONE slice buffer per CTA (single-buffered groups)
    p = ipt.plan(4096, 8192, 4, m=4096, n=2048)         # 32 MB: single-buffered group
    assert V[p.variant[1]] == "tile_onchip"
    # up to ~148 x (227 KB smem + 256 KB TMEM) for whole-GPU tiles (tile_group_rf)
    p = ipt.plan(8192, 8192, 4, m=8192, n=2048)         # 64 MB: smem + tensor memory
    assert V[p.variant[1]] == "tile_onchip" and ipt.stage_kernels(p)[1] == "tile_group_rf"
    p = ipt.plan(8192, 8192, 4, m=8192, n=4096)         # 128 MB: beyond on-chip storage
    assert V[p.variant[1]] == "cycle_global"
    assert ipt.lib().ipt_stage_workspace_bytes(3, 120, 7200, 1, 4) >= 8192
    assert ipt.lib().ipt_stage_workspace_bytes(1, 4, 4, 5, 4) < 8192   # cycle stage: flags only


def test_square_matrices_plan_single_swap_pass():
    """a square matrix is transposed by swapping symmetric elements (cycles of length
    2) -- the planner makes it one stage, stage 2 with the whole matrix as one square tile
    executed by the swap kernel (no flags, no workspace), for any side incl. primes."""
    V = ipt.VARIANTS
    for M in [1000, 2048, 4096, 10007, 16384, 20000]:
        for eb in (4, 8, 16):
            if M * M * eb <= (1 << 24):   # squares up to ~16 MB may stay on chip (CTA groups)
                continue
            p = ipt.plan(M, M, eb)
            assert (p.m, p.n, p.n_stages) == (M, M, 1), (M, eb)
            assert [V[v] for v in p.variant] == ["identity", "square_swap", "identity"]
            assert p.workspace_bytes == 0
    # rectangular shapes never get a swap stage unless their tiles are square
    for (M, N) in [(7200, 18000), (9998, 12288), (1_000_000, 256), (4096, 3000)]:
        p = ipt.plan(M, N, 4)
        assert V[p.variant[1]] != "square_swap" or p.m == p.n


def test_forced_square_tiles_plan_validation():
    """Square stage-2 tiles may be forced (m = n | gcd(M, N)); a hand-made plan with a swap
    stage on non-square tiles is rejected before any launch."""
    p = ipt.plan(7200, 1800, 4, m=1800, n=1800)
    assert ipt.VARIANTS[p.variant[1]] in ("square_swap", "tile_onchip")
    q = ipt.plan(7200, 1800, 4, m=120, n=200)
    q.variant[1] = 4
    assert ipt.lib().ipt_workspace_bytes(ctypes.byref(q), 1) == 0   # invalid plan -> 0


def test_cost_model_hook_ranks_single_pass_squares_and_rejects_bad_tiles():
    """ipt__plan_cost (tooling hook): invalid tiles -> -1; for a square matrix the
    single swap pass is predicted cheaper than any 2-stage panel plan; small jobs pay
    per-stage overheads (a 3-stage plan costs more per byte on a small matrix than on a
    large one with the same tiles)."""
    L = ipt.lib()
    f = L.ipt__plan_cost
    f.restype = ctypes.c_double
    f.argtypes = [ctypes.c_int64] * 4 + [ctypes.c_int, ctypes.c_int]
    assert f(100, 100, 7, 10, 4, -1) == -1.0
    sq = f(16384, 16384, 16384, 16384, 4, -1)
    assert sq > 0 and all(sq < f(16384, 16384, m, 16384, 4, -1) for m in (64, 128, 256))
    assert f(1800, 7200, 120, 120, 4, -1) > f(18000, 72000, 120, 120, 4, -1)


def test_cycle_segments_cover_every_position_once():
    """Host logic of the segmented cycle stage (cycle_seg.cu): the segments built for at
    most W walkers read and write every moved unit exactly once (fixed points untouched,
    P:86-89 Eq. (1) on units), with L the smallest length that fits W; the cycle count
    bounds it from below (one segment per cycle at least)."""
    f = ipt.lib().ipt__seg_check
    f.restype = ctypes.c_int64
    f.argtypes = [ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint64, ctypes.POINTER(ctypes.c_uint64)]
    L = ctypes.c_uint64(0)
    for (A, B, W) in [(5, 3, 4), (5, 3, 100), (3, 5, 2), (64, 64, 100), (64, 64, 10000),
                      (1800, 40, 9472), (40, 1800, 9472), (97, 89, 50), (1, 7, 3), (7, 1, 3),
                      (2, 2, 1), (360, 1000, 3000), (17, 31, 5)]:
        nseg = f(A, B, W, ctypes.byref(L))
        if A == 1 or B == 1:
            assert nseg == 0, (A, B)
            continue
        if nseg == -1:       # more cycles than walkers: the stage uses the flag kernel
            assert (A, B, W) in [(64, 64, 100), (97, 89, 50), (17, 31, 5)] or W < 4, (A, B, W)
            continue
        assert 0 < nseg <= W, (A, B, W, nseg)
        moved = A * B - sum(1 for k in range(A * B) if (k % B) * A + k // B == k)
        assert L.value >= -(-moved // W), (A, B, W, L.value)
    # 5 x 3: 5 cycles, 3 of them fixed points -> 12 moved units in two cycles of 6
    assert f(5, 3, 100, ctypes.byref(L)) == 12 and L.value == 1   # one unit per walker
    assert f(5, 3, 4, ctypes.byref(L)) == 4 and L.value == 3      # 6 = 3 + 3, twice
    assert f(5, 3, 2, ctypes.byref(L)) == 2 and L.value == 6      # one walker per cycle
    assert f(5, 3, 1, ctypes.byref(L)) == -1                      # 2 cycles > 1 walker


def _build_c_example(tmp_path):
    import shutil
    import subprocess
    gcc = shutil.which("gcc")
    if not gcc or not os.path.exists("/usr/local/cuda/include/cuda_runtime.h"):
        pytest.skip("gcc / CUDA headers not available")
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    pkg = os.path.join(root, "paper_conf_ppopp_sunggggh14_b200")
    exe = str(tmp_path / "transpose_example")
    r = subprocess.run([gcc, "-O2", "-I", os.path.join(root, "include"), "-I", "/usr/local/cuda/include",
                        os.path.join(root, "examples", "transpose_example.c"), "-L", pkg, "-lipt",
                        f"-Wl,-rpath,{pkg}", "-L", "/usr/local/cuda/lib64", "-lcudart", "-o", exe],
                       capture_output=True, text=True)
    assert r.returncode == 0, r.stderr
    return exe


def test_c_example_compiles_and_links_against_the_abi(tmp_path):
    """A plain C program (examples/transpose_example.c) builds against include/ipt.h and
    links libipt.so: the boundary is usable without Python or torch."""
    ipt.lib()
    _build_c_example(tmp_path)


def test_edited_plans_rejected_before_device():
    """validate_plan: each stage's variant must fit its shape -- stages 1 and 3
    cycle following (identity only when a swapped dimension is 1), stage 2 tile / swap
    (square tiles) / cycle following (identity only when m or n is 1).  Rejected before
    any device use (IPT_ERR_INVALID_ARG = 1); a valid plan gets to the device query
    (IPT_ERR_NO_DEVICE = 6 without a GPU)."""
    L = ipt.lib()
    null = ctypes.c_void_p(0)
    p = ipt.plan(720, 1800, 4, -1, m=120, n=200)
    assert [ipt.VARIANTS[v] for v in p.variant] == ["cycle_global", "tile_onchip", "cycle_global"]
    ok = L.ipt_transpose_plan(ctypes.c_void_p(256), ctypes.byref(p), null, 0, null)
    assert ok in (0, 6)
    for st, v in [(0, 1), (2, 1), (0, 4), (0, 0), (2, 0), (1, 0), (1, 4), (1, 2), (0, 7), (1, -1)]:
        bad = ipt.Plan.from_buffer_copy(p)
        bad.variant[st] = v
        assert L.ipt_transpose_plan(ctypes.c_void_p(256), ctypes.byref(bad), null, 0, null) == 1, (st, v)
    sq = ipt.plan(720, 1800, 4, -1, m=120, n=120)
    sq.variant[1] = 4                                   # square tiles may be swapped
    assert L.ipt_transpose_plan(ctypes.c_void_p(256), ctypes.byref(sq), null, 0, null) in (0, 6)
    one = ipt.plan(720, 1800, 4, -1, m=720, n=1800)     # stages 1 and 3 identities
    assert [ipt.VARIANTS[v] for v in one.variant][0] == "identity"
    assert L.ipt_transpose_plan(ctypes.c_void_p(256), ctypes.byref(one), null, 0, null) in (0, 6)


def test_graph_wrapper_checks_sizes_without_gpu():
    import torch

    p = ipt.plan(36, 10, 4, -1)
    t = torch.zeros(359, dtype=torch.int32)
    with pytest.raises(ipt.IptError):
        ipt.Graph(t, 36, 10, p)                         # 359 < 360 elements
    with pytest.raises(ipt.IptError):
        ipt.Graph(torch.zeros(360, dtype=torch.int32), 10, 36, p)   # plan for 36 x 10
