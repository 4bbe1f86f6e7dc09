"""GPU parity: libipt's CUDA kernels (through the C ABI) vs the CPU oracle, bit-exact.

Small/medium sizes span many tiles, chains and ragged tails and are compared element by
element with the oracle's output on the same seeded input.  Full BASELINE sizes are run
in the bench's launch configuration and checked (a) on sampled outputs computed one by
one by the oracle's Eq. (1) and the generator, and (b) on every element through the
transposition's definition A^T(j, i) = A(i, j) evaluated with torch index arithmetic.
"""
import os
import random

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")

import paper_conf_ppopp_sunggggh14_b200 as ipt  # noqa: E402
from inputs import seeded  # noqa: E402
from oracle import oracle  # noqa: E402

_TDT = {1: torch.uint8, 2: torch.int16, 4: torch.int32, 8: torch.int64}
_NDT = {1: np.uint8, 2: np.int16, 4: np.int32, 8: np.int64}


def to_dev(a: np.ndarray, eb: int):
    if eb == 16:
        return torch.from_numpy(a.view(np.int64).copy()).cuda()
    return torch.from_numpy(a.view(_NDT[eb]).copy()).cuda()


def to_np(t, eb: int):
    a = t.cpu().numpy()
    if eb == 16:
        return a.view(np.uint64)
    return a.view(oracle.dtype_for(eb))


def gen(n_elems: int, eb: int, seed=seeded.SEED):
    if eb == 16:
        return seeded.values_np(np.arange(2 * n_elems), 8, seed)
    return seeded.values_np(np.arange(n_elems), eb, seed)


def oracle_P(a, batch, A, B, s, eb):
    if eb == 16:  # 16-byte elements = super-elements of two 8-byte words
        return oracle.permute_inplace(a, batch, A, B, 2 * s)
    return oracle.permute_inplace(a, batch, A, B, s)


@pytest.fixture(autouse=True)
def _env_clean(monkeypatch):
    for k in list(os.environ):
        if k.startswith("IPT_"):
            monkeypatch.delenv(k, raising=False)
    yield


# -------------------------------------------------------------- elementary: 100! / 0100!
@pytest.mark.parametrize("eb", [4, 8])
@pytest.mark.parametrize("seg", ["0", "1", "2"])
def test_ipt_100_random_shapes(monkeypatch, eb, seg):
    """Cycle following of super-elements: flag-based PTTWAC (IPT_CYC_SEG=0), the default
    choice, and precomputed cycle segments wherever applicable (2)."""
    monkeypatch.setenv("IPT_CYC_SEG", seg)
    rnd = random.Random(100 + eb)
    for _ in range(60):
        batch = rnd.choice([1, 1, 2, 3, 5])
        A, B = rnd.randint(1, 70), rnd.randint(1, 70)
        s = rnd.choice([1, 2, 3, 4, 7, 8, 16, 25, 32, 50, 64, 100, 129, 200, 333])
        a = gen(batch * A * B * s, eb)
        t = to_dev(a, eb)
        ipt.ipt_100_(t, batch, A, B, s)
        ref = oracle_P(a.copy(), batch, A, B, s, eb)
        assert np.array_equal(to_np(t, eb), ref), (batch, A, B, s, eb)


@pytest.mark.parametrize("batch,A,s", [(128, 128, 128), (16, 128, 128), (128, 64, 128),
                                       (128, 128, 4), (128, 128, 1), (1, 1024, 4), (1, 2048, 1),
                                       (64, 200, 32)])
def test_ipt_100_square(batch, A, s):
    """Square A x A super-element matrices: every cycle has length 2 and closes at its
    start, the case that exposed the unclaimed cycle-close race (tools/protocol_sim.py)."""
    n = batch * A * A * s
    t = torch.empty(n, dtype=torch.int32, device="cuda")
    seeded.fill_device_(t, n, 1, 4)
    ref = t.clone()
    for _ in range(2):
        ipt.ipt_100_(t, batch, A, A, s)
        ref = ref.view(batch, A, A, s).permute(0, 2, 1, 3).contiguous().view(-1)
        assert torch.equal(t, ref)
    # sampled against the oracle's own Eq. (1) as well
    a = gen(min(n, 3 * A * A * s), 4)
    tt = to_dev(a, 4)
    b3 = len(a) // (A * A * s)
    ipt.ipt_100_(tt, b3, A, A, s)
    assert np.array_equal(to_np(tt, 4), oracle.permute_inplace(a.copy(), b3, A, A, s))


@pytest.mark.parametrize("eb", [1, 2, 16])
def test_ipt_100_other_elem_sizes(eb):
    rnd = random.Random(7 + eb)
    for _ in range(25):
        batch, A, B, s = rnd.randint(1, 3), rnd.randint(1, 40), rnd.randint(1, 40), rnd.choice([1, 3, 5, 16, 33])
        a = gen(batch * A * B * s, eb)
        t = to_dev(a, eb)
        ipt.ipt_100_(t, batch, A, B, s, elem_bytes=eb)
        ref = oracle_P(a.copy(), batch, A, B, s, eb)
        assert np.array_equal(to_np(t, eb), ref), (batch, A, B, s, eb)


def test_ipt_0100_and_1000_definitions():
    d0, d1, d2, d3 = 3, 7, 5, 24
    a = gen(d0 * d1 * d2 * d3, 4)
    t = to_dev(a, 4)
    ipt.ipt_0100_(t, d0, d1, d2, d3)
    ref = oracle.permute_inplace(a.copy(), d0, d1, d2, d3)
    assert np.array_equal(to_np(t, 4), ref)
    t = to_dev(a, 4)
    ipt.ipt_1000_(t, d0, d1, d2, d3)
    ref = oracle.permute_inplace(a.copy(), 1, d0, d1, d2 * d3)
    assert np.array_equal(to_np(t, 4), ref)


@pytest.mark.parametrize("G,R,maxvec", [(32, 1, 128), (16, 2, 128), (8, 4, 128), (4, 4, 128),
                                        (32, 4, 128), (32, 2, 7), (32, 1, 3)])
def test_ipt_100_forced_walker_shapes(monkeypatch, G, R, maxvec):
    """Every walker shape (lanes per walker G, vectors per lane R) and super-element
    chunking gives identical bytes."""
    monkeypatch.setenv("IPT_CYC_G", str(G))
    monkeypatch.setenv("IPT_CYC_R", str(R))
    monkeypatch.setenv("IPT_CYC_MAXVEC", str(maxvec))
    for (batch, A, B, s) in [(1, 61, 47, 8), (2, 33, 20, 12), (1, 128, 96, 4), (3, 17, 19, 2)]:
        a = gen(batch * A * B * s, 4)
        t = to_dev(a, 4)
        ipt.ipt_100_(t, batch, A, B, s)
        assert np.array_equal(to_np(t, 4), oracle.permute_inplace(a.copy(), batch, A, B, s)), (G, R, batch, A, B, s)


# -------------------------------------------------------------- elementary: 010! / 0010!
@pytest.mark.parametrize("eb", [4, 8, 16])
def test_ipt_010_tile_fast_path(eb):
    V = 16 // eb
    rnd = random.Random(eb)
    for _ in range(30):
        batch = rnd.randint(1, 400)
        A, B = V * rnd.randint(1, 40), V * rnd.randint(1, 40)
        a = gen(batch * A * B, eb)
        t = to_dev(a, eb)
        ipt.ipt_010_(t, batch, A, B, elem_bytes=eb)
        ref = oracle_P(a.copy(), batch, A, B, 1, eb)
        assert np.array_equal(to_np(t, eb), ref), (batch, A, B, eb)


@pytest.mark.parametrize("eb", [1, 2, 4, 8, 16])
def test_ipt_010_tile_generic_path(eb):
    rnd = random.Random(50 + eb)
    for _ in range(20):
        batch, A, B = rnd.randint(1, 200), rnd.randint(1, 61), rnd.randint(1, 61)
        a = gen(batch * A * B, eb)
        t = to_dev(a, eb)
        ipt.ipt_010_(t, batch, A, B, elem_bytes=eb)
        ref = oracle_P(a.copy(), batch, A, B, 1, eb)
        assert np.array_equal(to_np(t, eb), ref), (batch, A, B, eb)


def test_ipt_010_large_tile_falls_back_to_cycles():
    """A tile larger than shared memory uses cycle following (s = 1)."""
    batch, A, B = 3, 301, 257        # 309 KB f32 tiles
    a = gen(batch * A * B, 4)
    t = to_dev(a, 4)
    ipt.ipt_0010_(t, 1, batch, A, B)
    assert np.array_equal(to_np(t, 4), oracle.permute_inplace(a.copy(), batch, A, B, 1))


def test_ipt_010_forced_generic(monkeypatch):
    monkeypatch.setenv("IPT_TILE_GENERIC", "1")
    batch, A, B = 37, 64, 48
    a = gen(batch * A * B, 4)
    t = to_dev(a, 4)
    ipt.ipt_010_(t, batch, A, B)
    assert np.array_equal(to_np(t, 4), oracle.permute_inplace(a.copy(), batch, A, B, 1))


# ------------------------------------------------------------------- full transposition
SMALL_SHAPES = [(5, 3), (3, 5), (2, 2), (64, 64), (100, 36), (36, 100), (97, 89), (89, 97),
                (1021, 13), (13, 1021), (256, 1000), (480, 360), (720, 180), (1, 1000),
                (1000, 1), (331, 337), (128, 1024), (600, 999), (2 * 499, 1024)]


@pytest.mark.parametrize("eb", [4, 8])
def test_transpose_small_shapes(eb):
    for (M, N) in SMALL_SHAPES:
        a = seeded.matrix_np(M, N, eb)
        t = to_dev(a, eb)
        out = ipt.transpose_(t, M, N)
        assert tuple(out.shape) == (N, M)
        ref = oracle.transpose_inplace(a.copy(), M, N)
        assert np.array_equal(to_np(t, eb), ref), (M, N, eb)


@pytest.mark.parametrize("eb", [1, 2, 16])
def test_transpose_other_elem_sizes(eb):
    for (M, N) in [(5, 3), (64, 48), (97, 89), (300, 120)]:
        a = gen(M * N, eb)
        t = to_dev(a, eb)
        ipt.transpose_(t, M, N, elem_bytes=eb)
        ref = oracle_P(a.copy(), 1, M, N, 1, eb)
        assert np.array_equal(to_np(t, eb), ref), (M, N, eb)


def test_plan_independence_all_tilings():
    """Every valid (m, n) gives identical bytes."""
    M, N = 120, 72
    a = seeded.matrix_np(M, N, 4)
    ref = oracle.transpose_inplace(a.copy(), M, N)
    divs = lambda x: [d for d in range(1, x + 1) if x % d == 0]
    for m in divs(M):
        for n in divs(N):
            p = ipt.plan(M, N, 4, m=m, n=n)
            t = to_dev(a, 4)
            ipt.transpose_(t, M, N, plan_=p)
            assert np.array_equal(to_np(t, 4), ref), (m, n)


def test_random_bits_and_double_transpose():
    for eb in (4, 8):
        M, N = 777, 360
        a = seeded.random_bits_np(M * N, eb, seed=9)
        t = to_dev(a, eb)
        ipt.transpose_(t, M, N)
        assert np.array_equal(to_np(t, eb), a.reshape(M, N).T.reshape(-1))
        ipt.transpose_(t, N, M)
        assert np.array_equal(to_np(t, eb), a)


def test_user_workspace_and_events():
    M, N = 1800, 720
    p = ipt.plan(M, N, 4, device=0)
    ws = torch.empty(ipt.workspace_bytes(p, 1), dtype=torch.uint8, device="cuda")
    evs = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
    for e in evs:
        e.record()
    a = seeded.matrix_np(M, N, 4)
    t = to_dev(a, 4)
    ipt.transpose_(t, M, N, plan_=p, workspace=ws, events=evs)
    torch.cuda.synchronize()
    assert np.array_equal(to_np(t, 4), oracle.transpose_inplace(a.copy(), M, N))
    assert all(evs[i].elapsed_time(evs[i + 1]) >= 0 for i in range(3))


def test_workspace_too_small_rejected():
    p = ipt.plan(1800, 720, 4, device=0)
    ws = torch.empty(16, dtype=torch.uint8, device="cuda")
    t = torch.zeros(1800 * 720, dtype=torch.int32, device="cuda")
    with pytest.raises(ipt.IptError, match="NO_MEMORY"):
        ipt.transpose_(t, 1800, 720, plan_=p, workspace=ws)


def test_cpu_tensor_refused():
    with pytest.raises(ipt.IptError):
        ipt.transpose_(torch.zeros(12, dtype=torch.int32), 3, 4)


def test_native_kernels_launched():
    before = ipt.kernel_launch_count()
    t = to_dev(seeded.matrix_np(720, 1800, 4), 4)
    ipt.transpose_(t, 720, 1800)
    torch.cuda.synchronize()
    assert ipt.kernel_launch_count() - before == ipt.plan(720, 1800, 4, device=0).n_stages


# -------------------------------------------------------------------------------- batch
def test_batched_with_stride():
    count, M, N = 7, 360, 96
    stride = M * N + 40
    a = seeded.values_np(np.arange(count * stride), 4)
    t = to_dev(a, 4)
    ipt.transpose_batched_(t, count, M, N, stride_elems=stride)
    ref = a.copy()
    for i in range(count):
        seg = ref[i * stride: i * stride + M * N]
        oracle.transpose_inplace(seg, M, N)
    assert np.array_equal(to_np(t, 4), ref)


def test_batched_plan_events():
    count, M, N = 5, 720, 1800
    p = ipt.plan(M, N, 4, device=0)
    evs = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
    for e in evs:
        e.record()
    a = seeded.values_np(np.arange(count * M * N), 4)
    t = to_dev(a, 4)
    ipt.transpose_batched_(t, count, M, N, plan_=p, events=evs)
    torch.cuda.synchronize()
    ref = a.copy()
    for i in range(count):
        oracle.transpose_inplace(ref[i * M * N:(i + 1) * M * N], M, N)
    assert np.array_equal(to_np(t, 4), ref)
    assert all(evs[i].elapsed_time(evs[i + 1]) >= 0 for i in range(3))


# ------------------------------------------------------------------ race stress (T6)
def test_stress_varied_occupancy(monkeypatch):
    """Repeat with different persistent-grid sizes and walker shapes so chains
    interleave differently; every run must be bit-exact."""
    M, N = 1200, 1800
    a = seeded.matrix_np(M, N, 4)
    ref = oracle.transpose_inplace(a.copy(), M, N)
    rnd = random.Random(1)
    for it in range(40):
        monkeypatch.setenv("IPT_CYC_BLOCKS_PER_SM", str(rnd.choice([1, 2, 3, 8])))
        monkeypatch.setenv("IPT_CYC_REFRESH", str(rnd.choice([0, 1])))
        m, n = rnd.choice([(120, 120), (60, 90), (40, 200), (300, 24), (8, 1800)])
        t = to_dev(a, 4)
        ipt.transpose_(t, M, N, plan_=ipt.plan(M, N, 4, m=m, n=n))
        assert np.array_equal(to_np(t, 4), ref), (it, m, n)


# ------------------------------------------------------- full BASELINE sizes (sampled)
def _check_full(t, M, N, eb, t_idx=0, nsamp=20000, seed=0):
    """(a) sampled outputs via the oracle's Eq. (1), one by one; (b) every element via the
    definition with torch index arithmetic (on the device)."""
    rnd = random.Random(seed)
    n = M * N
    ks = [rnd.randrange(n) for _ in range(nsamp)] + [0, 1, n - 2, n - 1]
    dst = torch.tensor([oracle.eq1_dest(k, M, N) for k in ks], device=t.device)
    exp = seeded.values_torch_sample(torch.tensor(ks, device=t.device) + t_idx * n, eb)
    got = t.view(-1)[:n][dst]
    assert torch.equal(got, exp.to(t.dtype))
    # whole array, in chunks: position p = j*M + i holds v(i*N + j)
    CH = 1 << 27
    for p0 in range(0, n, CH):
        p = torch.arange(p0, min(n, p0 + CH), device=t.device, dtype=torch.int64)
        j, i = p // M, p % M
        exp = seeded.values_torch_sample(i * N + j + t_idx * n, eb)
        assert torch.equal(t.view(-1)[p0:p0 + p.numel()], exp.to(t.dtype)), p0


@pytest.mark.parametrize("M,N,eb", [(1800, 7200, 4), (7200, 1800, 4)])
def test_full_config_C1_vs_oracle(M, N, eb):
    a = seeded.matrix_np(M, N, eb)
    t = to_dev(a, eb)
    ipt.transpose_(t, M, N)
    assert np.array_equal(to_np(t, eb), oracle.transpose_inplace(a.copy(), M, N))


SWEEP_FULL = [(7200, 18000), (18000, 7200), (16384, 16384), (12800, 15000), (19200, 10000),
              (9998, 12288), (14803, 8192), (20000, 20000), (5100, 2500), (4000, 3200),
              (3300, 3900), (2500, 5100), (1021, 4093), (19997, 1024)]


@pytest.mark.parametrize("M,N", SWEEP_FULL)
def test_full_config_sweep_f32(M, N):
    t = torch.empty(M * N, dtype=torch.int32, device="cuda")
    seeded.fill_device_(t, M, N, 4)
    ipt.transpose_(t, M, N)
    _check_full(t, M, N, 4)


def test_full_config_C3_skinny():
    M, N = 1_000_000, 256
    t = torch.empty(M * N, dtype=torch.int32, device="cuda")
    seeded.fill_device_(t, M, N, 4)
    ipt.transpose_(t, M, N)
    _check_full(t, M, N, 4)


def test_full_config_C4_large_f64():
    M, N = 20000, 30000
    t = torch.empty(M * N, dtype=torch.int64, device="cuda")
    seeded.fill_device_(t, M, N, 8)
    ipt.transpose_(t, M, N)
    _check_full(t, M, N, 8)
    del t
    torch.cuda.empty_cache()


def test_full_config_C5_batch_sampled():
    count, M, N = 64, 4096, 3000      # one GPU's shard at G = 8
    t = torch.empty(count * M * N, dtype=torch.int32, device="cuda")
    seeded.fill_device_(t, M, N, 4, count=count)
    ipt.transpose_batched_(t, count, M, N)
    for ti in (0, 1, count // 2, count - 1):
        _check_full(t[ti * M * N:(ti + 1) * M * N], M, N, 4, t_idx=ti, nsamp=2000, seed=ti)
    del t
    torch.cuda.empty_cache()


def test_prime_both_scalar_fallback():
    M, N = 10007, 19997
    t = torch.empty(M * N, dtype=torch.int32, device="cuda")
    seeded.fill_device_(t, M, N, 4)
    ipt.transpose_(t, M, N)
    _check_full(t, M, N, 4, nsamp=5000)


# ------------------------------------------------------ host-delegated scheme (Sec. 6)
@pytest.mark.parametrize("queues", [1, 3, 8])
def test_transpose_host_queues(queues):
    for (M, N) in [(1800, 7200), (360, 1000), (97, 89)]:
        a = seeded.matrix_np(M, N, 4)
        h = torch.from_numpy(a.view(np.int32).copy()).pin_memory()
        out = ipt.transpose_host_(h, M, N, queues=queues)
        assert tuple(out.shape) == (N, M)
        ref = oracle.transpose_inplace(a.copy(), M, N)
        assert np.array_equal(h.numpy().view(np.uint32), ref), (M, N, queues)


# ------------------------------------------------- cluster-split tiles (> 227 KB)
@pytest.mark.parametrize("eb,batch,A,B", [(4, 3, 512, 512), (4, 2, 7200 // 4, 60), (4, 5, 640, 600),
                                          (8, 3, 400, 400), (16, 2, 256, 256), (4, 7, 960, 400)])
@pytest.mark.parametrize("split", ["0", "1"])
def test_ipt_010_cluster_tiles(monkeypatch, split, eb, batch, A, B):
    """Tiles larger than one CTA's shared memory are split over a thread-block cluster
    (one barrier.cluster per tile); bit-exact vs the oracle."""
    monkeypatch.setenv("IPT_TILE_GROUP_SPLIT", split)   # cluster vs group split
    a = gen(batch * A * B, eb)
    t = to_dev(a, eb)
    ipt.ipt_010_(t, batch, A, B, elem_bytes=eb)
    assert np.array_equal(to_np(t, eb), oracle_P(a.copy(), batch, A, B, 1, eb)), (eb, batch, A, B)


# ---------------------------------------- unaligned super-elements (S % 16 != 0)
@pytest.mark.parametrize("batch,A,B,s,eb", [(1, 61, 47, 131, 4), (3, 20, 30, 17, 4), (2, 9, 11, 4999, 4),
                                            (4, 33, 31, 65, 4), (1, 50, 70, 63, 8), (2, 40, 44, 1001, 8),
                                            (1, 256, 131, 131, 4), (1, 97, 103, 127, 4),
                                            (2, 30, 41, 509, 4), (1, 23, 29, 1021, 4)])
@pytest.mark.parametrize("seg", ["0", "2"])
def test_ipt_100_unaligned_realigning_walker(monkeypatch, seg, batch, A, B, s, eb):
    """4-byte-granular super-elements whose start phases differ mod 16 B: the realigning
    flag walker (IPT_CYC_SEG=0: covering 16-B loads, shared-memory carry, partial stores)
    and the segmented unaligned walker (2: covering loads, lane funnel shifts, edge words;
    one chunk up to 508 words, 508-word chunks beyond)."""
    monkeypatch.setenv("IPT_CYC_SEG", seg)
    a = gen(batch * A * B * s, eb)
    t = to_dev(a, eb)
    ipt.ipt_100_(t, batch, A, B, s)
    assert np.array_equal(to_np(t, eb), oracle.permute_inplace(a.copy(), batch, A, B, s))


# words per unit at each walker-shape boundary of the segmented unaligned walker (G lanes x R
# vectors, R = 1..6, the smallest that covers a chunk; 764 words = one full 32 x 6 walker,
# 765+ two or more balanced chunks), f32 and the f64 equivalents
UA_WORDS = [5, 29, 61, 93, 127, 157, 189, 253, 317, 381, 509, 764, 765, 766, 1021, 1529, 2301]


@pytest.mark.parametrize("s", UA_WORDS)
def test_ipt_100_unaligned_segmented_walker_shapes(monkeypatch, s):
    """Every walker shape of cycle_seg_ua (and the chunk split beyond one walker) against
    the oracle, on a small permutation with long and short cycles."""
    monkeypatch.setenv("IPT_CYC_SEG", "2")
    A, B = (13, 7) if s > 700 else (37, 29)
    a = gen(A * B * s, 4)
    t = to_dev(a, 4)
    ipt.ipt_100_(t, 1, A, B, s)
    assert np.array_equal(to_np(t, 4), oracle.permute_inplace(a.copy(), 1, A, B, s)), s


@pytest.mark.parametrize("seg", ["0", "2"])
@pytest.mark.parametrize("off,batch,A,B,s", [(1, 1, 61, 47, 32), (3, 2, 30, 20, 64), (2, 1, 40, 31, 7)])
def test_ipt_100_misaligned_base(monkeypatch, seg, off, batch, A, B, s):
    """Data starting 4-12 bytes past a 16-byte boundary (16-byte multiple super-elements at
    shifted phases): the unaligned walkers, bit-exact, neighbours untouched."""
    monkeypatch.setenv("IPT_CYC_SEG", seg)
    n = batch * A * B * s
    a = gen(n + 8, 4)
    t = to_dev(a, 4)
    ipt.ipt_100_(t[off:off + n], batch, A, B, s)
    got = to_np(t, 4)
    assert np.array_equal(got[off:off + n], oracle.permute_inplace(a[off:off + n].copy(), batch, A, B, s))
    assert np.array_equal(got[:off], a[:off]) and np.array_equal(got[off + n:], a[off + n:])


@pytest.mark.parametrize("eb,batch,A,B", [(4, 2, 4999, 32), (4, 3, 1999, 31), (8, 2, 3001, 17),
                                          (2, 2, 997, 301), (4, 1, 9998, 24)])
def test_ipt_010_generic_cluster_tiles(eb, batch, A, B):
    """Element-path tiles larger than one CTA: uneven row slices over a cluster."""
    a = gen(batch * A * B, eb)
    t = to_dev(a, eb)
    ipt.ipt_010_(t, batch, A, B, elem_bytes=eb)
    assert np.array_equal(to_np(t, eb), oracle_P(a.copy(), batch, A, B, 1, eb)), (eb, batch, A, B)


@pytest.mark.parametrize("eb,batch,A,B", [(4, 2, 32, 9998), (4, 3, 24, 4999), (8, 2, 17, 3001), (1, 2, 7, 40001)])
def test_ipt_010_generic_cluster_column_split(monkeypatch, eb, batch, A, B):
    """Few long rows: each cluster CTA owns a column range, writes whole output rows."""
    monkeypatch.setenv("IPT_TILE_COLSPLIT", "1")
    a = gen(batch * A * B, eb)
    t = to_dev(a, eb)
    ipt.ipt_010_(t, batch, A, B, elem_bytes=eb)
    assert np.array_equal(to_np(t, eb), oracle_P(a.copy(), batch, A, B, 1, eb)), (eb, batch, A, B)


# ------------------------------------------------ 4-stage baseline (NEXT-2)
@pytest.mark.parametrize("M,N,m,n", [(120, 72, 8, 6), (360, 1000, 40, 25), (97, 64, 97, 8),
                                     (1800, 720, 0, 0), (256, 256, 16, 16)])
def test_4stage_matches_oracle(M, N, m, n):
    a = seeded.matrix_np(M, N, 4)
    t = to_dev(a, 4)
    ipt.transpose_4stage_(t, M, N, m, n)
    ref = oracle.transpose_inplace(a.copy(), M, N)
    assert np.array_equal(to_np(t, 4), ref)
    if m and n:   # and stage by stage equal to the oracle's own 4-stage composition
        assert np.array_equal(ref, oracle.transpose_4stage(a.copy(), M, N, m, n))


# ---------------------------------------- layout marshaling AoS/SoA <-> ASTA (NEXT-3)
@pytest.mark.parametrize("M,N,m", [(1000, 256, 100), (4096, 64, 32), (999, 7, 37), (1_000_000, 256, 64)])
def test_layout_marshaling(M, N, m):
    """AoS (M x N) -> ASTA (M/m x N x m) = 010!; SoA (N x M) -> ASTA = 100!; and
    their inverses.  K-Means descriptor shape included (1e6 x 256)."""
    Mp = M // m
    a = seeded.matrix_np(M, N, 4)
    asta = a.reshape(Mp, m, N).transpose(0, 2, 1).reshape(-1)
    t = to_dev(a, 4)
    ipt.aos_to_asta_(t, M, N, m)
    if M * N <= 4_000_000:
        assert np.array_equal(to_np(t, 4), oracle.permute_inplace(a.copy(), Mp, m, N, 1))
    assert np.array_equal(to_np(t, 4), asta)
    ipt.asta_to_aos_(t, M, N, m)
    assert np.array_equal(to_np(t, 4), a)
    soa = a.reshape(M, N).T.reshape(-1).copy()
    t = to_dev(soa, 4)
    ipt.soa_to_asta_(t, M, N, m)
    assert np.array_equal(to_np(t, 4), asta)
    ipt.asta_to_soa_(t, M, N, m)
    assert np.array_equal(to_np(t, 4), soa)


@pytest.mark.parametrize("eb,batch,A,B", [(4, 2, 1800, 240), (8, 3, 902, 100), (4, 2, 3004, 128)])
@pytest.mark.parametrize("split", ["0", "1"])
def test_ipt_010_cluster_uneven_slices(monkeypatch, split, eb, batch, A, B):
    """16-byte cluster path with row slices of unequal length (multiples of V rows)."""
    monkeypatch.setenv("IPT_TILE_GROUP_SPLIT", split)   # cluster vs group split
    a = gen(batch * A * B, eb)
    t = to_dev(a, eb)
    ipt.ipt_010_(t, batch, A, B, elem_bytes=eb)
    assert np.array_equal(to_np(t, eb), oracle_P(a.copy(), batch, A, B, 1, eb)), (eb, batch, A, B)


@pytest.mark.parametrize("eb,batch,A,B", [(4, 2, 7200, 120), (4, 1, 9998, 64)])
def test_ipt_010_cluster16(monkeypatch, eb, batch, A, B):
    """Non-portable 16-CTA clusters (panels up to 16 x 227 KB)."""
    monkeypatch.setenv("IPT_TILE_GROUP_SPLIT", "0")
    a = gen(batch * A * B, eb)
    t = to_dev(a, eb)
    ipt.ipt_010_(t, batch, A, B, elem_bytes=eb)
    assert np.array_equal(to_np(t, eb), oracle_P(a.copy(), batch, A, B, 1, eb)), (eb, batch, A, B)


@pytest.mark.parametrize("eb,batch,A,B", [(4, 2, 120, 7200), (8, 2, 64, 2000), (16, 2, 32, 3000),
                                          (4, 3, 256, 1000)])
@pytest.mark.parametrize("split", ["0", "1"])
def test_ipt_010_cluster_column_split_fast(monkeypatch, split, eb, batch, A, B):
    """16-byte cluster path, fewer rows than columns: each CTA owns a range of 16-byte
    columns and writes whole contiguous output rows."""
    monkeypatch.setenv("IPT_TILE_GROUP_SPLIT", split)   # cluster vs group split
    a = gen(batch * A * B, eb)
    t = to_dev(a, eb)
    ipt.ipt_010_(t, batch, A, B, elem_bytes=eb)
    assert np.array_equal(to_np(t, eb), oracle_P(a.copy(), batch, A, B, 1, eb)), (eb, batch, A, B)


@pytest.mark.parametrize("segsh", [0, 2, 5])
def test_ipt_100_fetch_segments(monkeypatch, segsh):
    """Start units handed out as 1/2^segsh of a flag word (small stages) -- bit-exact."""
    monkeypatch.setenv("IPT_CYC_SEGSH", str(segsh))
    for (batch, A, B, s) in [(1, 61, 47, 8), (3, 17, 19, 131), (1, 1800, 15, 480), (2, 33, 20, 12)]:
        a = gen(batch * A * B * s, 4)
        t = to_dev(a, 4)
        ipt.ipt_100_(t, batch, A, B, s)
        assert np.array_equal(to_np(t, 4), oracle.permute_inplace(a.copy(), batch, A, B, s)), (segsh, batch, A, B, s)


def test_transpose_host_async_two_streams():
    """Asynchronous host-delegated calls on two streams (overlapping PCIe directions)."""
    shapes = [(1800, 7200), (720, 1800), (97, 89), (4096, 300)]
    hs, refs = [], []
    for (M, N) in shapes:
        a = seeded.matrix_np(M, N, 4)
        hs.append(torch.from_numpy(a.view(np.int32).copy()).pin_memory())
        refs.append(oracle.transpose_inplace(a.copy(), M, N))
    sts = [torch.cuda.Stream(), torch.cuda.Stream()]
    for i, ((M, N), h) in enumerate(zip(shapes, hs)):
        ipt.transpose_host_async_(h, M, N, queues=3, stream=sts[i % 2])
    for s in sts:
        s.synchronize()
    for h, ref in zip(hs, refs):
        assert np.array_equal(h.numpy().view(np.uint32), ref)


@pytest.mark.parametrize("eb,batch,A,B", [(4, 5, 256, 200), (8, 4, 120, 200), (16, 3, 100, 120),
                                          (4, 3, 7200, 120), (4, 7, 1800, 160), (8, 2, 1000, 96)])
def test_ipt_010_streaming_slices(monkeypatch, eb, batch, A, B):
    """One CTA per SM (slices > 113 KB): write-out of tile t overlapped with the cp.async
    refill of tile t+1, group by group."""
    monkeypatch.setenv("IPT_TILE_GROUP_SPLIT", "0")
    a = gen(batch * A * B, eb)
    t = to_dev(a, eb)
    ipt.ipt_010_(t, batch, A, B, elem_bytes=eb)
    assert np.array_equal(to_np(t, eb), oracle_P(a.copy(), batch, A, B, 1, eb)), (eb, batch, A, B)


def test_plan_autotune_restores_data_and_is_used():
    M, N = 1800, 2400
    a = seeded.matrix_np(M, N, 4)
    t = to_dev(a, 4)
    p = ipt.plan_autotune(t, M, N, 4)
    assert np.array_equal(to_np(t, 4), a)               # data unchanged
    assert M % p.m == 0 and N % p.n == 0
    q = ipt.plan(M, N, 4, 0)                            # remembered for this device
    assert (q.m, q.n) == (p.m, p.n)
    ipt.transpose_(t, M, N)
    assert np.array_equal(to_np(t, 4), oracle.transpose_inplace(a.copy(), M, N))


def test_plan_autotune_batched_restores_data():
    count, M, N = 6, 360, 1200
    a = seeded.batch_np(count, M, N, 4)
    t = to_dev(a, 4)
    p = ipt.plan_autotune_batched(t, count, M, N, 4)
    assert np.array_equal(to_np(t, 4), a)
    ipt.transpose_batched_(t, count, M, N, plan_=p)
    ref = a.copy()
    for i in range(count):
        oracle.transpose_inplace(ref[i * M * N:(i + 1) * M * N], M, N)
    assert np.array_equal(to_np(t, 4), ref)


def test_idx64_path(monkeypatch):
    """64-bit index instantiations (used when a stage has >= 2^32 units) on medium shapes."""
    monkeypatch.setenv("IPT_CYC_IDX64", "1")
    for (M, N) in [(1800, 720), (97, 89), (1021, 130)]:
        for eb in (4, 8):
            a = seeded.matrix_np(M, N, eb)
            t = to_dev(a, eb)
            ipt.transpose_(t, M, N)
            assert np.array_equal(to_np(t, eb), oracle.transpose_inplace(a.copy(), M, N)), (M, N, eb)
    a = gen(2 * 40 * 30 * 131, 4)
    t = to_dev(a, 4)
    ipt.ipt_100_(t, 2, 40, 30, 131)                       # realigning walker, 64-bit
    assert np.array_equal(to_np(t, 4), oracle.permute_inplace(a.copy(), 2, 40, 30, 131))


def test_concurrent_streams_internal_workspace():
    """Calls on different streams use different internal workspaces and may overlap."""
    shapes = [(1800, 2400), (2400, 1800), (720, 1000), (97, 4093)]
    sts = [torch.cuda.Stream() for _ in shapes]
    ts, refs = [], []
    for (M, N) in shapes:
        a = seeded.matrix_np(M, N, 4)
        ts.append(to_dev(a, 4))
        refs.append(oracle.transpose_inplace(a.copy(), M, N))
    torch.cuda.synchronize()
    for rep in range(3):
        for (M, N), t, s in zip(shapes, ts, sts):
            a, b = (M, N) if rep % 2 == 0 else (N, M)
            ipt.transpose_(t, a, b, stream=s)
    torch.cuda.synchronize()
    for t, ref in zip(ts, refs):
        assert np.array_equal(to_np(t, 4), ref)


# ------------------------------------------ group-split tiles (co-resident CTA groups)
@pytest.mark.parametrize("eb,batch,A,B", [(4, 3, 120, 7200), (4, 2, 7200, 120), (4, 2, 60, 7200),
                                          (4, 3, 180, 7200), (8, 2, 400, 800), (16, 2, 300, 400),
                                          (4, 1, 1024, 1024), (4, 1, 128, 16384), (8, 1, 1000, 1000),
                                          (4, 5, 720, 720)])
def test_ipt_010_group_split(eb, batch, A, B):
    """Tiles split over a co-resident group of K CTAs (cooperative launch, software barrier
    per tile, double-buffered slices) -- including tiles beyond 16 x 227 KB clusters."""
    a = gen(batch * A * B, eb)
    t = to_dev(a, eb)
    ipt.ipt_010_(t, batch, A, B, elem_bytes=eb)
    assert np.array_equal(to_np(t, eb), oracle_P(a.copy(), batch, A, B, 1, eb)), (eb, batch, A, B)


@pytest.mark.parametrize("K", ["16", "17", "31", "37", "75", "148"])
@pytest.mark.parametrize("split", ["0", "1"])
def test_ipt_010_group_forced_sizes(monkeypatch, K, split):
    """Any group size (not only cluster sizes), uneven slices, both split directions."""
    monkeypatch.setenv("IPT_TILE_GROUP_K", K)
    monkeypatch.setenv("IPT_TILE_GROUP_COLSPLIT", split)
    batch, A, B = 7, 600, 1200
    a = gen(batch * A * B, 4)
    t = to_dev(a, 4)
    ipt.ipt_010_(t, batch, A, B)
    assert np.array_equal(to_np(t, 4), oracle_P(a.copy(), batch, A, B, 1, 4)), (K, split)


@pytest.mark.parametrize("tma", ["0", "1"])
@pytest.mark.parametrize("eb,batch,A,B,K", [(4, 3, 64, 16384, "0"), (4, 2, 384, 10000, "0"), (4, 3, 7200, 240, "0"),
                                            (4, 2, 10000, 384, "0"), (4, 2, 7200, 240, "71"), (4, 2, 240, 7200, "33"),
                                            (8, 2, 3000, 200, "0"), (8, 2, 200, 3000, "0"), (8, 1, 600, 6000, "0")])
def test_ipt_010_group_tma_slices(monkeypatch, tma, eb, batch, A, B, K):
    """Group tiles with slices fetched by 2-D TMA boxes: one or two column panels, several
    row boxes per panel, uneven row slices (the boxes read the neighbour's rows), f64 --
    and the same shapes on the cp.async path."""
    monkeypatch.setenv("IPT_TILE_GROUP_TMA", tma)
    monkeypatch.setenv("IPT_TILE_GROUP_K", K)
    a = gen(batch * A * B, eb)
    t = to_dev(a, eb)
    ipt.ipt_010_(t, batch, A, B, elem_bytes=eb)
    assert np.array_equal(to_np(t, eb), oracle_P(a.copy(), batch, A, B, 1, eb)), (tma, eb, batch, A, B, K)


@pytest.mark.parametrize("eb,batch,A,B,K", [(4, 2, 128, 9998, "0"), (4, 2, 9998, 128, "0"), (4, 1, 256, 14803, "0"),
                                            (4, 1, 14803, 256, "0"), (4, 2, 192, 9998, "0"), (4, 3, 601, 1203, "5"),
                                            (8, 2, 3001, 62, "0"), (8, 2, 62, 3001, "7"), (4, 2, 1998, 130, "9")])
def test_ipt_010_group_element_slices_forced_k(monkeypatch, eb, batch, A, B, K):
    """Element-path group tiles whose rows are 4- or 8-byte but not 16-byte aligned
    (row pieces at any 16-byte phase), forced group sizes, one or two slice buffers."""
    monkeypatch.setenv("IPT_TILE_GROUP_K", K)
    a = gen(batch * A * B, eb)
    t = to_dev(a, eb)
    ipt.ipt_010_(t, batch, A, B, elem_bytes=eb)
    assert np.array_equal(to_np(t, eb), oracle_P(a.copy(), batch, A, B, 1, eb)), (eb, batch, A, B, K)


@pytest.mark.parametrize("batch,A,B", [(10, 256, 15000), (10, 7200, 240), (20, 64, 16384),
                                       (5, 14803, 256), (6, 192, 9998)])
def test_group_split_stress_relaxed_arrivals(batch, A, B):
    """Stress of the group kernels' relaxed arrivals on the sweep's
    panel tiles at full size: 24 transposes back and forth, checked against torch after an
    odd count and against the original after an even one."""
    import torch
    t = torch.randint(-2**31, 2**31 - 1, (batch * A * B,), dtype=torch.int32, device="cuda")
    orig = t.clone()
    ref_t = orig.view(batch, A, B).transpose(1, 2).contiguous().view(-1)
    for rep in range(24):
        x, y = (A, B) if rep % 2 == 0 else (B, A)
        ipt.ipt_010_(t, batch, x, y)
        if rep == 10:
            torch.cuda.synchronize()
            assert torch.equal(t, ref_t), rep
    torch.cuda.synchronize()
    assert torch.equal(t, orig)


_CONCURRENT_GROUPS = r"""
import sys, torch
sys.path.insert(0, sys.argv[1])
import paper_conf_ppopp_sunggggh14_b200 as ipt
shapes = [(3, 120, 7200), (2, 7200, 120), (1, 1024, 1024), (4, 720, 720)]
sts = [torch.cuda.Stream() for _ in shapes]
ts = [torch.randint(0, 2**31 - 1, (b * A * B,), dtype=torch.int32, device="cuda") for (b, A, B) in shapes]
refs = [t.clone() for t in ts]
for rep in range(40):
    for (b, A, B), t, s in zip(shapes, ts, sts):
        x, y = (A, B) if rep % 2 == 0 else (B, A)
        ipt.ipt_010_(t, b, x, y, stream=s)
torch.cuda.synchronize()
assert all(torch.equal(t, r) for t, r in zip(ts, refs))
print("ok")
"""


def test_group_split_concurrent_streams():
    """Cooperative group-split launches on four streams at once (each with its own
    counters) complete and are exact; run in a child with a deadline so a co-residency
    failure cannot hang the suite."""
    import subprocess, sys, os
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, "-c", _CONCURRENT_GROUPS, root], capture_output=True,
                       text=True, timeout=180)
    assert r.returncode == 0 and "ok" in r.stdout, r.stderr[-2000:]


@pytest.mark.parametrize("eb,batch,A,B", [(4, 2, 64, 9998), (4, 2, 9998, 64), (4, 2, 113, 8192),
                                          (4, 1, 14803, 32), (4, 1, 14803, 128), (8, 2, 3001, 61),
                                          (8, 2, 61, 3001), (4, 3, 301, 257), (4, 2, 7, 40001),
                                          (4, 3, 1999, 31), (8, 1, 2999, 257), (4, 2, 9998, 192),
                                          (4, 1, 14803, 256), (8, 2, 4999, 96), (4, 3, 1001, 48)])
def test_ipt_010_group_split_element_path(eb, batch, A, B):
    """Element-path tiles (sides not multiples of 16/elem) over a CTA group: row pieces
    fetched at their global 16-byte phase and realigned in registers on write-out."""
    a = gen(batch * A * B, eb)
    t = to_dev(a, eb)
    ipt.ipt_010_(t, batch, A, B, elem_bytes=eb)
    assert np.array_equal(to_np(t, eb), oracle_P(a.copy(), batch, A, B, 1, eb)), (eb, batch, A, B)


@pytest.mark.parametrize("K", ["2", "5", "37", "148"])
@pytest.mark.parametrize("split", ["0", "1"])
def test_ipt_010_group_element_forced_sizes(monkeypatch, K, split):
    monkeypatch.setenv("IPT_TILE_GROUP_K", K)
    monkeypatch.setenv("IPT_TILE_GROUP_COLSPLIT", split)
    batch, A, B = 5, 601, 1203
    a = gen(batch * A * B, 4)
    t = to_dev(a, 4)
    ipt.ipt_010_(t, batch, A, B)
    assert np.array_equal(to_np(t, 4), oracle_P(a.copy(), batch, A, B, 1, 4)), (K, split)


@pytest.mark.parametrize("eb,batch,A,B,gr", [(4, 5, 601, 1203, "0"), (4, 2, 1279, 6353, "0"), (4, 2, 1279, 6353, "8"),
                                             (4, 3, 2362, 1453, "0"), (8, 2, 1201, 3001, "0"), (8, 2, 3001, 1201, "3"),
                                             (4, 3, 301, 257, "2"), (4, 2, 1999, 310, "0"), (4, 1, 9797, 103, "0")])
def test_ipt_010_group_element_grid2d(monkeypatch, eb, batch, A, B, gr):
    """Element-path group tiles over a 2-D slice grid (gr row bands x gc column pieces, the
    CTA's piece at its own 16-byte phase): forced for every shape (IPT_TILE_GROUP_COLSPLIT=2),
    uneven bands and pieces, f64, the sweep's 1279 x 6353 and 2362 x 1453 tiles."""
    monkeypatch.setenv("IPT_TILE_GROUP_COLSPLIT", "2")
    monkeypatch.setenv("IPT_TILE_GROUP_GR", gr)
    a = gen(batch * A * B, eb)
    t = to_dev(a, eb)
    ipt.ipt_010_(t, batch, A, B, elem_bytes=eb)
    assert np.array_equal(to_np(t, eb), oracle_P(a.copy(), batch, A, B, 1, eb)), (eb, batch, A, B, gr)


def test_ipt_010_group_element_misaligned_base():
    """A 16-byte-vectorisable tile at a base that is only 4-byte aligned takes the
    element-path group kernel (any phase)."""
    batch, A, B = 3, 400, 800
    a = gen(batch * A * B + 1, 4)
    t = to_dev(a, 4)
    ipt.ipt_010_(t[1:], batch, A, B)
    ref = a.copy()
    ref[1:] = oracle_P(a[1:].copy(), batch, A, B, 1, 4)
    assert np.array_equal(to_np(t, 4), ref)


# ------------------------------------------- square items: symmetric swaps
SQ_SIDES = [2, 3, 7, 15, 16, 17, 63, 64, 65, 100, 127, 128, 129, 255, 256, 257, 300, 1021]


@pytest.mark.parametrize("eb", [1, 2, 4, 8, 16])
@pytest.mark.parametrize("path", ["auto", "vec", "elem", "elem_pf32", "elem_pf64", "elem_plain", "tb512",
                                  "tb512nt512", "swz", "swz512", "noswz"])
def test_square_swap_sides(monkeypatch, eb, path):
    """ipt_010 on square items through the swap kernel (register-staged 16-byte path,
    element path): every side spans ragged block edges (g not a multiple of the
    block) and, for g % (16/b) != 0, the element path; batches fold several items into
    one launch (rows of a ragged last block belong to the next item)."""
    monkeypatch.setenv("IPT_SQ_FORCE", "1")
    if path.startswith("elem"):
        monkeypatch.setenv("IPT_SQ_ELEM", "1")
    if path.startswith("elem_p"):   # the element path's prefetching variants / the plain kernel
        monkeypatch.setenv("IPT_SQ_ELEM_PF", {"elem_pf32": "32", "elem_pf64": "64", "elem_plain": "0"}[path])
    if path.startswith("tb512"):
        monkeypatch.setenv("IPT_SQ_TB", "512")
    if path == "tb512nt512":
        monkeypatch.setenv("IPT_SQ_NT", "512")
    if path.startswith("swz"):
        monkeypatch.setenv("IPT_SQ_SWZ", "1")
        monkeypatch.setenv("IPT_SQ_TB", "512" if path == "swz512" else "256")
    if path == "noswz":
        monkeypatch.setenv("IPT_SQ_SWZ", "0")
    rnd = random.Random(eb * 7 + len(path))
    for g in SQ_SIDES:
        batch = rnd.choice([1, 1, 2, 3]) if g > 256 else rnd.choice([1, 2, 5, 17])
        a = gen(batch * g * g, eb)
        t = to_dev(a, eb)
        ipt.ipt_010_(t, batch, g, g, elem_bytes=eb)
        ref = oracle_P(a.copy(), batch, g, g, 1, eb)
        assert np.array_equal(to_np(t, eb), ref), (batch, g, eb, path)


def test_square_swap_misaligned_base(monkeypatch):
    """A base 4 bytes off 16-byte alignment takes the element path; neighbours untouched."""
    monkeypatch.setenv("IPT_SQ_FORCE", "1")
    batch, g = 3, 200
    a = gen(batch * g * g + 3, 4)
    t = to_dev(a, 4)
    ipt.ipt_010_(t[1:1 + batch * g * g], batch, g, g)
    got = to_np(t, 4)
    assert got[0] == a.view(np.uint32)[0] and np.array_equal(got[-2:], a.view(np.uint32)[-2:])
    ref = oracle_P(a[1:1 + batch * g * g].copy(), batch, g, g, 1, 4)
    assert np.array_equal(got[1:1 + batch * g * g], ref)


@pytest.mark.parametrize("M,eb", [(2, 4), (5, 8), (64, 4), (1000, 4), (1024, 8), (2049, 4),
                                  (4096, 4), (997, 8)])
def test_square_matrix_single_pass_plan(monkeypatch, M, eb):
    """M == N plans run one stage (square_swap; forced for the small sides, which the
    planner may keep on chip) and match the oracle bit for bit."""
    monkeypatch.setenv("IPT_SQ_FORCE", "1")
    p = ipt.plan(M, M, eb, 0, m=M, n=M)
    assert p.n_stages == 1 and ipt.VARIANTS[p.variant[1]] == "square_swap", p.as_dict()
    if M * M * eb > (1 << 22):
        q = ipt.plan(M, M, eb, 0)
        assert (q.m, q.n, list(q.variant)) == (p.m, p.n, list(p.variant))
    a = seeded.matrix_np(M, M, eb)
    t = to_dev(a, eb)
    before = ipt.kernel_launch_count()
    ipt.transpose_(t, M, M, plan_=p)
    torch.cuda.synchronize()
    assert ipt.kernel_launch_count() - before == 1
    assert np.array_equal(to_np(t, eb), oracle.transpose_inplace(a.copy(), M, M)), (M, eb)


def test_square_batched_with_stride():
    """A batch of square matrices with a gap between them: gaps untouched."""
    count, M, gap = 5, 384, 40
    stride = M * M + gap
    a = gen(count * stride, 4)
    t = to_dev(a, 4)
    ipt.transpose_batched_(t, count, M, M, stride_elems=stride)
    got = to_np(t, 4)
    src = a.view(np.uint32)
    for k in range(count):
        blk = src[k * stride:k * stride + M * M].copy()
        assert np.array_equal(got[k * stride:k * stride + M * M],
                              oracle.transpose_inplace(blk, M, M)), k
        assert np.array_equal(got[k * stride + M * M:(k + 1) * stride],
                              src[k * stride + M * M:(k + 1) * stride])


@pytest.mark.parametrize("M,N,m", [(7200, 1800, 1800), (1800, 7200, 1800), (4096, 4096, 1024),
                                   (3000, 6000, 1000), (640, 960, 320)])
def test_square_tiles_in_3stage_plan(monkeypatch, M, N, m):
    """Plans with square stage-2 tiles m = n of any size (up to 13 MB here) run stage 2
    with the swap kernel inside the 3-stage method."""
    monkeypatch.setenv("IPT_SQ_FORCE", "1")
    p = ipt.plan(M, N, 4, 0, m=m, n=m)
    assert ipt.VARIANTS[p.variant[1]] == "square_swap", p.as_dict()
    a = seeded.matrix_np(M, N, 4)
    t = to_dev(a, 4)
    ipt.transpose_(t, M, N, plan_=p)
    assert np.array_equal(to_np(t, 4), oracle.transpose_inplace(a.copy(), M, N)), (M, N, m)


def test_square_host_path():
    """The host-delegated scheme (Sec. 6) on a square matrix (single-pass plan)."""
    M = 1536
    a = seeded.matrix_np(M, M, 4)
    h = torch.from_numpy(a.view(np.int32).copy()).pin_memory()
    ipt.transpose_host_(h, M, M, queues=2)
    assert np.array_equal(h.numpy().view(np.uint32), oracle.transpose_inplace(a.copy(), M, M))


def test_square_swap_strided_batch(monkeypatch):
    """Outer items at a stride (a gap after every item) -- gaps untouched."""
    count, M, gap = 4, 1000, 4 * 7
    stride = M * M + gap
    a = gen(count * stride, 4)
    t = to_dev(a, 4)
    ipt.transpose_batched_(t, count, M, M, stride_elems=stride)
    got = to_np(t, 4)
    src = a.view(np.uint32)
    for k in range(count):
        blk = src[k * stride:k * stride + M * M].copy()
        assert np.array_equal(got[k * stride:k * stride + M * M], oracle.transpose_inplace(blk, M, M)), k
        assert np.array_equal(got[k * stride + M * M:(k + 1) * stride], src[k * stride + M * M:(k + 1) * stride])


@pytest.mark.parametrize("M,N,m,n", [(1800, 7200, 1800, 180), (7200, 1800, 144, 1800),
                                     (1800, 7200, 1800, 1800), (360, 1000, 8, 1000),
                                     (4096, 3000, 128, 120)])
def test_cycle_seg_full_plans(monkeypatch, M, N, m, n):
    """Segmented cycle following inside full 2/3-stage plans (configs[0] shapes) vs the
    oracle; and the batched form (items x segments x chunks walkers)."""
    monkeypatch.setenv("IPT_CYC_SEG", "2")
    p = ipt.plan(M, N, 4, 0, m=m, n=n)
    a = seeded.matrix_np(M, N, 4)
    t = to_dev(a, 4)
    ipt.transpose_(t, M, N, plan_=p)
    assert np.array_equal(to_np(t, 4), oracle.transpose_inplace(a.copy(), M, N)), (M, N, m, n)


@pytest.mark.parametrize("reset", ["1", "0"])
def test_cycle_seg_batched_and_chunked(monkeypatch, reset):
    """Several items and super-elements larger than one walker (chunks), 8/16-byte units;
    self-resetting barrier counters (reused launch after launch on one stream) or a
    memset of the workspace counters per launch."""
    monkeypatch.setenv("IPT_CYC_SEG", "2")
    monkeypatch.setenv("IPT_SEG_RESET", reset)
    for (batch, A, B, s, eb) in [(3, 40, 56, 600, 4), (5, 17, 31, 64, 8), (2, 100, 3, 2, 16),
                                 (7, 64, 64, 32, 4), (1, 997, 13, 4, 4)]:
        a = gen(batch * A * B * s, eb)
        t = to_dev(a, eb)
        ipt.ipt_100_(t, batch, A, B, s, elem_bytes=eb)
        assert np.array_equal(to_np(t, eb), oracle_P(a.copy(), batch, A, B, s, eb)), (batch, A, B, s, eb)


def test_graph_capture_of_a_plan(monkeypatch):
    """A full transposition captured into a CUDA graph and replayed (segment plans are
    built outside capture; a first use inside capture falls back to the flag kernel)."""
    M, N = 1800, 7200
    a = seeded.matrix_np(M, N, 4)
    t = to_dev(a, 4)
    p1, p2 = ipt.plan(M, N, 4, 0), ipt.plan(N, M, 4, 0)
    s = torch.cuda.Stream()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.stream(s):
        ipt.transpose_(t, M, N, plan_=p1, stream=s)      # warm-up: builds cached state
        ipt.transpose_(t, N, M, plan_=p2, stream=s)
    torch.cuda.synchronize()
    with torch.cuda.graph(g, stream=s):
        ipt.transpose_(t, M, N, plan_=p1, stream=s)
    g.replay()
    torch.cuda.synchronize()
    assert np.array_equal(to_np(t, 4), oracle.transpose_inplace(a.copy(), M, N))


@pytest.mark.parametrize("M,N,eb", [(7200, 18000, 4), (18000, 7200, 4), (9998, 12288, 4),
                                    (14803, 8192, 4), (16384, 16384, 4), (1800, 7200, 4),
                                    (20000, 30000, 8)])
def test_bench_launch_configuration_autotuned(M, N, eb):
    """The bench's launch configuration: ipt_plan_autotune (4 candidates, as bench.py) runs
    every candidate plan forward and the model plan back -- the data must come back
    unchanged, bit for bit -- then the tuned plan (what the timed region launches, both
    orientations) is checked on oracle samples and on every element by the definition."""
    dt = torch.int32 if eb == 4 else torch.int64
    t = torch.empty(M * N, dtype=dt, device="cuda")
    seeded.fill_device_(t, M, N, eb)
    p = ipt.plan_autotune(t, M, N, 4)
    ref = torch.empty_like(t)
    seeded.fill_device_(ref, M, N, eb)
    assert torch.equal(t, ref), "autotune must leave the data unchanged"
    del ref
    ipt.transpose_(t, M, N, plan_=p)
    _check_full(t, M, N, eb, nsamp=3000)
    q = ipt.plan_autotune(t, N, M, 4)          # the reverse orientation (next bench step)
    ipt.transpose_(t, N, M, plan_=q)
    ref = torch.empty_like(t)
    seeded.fill_device_(ref, M, N, eb)
    assert torch.equal(t, ref), (p.as_dict(), q.as_dict())
    del t, ref
    torch.cuda.empty_cache()


def test_full_square_f64_single_pass():
    """A 3.2 GB square (20000^2 float64, > 2^31 bytes): the single swap pass, checked on
    oracle samples and on every element by the definition."""
    M = 20000
    p = ipt.plan(M, M, 8, 0)
    assert p.n_stages == 1 and ipt.VARIANTS[p.variant[1]] == "square_swap"
    t = torch.empty(M * M, dtype=torch.int64, device="cuda")
    seeded.fill_device_(t, M, M, 8)
    ipt.transpose_(t, M, M)
    _check_full(t, M, M, 8, nsamp=3000)
    del t
    torch.cuda.empty_cache()


def test_c_example_runs(tmp_path):
    """The C example (examples/transpose_example.c) transposes on the device through the
    plain C ABI and verifies A^T(j, i) = A(i, j) on the host (odd and square shapes)."""
    import subprocess
    import importlib.util
    spec = importlib.util.spec_from_file_location(
        "abi_cpu", os.path.join(os.path.dirname(os.path.abspath(__file__)), "test_abi_cpu.py"))
    mod = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(mod)
    exe = mod._build_c_example(tmp_path)
    for (M, N) in [(1800, 7200), (997, 4093), (2048, 2048), (1, 5)]:
        r = subprocess.run([exe, str(M), str(N)], capture_output=True, text=True, timeout=120)
        assert r.returncode == 0 and "ok: 0 mismatches" in r.stdout, (M, N, r.stdout, r.stderr)


@pytest.mark.parametrize("eb", [4, 8])
def test_transpose_host_pipeline(eb):
    """Host pipeline across matrices (two device slots, copy-in / compute / copy-out
    streams): every host matrix comes back transposed, bit-exact vs the oracle, including
    different shapes in one call, a square, a 1 x N no-op and a reuse of the slots."""
    shapes = [(1800, 7200), (97, 89), (1024, 1024), (1, 500), (360, 1000), (7200, 1800), (13, 1021)]
    hs, refs = [], []
    for (M, N) in shapes:
        a = seeded.matrix_np(M, N, eb)
        hs.append(torch.from_numpy(a.view(_NDT[eb]).copy()).pin_memory())
        refs.append(oracle.transpose_inplace(a.copy(), M, N))
    ipt.transpose_host_pipeline_(hs, shapes)
    torch.cuda.synchronize()
    for h, ref, sh in zip(hs, refs, shapes):
        assert np.array_equal(h.numpy().view(ref.dtype), ref), sh
    # and back (the reverse shapes), twice in a row on the same stream
    ipt.transpose_host_pipeline_(hs, [(N, M) for (M, N) in shapes])
    ipt.transpose_host_pipeline_(hs, shapes)
    torch.cuda.synchronize()
    for h, ref, sh in zip(hs, refs, shapes):
        assert np.array_equal(h.numpy().view(ref.dtype), ref), sh


def test_cycle_seg_counters_across_streams_and_many_launches(monkeypatch):
    """Self-resetting barrier counters: many back-to-back segmented launches on two streams
    (one counter pair each), every result bit-exact."""
    monkeypatch.setenv("IPT_CYC_SEG", "2")
    streams = [torch.cuda.Stream(), torch.cuda.Stream()]
    cases = [(2, 40, 56, 64), (1, 180, 40, 36)]
    ts, refs = [], []
    for (b, A, B, s_) in cases:
        a = gen(b * A * B * s_, 4)
        ts.append(to_dev(a, 4))
        refs.append(a)
    torch.cuda.synchronize()
    for it in range(40):
        for k, (b, A, B, s_) in enumerate(cases):
            with torch.cuda.stream(streams[k]):
                if it % 2 == 0:
                    ipt.ipt_100_(ts[k], b, A, B, s_, stream=streams[k])
                else:
                    ipt.ipt_100_(ts[k], b, B, A, s_, stream=streams[k])
    torch.cuda.synchronize()
    for k in range(2):
        assert np.array_equal(to_np(ts[k], 4), refs[k].view(np.uint32)), k


def test_fuzz_plans_and_kernel_variants(monkeypatch):
    """Seeded fuzz: random shapes, random valid tilings (m | M, n | N) and random kernel
    choices (flag / segmented cycles, swizzled / padded square swaps, TMA / cp.async tile
    slices, self-resetting / memset counters) -- every result bit-exact vs the oracle."""
    rnd = random.Random(2024)

    def divs(x):
        return [d for d in range(1, x + 1) if x % d == 0]

    knobs = {"IPT_CYC_SEG": ["0", "1", "2"], "IPT_SQ_SWZ": ["0", "1"],
             "IPT_TILE_GROUP_TMA": ["0", "1"], "IPT_TILE_GEN_TMAA": ["0", "1"],
             "IPT_SEG_RESET": ["0", "1"], "IPT_TILE_RESET": ["0", "1"]}
    for it in range(300):
        for k, vals in knobs.items():
            monkeypatch.setenv(k, rnd.choice(vals))
        eb = rnd.choice([4, 4, 8])
        M = rnd.choice([rnd.randint(2, 120), rnd.randint(100, 900), rnd.choice([360, 720, 1000, 1024])])
        N = rnd.choice([M, rnd.randint(2, 120), rnd.randint(100, 900)])
        m, n = rnd.choice(divs(M)), rnd.choice(divs(N))
        p = ipt.plan(M, N, eb, 0, m=m, n=n)
        a = seeded.matrix_np(M, N, eb, seed=seeded.SEED + it)
        t = to_dev(a, eb)
        ipt.transpose_(t, M, N, plan_=p)
        ok = np.array_equal(to_np(t, eb), oracle.transpose_inplace(a.copy(), M, N))
        assert ok, (it, M, N, m, n, eb, {k: os.environ.get(k) for k in knobs})


@pytest.mark.parametrize("M,N,eb", [(1800, 7200, 4), (360, 1000, 4), (2048, 2048, 8), (9998, 192, 4),
                                    (720, 1800, 8), (97, 89, 4)])
def test_cuda_graph_api(M, N, eb):
    """ipt_graph_create / ipt_graph_launch: an M x N graph and an N x M graph replayed
    A, B, A (after one uncaptured warm-up round trip) leave A^T, bit-exact."""
    a = seeded.matrix_np(M, N, eb)
    t = to_dev(a, eb)
    p, q = ipt.plan(M, N, eb, 0), ipt.plan(N, M, eb, 0)
    ipt.transpose_(t, M, N, plan_=p)
    ipt.transpose_(t, N, M, plan_=q)
    gA, gB = ipt.Graph(t, M, N, p), ipt.Graph(t, N, M, q)
    before = ipt.kernel_launch_count()
    for g in (gA, gB, gA):
        g.launch()
    torch.cuda.synchronize()
    assert ipt.kernel_launch_count() == before      # replays launch no kernels from the host
    assert np.array_equal(to_np(t, eb), oracle.transpose_inplace(a.copy(), M, N)), (M, N, eb)


def test_cuda_graph_batched():
    """A graph over a batch of matrices with a stride (gaps untouched)."""
    count, M, N, gap = 3, 360, 1000, 64
    stride = M * N + gap
    a = gen(count * stride, 4)
    t = to_dev(a, 4)
    p = ipt.plan(M, N, 4, 0)
    g = ipt.Graph(t, M, N, p, count=count, stride_elems=stride)
    g.launch()
    torch.cuda.synchronize()
    got, src = to_np(t, 4), a.view(np.uint32)
    for k in range(count):
        blk = src[k * stride:k * stride + M * N].copy()
        assert np.array_equal(got[k * stride:k * stride + M * N], oracle.transpose_inplace(blk, M, N)), k
        assert np.array_equal(got[k * stride + M * N:(k + 1) * stride], src[k * stride + M * N:(k + 1) * stride])


@pytest.mark.parametrize("eb", [1, 2, 4, 8, 16])
def test_public_api_degenerate_shapes(eb):
    """The planner path of ipt_transpose / ipt_transpose_batched on the degenerate cases:
    1 x N and M x 1 (no-ops, C6), 1 x 1, 2 x 2, 2 x 3, a prime x prime pair, an empty batch
    (count 0: nothing touched) and a batch of one -- each against the oracle."""
    for (M, N) in [(1, 17), (23, 1), (1, 1), (2, 2), (2, 3), (13, 7), (3, 1024)]:
        a = gen(M * N, eb)
        t = to_dev(a, eb)
        ipt.transpose_(t, M, N, elem_bytes=eb)
        assert np.array_equal(to_np(t, eb), oracle_P(a.copy(), 1, M, N, 1, eb)), (M, N, eb)
    a = gen(64, eb)
    t = to_dev(a, eb)
    ipt.transpose_batched_(t, 0, 4, 16, elem_bytes=eb)
    assert np.array_equal(to_np(t, eb), a)
    ipt.transpose_batched_(t, 1, 4, 16, elem_bytes=eb)
    assert np.array_equal(to_np(t, eb), oracle_P(a.copy(), 1, 4, 16, 1, eb))
