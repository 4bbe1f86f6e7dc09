"""Full-size GPU parity of every shape bench.py times, in the bench's launch configuration.

For each matrix of the BASELINE workloads (inputs/workloads.py: C1, C3, C4, the paper's
Table 2 shapes, the whole C2 sweep incl. few-factor and seeded random shapes, the prime
shapes) the test does what the bench does -- ipt_plan_autotune with 8 candidates in both
orientations (every candidate runs forward and the model plan back: the data must come
back bit for bit) -- then transposes with the tuned plan and checks the result (a) on
sampled outputs computed one by one by the oracle's Eq. (1) and the generator and (b) on
every element through the definition A^T(j, i) = A(i, j) (torch index arithmetic on the
device), transposes back with the tuned reverse plan and checks the input is restored.

The C5 headline (512 x 4096 x 3000 float32, 25.17 GB on one GPU) is checked the same way
on all 512 matrices: oracle samples of every matrix plus every element of every matrix by
the definition.
"""
import random

import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")

import paper_conf_ppopp_sunggggh14_b200 as ipt  # noqa: E402
from inputs import seeded, workloads as W  # noqa: E402
from oracle import oracle  # noqa: E402

AUTOTUNE = 8   # bench.py --autotune default

SHAPES = ([(M, N, 4) for (M, N) in W.C1 + W.C3 + W.SWEEP_ALL + W.PRIMES]
          + [(M, N, 8) for (M, N) in W.C4])


def _oracle_samples(t, M, N, eb, t_idx, nsamp, seed):
    """Outputs at Eq. (1) destinations of random sources, one by one (the oracle's Eq. 1)."""
    rnd = random.Random(seed)
    n = M * N
    ks = [rnd.randrange(n) for _ in range(nsamp)] + [0, 1, n - 2, n - 1]
    dst = torch.tensor([oracle.eq1_dest(k, M, N) for k in ks], device=t.device)
    exp = seeded.values_torch_sample(torch.tensor(ks, device=t.device) + t_idx * n, eb)
    return torch.equal(t.view(-1)[dst], exp.to(t.dtype))


def _definition(t, M, N, eb, t_idx):
    """Every element: position p = j*M + i of A^T holds v(i*N + j) of matrix t_idx."""
    n = M * N
    CH = 1 << 27
    flat = t.view(-1)
    for p0 in range(0, n, CH):
        p = torch.arange(p0, min(n, p0 + CH), device=t.device, dtype=torch.int64)
        exp = seeded.values_torch_sample((p % M) * N + p // M + t_idx * n, eb)
        if not torch.equal(flat[p0:p0 + p.numel()], exp.to(t.dtype)):
            return False
    return True


def _is_input(t, M, N, eb, t0=0, count=1):
    CH = 1 << 27
    flat = t.view(-1)
    tot = count * M * N
    for p0 in range(0, tot, CH):
        p = torch.arange(p0, min(tot, p0 + CH), device=t.device, dtype=torch.int64)
        if not torch.equal(flat[p0:p0 + p.numel()], seeded.values_torch_sample(p + t0 * M * N, eb).to(t.dtype)):
            return False
    return True


@pytest.mark.parametrize("M,N,eb", SHAPES, ids=[f"{M}x{N}x{eb}" for (M, N, eb) in SHAPES])
def test_benched_shape_full_parity(M, N, eb):
    dt = torch.int32 if eb == 4 else torch.int64
    t = torch.empty(M * N, dtype=dt, device="cuda")
    seeded.fill_device_(t, M, N, eb)
    p = ipt.plan_autotune(t, M, N, AUTOTUNE)
    assert _is_input(t, M, N, eb), "autotune must leave the data unchanged"
    ipt.transpose_(t, M, N, plan_=p)
    assert _oracle_samples(t, M, N, eb, 0, 3000, seed=M ^ N), p.as_dict()
    assert _definition(t, M, N, eb, 0), p.as_dict()
    q = ipt.plan_autotune(t, N, M, AUTOTUNE)
    ipt.transpose_(t, N, M, plan_=q)
    assert _is_input(t, M, N, eb), (p.as_dict(), q.as_dict())
    del t
    torch.cuda.empty_cache()


def test_c5_full_batch_one_gpu():
    """configs[4] on one GPU: 512 x 4096 x 3000 float32 (25.17 GB), the bench's tuned batch
    plans in both orientations; every matrix checked."""
    count, (M, N) = W.C5_COUNT, W.C5_SHAPE
    free, _ = torch.cuda.mem_get_info()
    if free < count * M * N * 4 + (6 << 30):
        pytest.skip("needs ~32 GB of free device memory")
    t = torch.empty(count * M * N, dtype=torch.int32, device="cuda")
    seeded.fill_device_(t, M, N, 4, count=count)
    p = ipt.plan_autotune_batched(t, count, M, N, AUTOTUNE)
    assert _is_input(t, M, N, 4, count=count), "autotune must leave the data unchanged"
    ipt.transpose_batched_(t, count, M, N, plan_=p)
    torch.cuda.synchronize()
    n = M * N
    for k in range(count):
        mk = t[k * n:(k + 1) * n]
        assert _oracle_samples(mk, M, N, 4, k, 64, seed=k), k
        assert _definition(mk, M, N, 4, k), k
    q = ipt.plan_autotune_batched(t, count, N, M, AUTOTUNE)
    ipt.transpose_batched_(t, count, N, M, plan_=q)
    assert _is_input(t, M, N, 4, count=count)
    del t
    torch.cuda.empty_cache()


def test_c5_fixed_orientation_steps():
    """The bench's headline steps (--orientation fixed): the full 512-matrix C5 batch
    transposed as 4096 x 3000 three times in a row (each result re-read as the next
    4096 x 3000 input), then once as 3000 x 4096 -- every element of three matrices and the
    first element block of all 512 checked against the composed definition (each a x b
    transpose moves position i*b + j to j*a + i)."""
    count, (M, N) = W.C5_COUNT, W.C5_SHAPE
    free, _ = torch.cuda.mem_get_info()
    if free < count * M * N * 4 + (6 << 30):
        pytest.skip("needs ~32 GB of free device memory")
    n = M * N
    t = torch.empty(count * n, dtype=torch.int32, device="cuda")
    seeded.fill_device_(t, M, N, 4, count=count)
    p = ipt.plan_autotune_batched(t, count, M, N, AUTOTUNE)
    q = ipt.plan_autotune_batched(t, count, N, M, AUTOTUNE)
    seq = [(M, N)] * 3 + [(N, M)]
    for (a, b) in seq:
        ipt.transpose_batched_(t, count, a, b, plan_=p if (a, b) == (M, N) else q)
    torch.cuda.synchronize()

    def src_of(pos):
        for (a, b) in reversed(seq):
            pos = (pos % a) * b + pos // a
        return pos

    CH = 1 << 26
    for k in (0, count // 2, count - 1):         # every element of three matrices
        flat = t[k * n:(k + 1) * n]
        for p0 in range(0, n, CH):
            pos = torch.arange(p0, min(n, p0 + CH), device="cuda", dtype=torch.int64)
            exp = seeded.values_torch_sample(src_of(pos) + k * n, 4)
            assert torch.equal(flat[p0:p0 + pos.numel()], exp.to(torch.int32)), k
    pos = torch.arange(0, 4096, device="cuda", dtype=torch.int64)
    src = src_of(pos)
    for k in range(count):                       # a block of every matrix
        exp = seeded.values_torch_sample(src + k * n, 4)
        assert torch.equal(t[k * n:k * n + 4096], exp.to(torch.int32)), k
    del t
    torch.cuda.empty_cache()


# ------------------------------------------------------- capture-safety
def _mat(M, N, t0=0):
    t = torch.empty(M * N, dtype=torch.int32, device="cuda")
    seeded.fill_device_(t, M, N, 4, t0=t0)
    torch.cuda.synchronize()          # filled on the current stream; tests use others
    return t


@pytest.mark.parametrize("M,N,m,n", [(1800, 7200, 120, 200), (360, 1000, 0, 0), (7200, 1800, 1800, 1800)])
def test_capture_without_warmup_graph_owned_workspace(M, N, m, n):
    """A plan captured by torch.cuda.graph with NO prior direct call (no cached state,
    NULL workspace): the captured sequence allocates and frees its own flags; replays
    (forward graph, then reverse graph) are exact."""
    t = _mat(M, N)
    p = ipt.plan(M, N, 4, 0, m=m, n=n) if m else ipt.plan(M, N, 4, 0)
    q = ipt.plan(N, M, 4, 0, m=n, n=m) if m else ipt.plan(N, M, 4, 0)
    s = torch.cuda.Stream()
    gA, gB = torch.cuda.CUDAGraph(), torch.cuda.CUDAGraph()
    with torch.cuda.graph(gA, stream=s):
        ipt.transpose_(t, M, N, plan_=p, stream=s)
    with torch.cuda.graph(gB, stream=s):
        ipt.transpose_(t, N, M, plan_=q, stream=s)
    torch.cuda.synchronize()
    assert _is_input(t, M, N, 4), "capture must not execute"
    for _ in range(3):
        gA.replay()
        torch.cuda.synchronize()
        assert _definition(t, M, N, 4, 0)
        gB.replay()
        torch.cuda.synchronize()
        assert _is_input(t, M, N, 4)


def test_graph_replay_on_other_stream_concurrent_with_direct_calls():
    """A graph captured on stream S replayed on stream T while direct calls run on S (its
    internal workspace / counters) on another matrix: both exact (no shared flags or
    counters between the replay and the direct calls)."""
    M, N = 1800, 7200
    p, q = ipt.plan(M, N, 4, 0, m=120, n=200), ipt.plan(N, M, 4, 0, m=200, n=120)
    a, b = _mat(M, N, t0=0), _mat(M, N, t0=1)
    S, T = torch.cuda.Stream(), torch.cuda.Stream()
    with torch.cuda.stream(S):                 # direct calls build the per-stream state of S
        ipt.transpose_(b, M, N, plan_=p, stream=S)
        ipt.transpose_(b, N, M, plan_=q, stream=S)
    torch.cuda.synchronize()
    gA, gB = torch.cuda.CUDAGraph(), torch.cuda.CUDAGraph()
    with torch.cuda.graph(gA, stream=S):
        ipt.transpose_(a, M, N, plan_=p, stream=S)
    with torch.cuda.graph(gB, stream=S):
        ipt.transpose_(a, N, M, plan_=q, stream=S)
    torch.cuda.synchronize()
    for _ in range(10):
        with torch.cuda.stream(T):
            gA.replay()
            gB.replay()
        ipt.transpose_(b, M, N, plan_=p, stream=S)
        ipt.transpose_(b, N, M, plan_=q, stream=S)
    torch.cuda.synchronize()
    assert _is_input(a, M, N, 4, t0=0) and _is_input(b, M, N, 4, t0=1)


def test_graph_survives_workspace_growth_on_capture_stream():
    """After a capture on S, a direct call on S needing a much larger internal workspace
    (the per-stream cache grows) must not invalidate the graph."""
    M, N = 720, 1800
    p, q = ipt.plan(M, N, 4, 0, m=120, n=200), ipt.plan(N, M, 4, 0, m=200, n=120)
    a = _mat(M, N)
    S = torch.cuda.Stream()
    with torch.cuda.stream(S):
        ipt.transpose_(a, M, N, plan_=p, stream=S)
        ipt.transpose_(a, N, M, plan_=q, stream=S)
    torch.cuda.synchronize()
    gA, gB = ipt.Graph(a, M, N, p), ipt.Graph(a, N, M, q)
    big_M, big_N = 10007, 19997                # scalar fallback: 25 MB of flags on S
    big = _mat(big_M, big_N, t0=7)
    ipt.transpose_(big, big_M, big_N, stream=S)
    torch.cuda.synchronize()
    for _ in range(3):
        gA.launch(S)
        gB.launch(S)
    torch.cuda.synchronize()
    assert _is_input(a, M, N, 4)
    assert _definition(big, big_M, big_N, 4, 7)


def test_graph_checks_sizes_and_plan():
    M, N = 360, 1000
    t = _mat(M, N)
    p = ipt.plan(M, N, 4, 0)
    with pytest.raises(ipt.IptError):
        ipt.Graph(t[:-1], M, N, p)                       # too small
    with pytest.raises(ipt.IptError):
        ipt.Graph(t, N, M, p)                            # plan for another shape
    with pytest.raises(ipt.IptError):
        ipt.Graph(t, M, N, p, count=2)                   # batch does not fit


def test_edited_plan_rejected():
    """validate_plan checks every stage's variant against its shape."""
    M, N = 720, 1800
    t = _mat(M, N)
    p = ipt.plan(M, N, 4, 0, m=120, n=200)
    for st, v in [(0, 1), (2, 1), (0, 4), (0, 0), (2, 0), (1, 0), (1, 4), (1, 2), (0, 7)]:
        bad = ipt.Plan.from_buffer_copy(p)
        bad.variant[st] = v
        with pytest.raises(ipt.IptError):
            ipt.transpose_(t, M, N, plan_=bad)
    assert _is_input(t, M, N, 4)                         # nothing was launched


# ------------------------- whole-GPU tiles in shared memory + tensor memory (tile_group_rf)
RF_CASES = [  # (M, N, eb, count, stride pad in elements, smem budget override or 0)
    (4096, 3000, 4, 3, 0, 0),          # C5 matrices: row split, 16 rows by TMA + 12 in TMEM
    (3000, 4096, 4, 2, 64, 0),         # strided batch: 3-D tensor map
    (1800, 7200, 4, 1, 0, 0),          # C1: column split
    (7200, 1800, 4, 1, 0, 0),
    (1024, 16384, 4, 1, 0, 0),         # 67 MB: TMEM part written out in row chunks
    (2048, 4096, 8, 1, 0, 0),          # float64
    (720, 1800, 4, 5, 0, 20000),       # small tiles forced through the rf path with a small
    (1200, 760, 8, 3, 8, 12000),       # smem budget: TMEM part in several row chunks
    (720, 1800, 4, 2, 0, 60000),       # everything in shared memory (no TMEM part)
    (4096, 3000, 4, 2, 0, -16),        # row slices on any 16-byte boundary (IPT_TILE_RF_RALIGN=0)
    (4000, 3200, 4, 2, 0, -64),        # 64-byte aligned row slices
    (600, 4096, 4, 3, 0, 0),           # column slices of one 128-byte line, TMA 128-byte swizzle:
    (2500, 4096, 4, 1, 0, 0),          #   no TMEM part / a TMEM part restaged swizzled,
    (1500, 2048, 8, 2, 24, 0),         #   float64, strided (3-D map)
    (3000, 4096, 4, 2, 0, -1),         # the same tile with the swizzled slices off (-1)
]


@pytest.mark.parametrize("M,N,eb,count,pad,smem", RF_CASES,
                         ids=[f"{c[0]}x{c[1]}x{c[2]}b{c[3]}p{c[4]}s{c[5]}" for c in RF_CASES])
def test_tile_group_rf(monkeypatch, M, N, eb, count, pad, smem):
    """The whole tile of a 1-stage plan (m = M, n = N) held over every SM in shared memory
    (TMA part) and TMEM (tcgen05.st / tcgen05.ld part): every element checked by the
    definition, strided gaps untouched, then transposed back."""
    monkeypatch.setenv("IPT_TILE_RF_FORCE", "1")
    if smem > 0:
        monkeypatch.setenv("IPT_TILE_SMEM_MAX", str(smem))
    elif smem == -1:
        monkeypatch.setenv("IPT_TILE_RF_SWZ", "0")
    elif smem < 0:
        monkeypatch.setenv("IPT_TILE_RF_RALIGN", str(-smem if smem != -16 else 0))
    dt = torch.int32 if eb == 4 else torch.int64
    stride = M * N + pad
    t = torch.empty(count * stride, dtype=dt, device="cuda")
    for k in range(count):
        seeded.fill_device_(t[k * stride:k * stride + M * N], M, N, eb, t0=k)
    gaps = [t[k * stride + M * N:(k + 1) * stride].clone() for k in range(count)]
    p = ipt.plan(M, N, eb, 0, m=M, n=N)
    q = ipt.plan(N, M, eb, 0, m=N, n=M)
    assert ipt.stage_kernels(p, count, t)[1] == "tile_group_rf"
    ipt.transpose_batched_(t, count, M, N, stride_elems=stride, plan_=p)
    torch.cuda.synchronize()
    for k in range(count):
        assert _definition(t[k * stride:k * stride + M * N], M, N, eb, k), k
        assert torch.equal(t[k * stride + M * N:(k + 1) * stride], gaps[k])
    ipt.transpose_batched_(t, count, N, M, stride_elems=stride, plan_=q)
    for k in range(count):
        assert _is_input(t[k * stride:k * stride + M * N], M, N, eb, t0=k), k
