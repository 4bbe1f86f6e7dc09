"""Pins for the CPU oracle (oracle/ipt_oracle.c) against things other than itself.

Each pin is chosen so that a plausible oracle mistake (a dropped term in Eq. (1), a
swapped M/N, an off-by-one in the k = MN-1 case, a transposed stage operand, a wrong
super-element stride) fails at least one of them:

  * numpy's out-of-place transpose / reshape-transpose (library routines, brute force);
  * the worked 5 x 3 example printed in the paper -- tests/golden/;
  * closed-form cycle counts from number theory (sympy's totient / n_order / divisors);
  * the definition k = i*N + j  ->  k' = j*M + i for Eq. (1);
  * invariants: double transpose = identity, 1 x N and M x 1 unchanged, square matrices
    swap symmetric pairs, raw bit patterns preserved.
"""
import math
import os
import random

import numpy as np
import pytest
import sympy

from inputs import seeded
from oracle import oracle

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _np_T(a, M, N):
    return a.reshape(M, N).T.copy().reshape(-1)


def _np_P(a, batch, A, B, s):
    return a.reshape(batch, A, B, s).transpose(0, 2, 1, 3).copy().reshape(-1)


def _divisors(x):
    return [d for d in range(1, x + 1) if x % d == 0]


# ----------------------------------------------------------------------------- Eq. (1)
def test_eq1_matches_definition_exhaustive():
    """A(i,j) at k = i*N + j moves to k' = j*M + i; Eq. (1) must agree everywhere."""
    for M in range(1, 25):
        for N in range(1, 25):
            for i in range(M):
                for j in range(N):
                    assert oracle.eq1_dest(i * N + j, M, N) == j * M + i


def test_eq1_large_no_overflow():
    """k*M exceeds 64 bits for these shapes; the oracle must still be exact."""
    M, N = 3_000_000_019, 3_000_000_017
    for i, j in [(0, 1), (M - 1, N - 2), (123456789, 987654321), (M - 2, N - 1)]:
        assert oracle.eq1_dest(i * N + j, M, N) == j * M + i


# -------------------------------------------------------------------- worked example
def _golden_cycles():
    rows = [l.split() for l in open(os.path.join(GOLDEN, "paper_5x3_cycles.txt"))
            if l.strip() and not l.startswith("#")]
    M = int(rows[0][1]); N = int(rows[1][1])
    return M, N, [tuple(int(x) for x in r) for r in rows[2:]]


def test_paper_5x3_cycles():
    """(0) (1 5 11 13 9 3) (7) (2 10 8 12 4 6) (14)."""
    M, N, cycles = _golden_cycles()
    got = oracle.cycles_list(M, N)
    assert sorted(got) == sorted(cycles)
    # first steps spelled out in the prose: element 1 -> location 5, 5 -> 11, 11 -> 13
    assert oracle.eq1_dest(1, M, N) == 5
    assert oracle.eq1_dest(5, M, N) == 11
    assert oracle.eq1_dest(11, M, N) == 13
    assert oracle.cycle_stats(M, N) == (5, 3, 6)


# ----------------------------------------------------------------------- closed forms
def closed_form_stats(M, N):
    """Number theory (not the paper): the offsets 0..MN-2 are permuted by k -> k*M mod
    calM (calM = MN-1, M invertible mod calM since M*N = 1 mod calM).  Offsets with
    gcd(k, calM) = calM/d form phi(d) elements on which the map acts as the unit group
    mod d, in orbits of length ord_d(M); offset calM is fixed.
      cycles  = 1 + sum_{d | calM} phi(d)/ord_d(M)
      fixed   = 1 + gcd(M-1, N-1)
      longest = ord_calM(M)"""
    calM = M * N - 1
    if calM == 0:
        return 1, 1, 1
    cyc = 1
    for d in sympy.divisors(calM):
        cyc += int(sympy.totient(d)) // (1 if d == 1 else int(sympy.n_order(M % d, d)))
    longest = 1 if calM == 1 else int(sympy.n_order(M % calM, calM))
    return cyc, 1 + math.gcd(M - 1, N - 1), longest


def test_cycle_stats_closed_form_small_exhaustive():
    for M in range(1, 30):
        for N in range(1, 30):
            assert oracle.cycle_stats(M, N) == closed_form_stats(M, N), (M, N)


@pytest.mark.parametrize("M,N,expect", [
    # values tabulated in SURVEY.md 8(c) (derived, then enumerated); re-derived here
    (1800, 7200, (558, 2, 40020)),
    (7200, 1800, (558, 2, 40020)),
    (4096, 3000, (4, 2, 6143999)),
    (19997, 1024, (118, 2, 179622)),
    (1021, 4093, (127, 13, 174096)),
    (9973, 256, (1540, 4, 3519)),
])
def test_cycle_stats_closed_form_paper_shapes(M, N, expect):
    assert closed_form_stats(M, N) == expect
    assert oracle.cycle_stats(M, N) == expect


# ------------------------------------------------------------- full transpose vs numpy
@pytest.mark.parametrize("b", [1, 2, 4, 8])
def test_transpose_vs_numpy_exhaustive_small(b):
    for M in range(1, 20):
        for N in range(1, 20):
            a = seeded.matrix_np(M, N, b)
            ref = _np_T(a, M, N)
            oracle.transpose_inplace(a, M, N)
            assert np.array_equal(a, ref), (M, N, b)


def test_transpose_vs_numpy_primes_and_random():
    rnd = random.Random(7)
    shapes = [(97, 101), (1021, 13), (13, 1021), (257, 255), (1, 5000), (5000, 1),
              (64, 64), (2, 3), (331, 337)]
    shapes += [(rnd.randint(1, 400), rnd.randint(1, 400)) for _ in range(20)]
    for (M, N) in shapes:
        for b in (4, 8):
            a = seeded.matrix_np(M, N, b)
            ref = _np_T(a, M, N)
            oracle.transpose_inplace(a, M, N)
            assert np.array_equal(a, ref), (M, N, b)


def test_random_bits_preserved():
    """Raw moves: NaN payloads / -0.0 / denormals survive."""
    for b in (4, 8):
        a = seeded.random_bits_np(123 * 77, b, seed=3)
        ref = _np_T(a, 123, 77)
        oracle.transpose_inplace(a, 123, 77)
        assert np.array_equal(a, ref)


# -------------------------------------------------------------------------- invariants
def test_double_transpose_identity():
    for (M, N) in [(5, 3), (17, 64), (100, 7), (128, 96)]:
        a = seeded.matrix_np(M, N, 4)
        orig = a.copy()
        oracle.transpose_inplace(a, M, N)
        oracle.transpose_inplace(a, N, M)
        assert np.array_equal(a, orig)


def test_vector_shapes_unchanged():
    for (M, N) in [(1, 1), (1, 37), (41, 1)]:
        a = seeded.matrix_np(M, N, 8)
        orig = a.copy()
        oracle.transpose_inplace(a, M, N)
        assert np.array_equal(a, orig)


def test_square_swaps_symmetric_pairs():
    """for square matrices the cycles are the symmetric pairs, diagonal fixed."""
    for n in (2, 3, 16, 33):
        cyc = oracle.cycles_list(n, n)
        assert sum(len(c) == 1 for c in cyc) == n
        assert all(len(c) in (1, 2) for c in cyc)
        for c in cyc:
            if len(c) == 2:
                i, j = divmod(c[0], n)
                assert c[1] == j * n + i


# ------------------------------------------------------------- elementary permutations
def test_permute_vs_numpy_random():
    rnd = random.Random(11)
    for _ in range(200):
        batch, A, B, s = rnd.randint(1, 4), rnd.randint(1, 30), rnd.randint(1, 30), rnd.randint(1, 9)
        for b in (4, 8):
            a = seeded.values_np(np.arange(batch * A * B * s), b)
            ref = _np_P(a, batch, A, B, s)
            oracle.permute_inplace(a, batch, A, B, s)
            assert np.array_equal(a, ref), (batch, A, B, s, b)


def test_stage_definitions_match_paper_views():
    """each stage as a numpy dimension permutation of the paper's views."""
    M, N, m, n = 12, 20, 3, 5
    Mp, Np = M // m, N // n
    a = seeded.matrix_np(M, N, 4)
    s1 = a.reshape(M, Np, n).transpose(1, 0, 2).copy().reshape(-1)          # 100!
    s2 = s1.reshape(Np, Mp, m, n).transpose(0, 1, 3, 2).copy().reshape(-1)  # 0010!
    s3 = s2.reshape(Np, Mp, n, m).transpose(0, 2, 1, 3).copy().reshape(-1)  # 0100!
    b = a.copy()
    oracle.permute_inplace(b, 1, M, Np, n)
    assert np.array_equal(b, s1)
    oracle.permute_inplace(b, Np * Mp, m, n, 1)
    assert np.array_equal(b, s2)
    oracle.permute_inplace(b, Np, Mp, n, m)
    assert np.array_equal(b, s3)
    assert np.array_equal(b, _np_T(a, M, N))


def test_3stage_and_4stage_all_tilings():
    """Sec. 4.1/4.2: every divisor pair (m, n) gives exactly the transpose."""
    for (M, N) in [(12, 18), (30, 8), (7, 14), (16, 16), (9, 25), (1, 6), (6, 1)]:
        ref = _np_T(seeded.matrix_np(M, N, 8), M, N)
        for m in _divisors(M):
            for n in _divisors(N):
                a = seeded.matrix_np(M, N, 8)
                oracle.transpose_3stage(a, M, N, m, n)
                assert np.array_equal(a, ref), ("3stage", M, N, m, n)
                a = seeded.matrix_np(M, N, 8)
                oracle.transpose_4stage(a, M, N, m, n)
                assert np.array_equal(a, ref), ("4stage", M, N, m, n)


def test_batch_folding_equals_per_matrix():
    """Batched transposition folds the batch into each stage."""
    count, M, N, m, n = 3, 12, 10, 4, 5
    Mp, Np = M // m, N // n
    a = seeded.batch_np(count, M, N, 4)
    ref = np.concatenate([_np_T(a[t * M * N:(t + 1) * M * N], M, N) for t in range(count)])
    oracle.permute_inplace(a, count, M, Np, n)
    oracle.permute_inplace(a, count * Np * Mp, m, n, 1)
    oracle.permute_inplace(a, count * Np, Mp, n, m)
    assert np.array_equal(a, ref)


def test_invalid_args():
    a = np.zeros(6, dtype=np.uint32)
    with pytest.raises(ValueError):
        oracle.transpose_3stage(a, 2, 3, 4, 1)
    assert oracle.lib().oracle_permute_inplace(a.ctypes.data, 1, 0, 1, 1, 4) == -1
    assert oracle.lib().oracle_permute_inplace(a.ctypes.data, 1, 2, 3, 1, 0) == -1
