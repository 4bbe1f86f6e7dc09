"""The BASELINE.json workloads as shape lists (no method arithmetic: shapes only).

Shared by bench.py (timed) and tests/test_gpu_parity.py (full-size parity of every shape
the bench times).  Shapes follow SURVEY.md 8(d) "Concrete synthetic inputs" and the
paper's workloads: Table 2 (~12.9 M single-precision elements each), the
K-Means descriptors, awkward and prime dimensions.
"""
from __future__ import annotations

import numpy as np

# configs[0]: single 1800 x 7200 float32 (the paper's Table 2 row)
C1 = [(1800, 7200)]
# configs[2]: 1,000,000 x 256 float32 K-Means descriptors, AoS -> SoA
C3 = [(1_000_000, 256)]
# configs[3]: 20000 x 30000 float64 (4.8 GB)
C4 = [(20000, 30000)]
# configs[4]: batch of 512 independent 4096 x 3000 float32 matrices (25.17 GB)
C5_SHAPE, C5_COUNT = (4096, 3000), 512

# the paper's Table 2 shapes, rows x cols; P:283 is a garbled duplicate (C17)
TABLE2 = [(7200, 1800), (5100, 2500), (4000, 3200), (3300, 3900), (2500, 5100), (1800, 7200)]

# configs[1]: shape sweep M, N in [1000, 20000] float32 including dims with few small
# factors.  Every class the survey lists:
SWEEP_POW2 = [(1024, 16384), (4096, 4096), (8192, 2048)]
SWEEP_FEW_FACTORS = [(9998, 4096),      # 9998 = 2 * 4999
                     (9797, 13081),     # 9797 = 97 * 101, 13081 = 103 * 127
                     (14803, 1024)]     # 14803 = 113 * 131
SWEEP_LARGE = [(7200, 18000), (18000, 7200), (16384, 16384), (12800, 15000), (19200, 10000),
               (9998, 12288), (14803, 8192), (20000, 20000)]


def sweep_random_pairs(n: int = 16, seed: int = 1):
    """n seeded (M, N) pairs, uniform in [1000, 20000] (numpy default_rng(seed))."""
    rng = np.random.default_rng(seed)
    return [(int(a), int(b)) for a, b in rng.integers(1000, 20001, size=(n, 2))]


SWEEP_RANDOM = sweep_random_pairs()

# prime / prime-containing dims: correctness only ("degrade")
PRIMES = [(19997, 1024), (1021, 4093), (1009, 7001), (10007, 19997),
          (10007, 10007)]    # a prime-sided square: the swap kernel's element path


def dedup(shapes):
    seen, out = set(), []
    for s in shapes:
        if s not in seen:
            seen.add(s)
            out.append(s)
    return out


# the full C2 list the bench times (primes are reported separately, correctness only)
SWEEP_ALL = dedup(TABLE2 + SWEEP_POW2 + SWEEP_FEW_FACTORS + SWEEP_LARGE + SWEEP_RANDOM)


def is_square(shape) -> bool:
    return shape[0] == shape[1]
