"""Seeded synthetic inputs shared by the tests, the bench and smoke().

This module holds NONE of the method's arithmetic (no index map, no permutation): it
only produces input values.  Both the oracle side and the CUDA side are fed from here.

Recipe: every element of every matrix is unique,
so any misplacement is caught, and any single value can be regenerated from its
(matrix, offset) pair without storing a copy:

    b = 4:  v(t, k) = uint32((k + t*M*N) * 0x9E3779B1 + seed)
    b = 8:  v(t, k) = uint64((k + t*M*N) * 0x9E3779B97F4A7C15 + seed)
    b = 1/2: the low 8/16 bits of the b = 4 formula (not unique; used only in small tests)

with k the row-major offset inside matrix t and seed = 0x5EED by default.  The
multipliers are odd, so v is a bijection of the linear index modulo 2^(8b).
"""
from __future__ import annotations

import numpy as np

SEED = 0x5EED
_MUL32 = 0x9E3779B1
_MUL64 = 0x9E3779B97F4A7C15
_DT = {1: np.uint8, 2: np.uint16, 4: np.uint32, 8: np.uint64}


def values_np(lin: np.ndarray, elem_bytes: int, seed: int = SEED) -> np.ndarray:
    """Generator values for linear indices ``lin`` (int64 / uint64 numpy array)."""
    lin = np.asarray(lin).astype(np.uint64)
    if elem_bytes == 8:
        with np.errstate(over="ignore"):
            return lin * np.uint64(_MUL64) + np.uint64(seed)
    with np.errstate(over="ignore"):
        v = (lin * np.uint64(_MUL32) + np.uint64(seed)) & np.uint64(0xFFFFFFFF)
    return v.astype(np.uint32).astype(_DT[elem_bytes])


def matrix_np(M: int, N: int, elem_bytes: int, t: int = 0, seed: int = SEED) -> np.ndarray:
    """Matrix t of a batch of M x N matrices, flat row-major numpy array."""
    base = t * M * N
    return values_np(np.arange(base, base + M * N, dtype=np.uint64), elem_bytes, seed)


def batch_np(count: int, M: int, N: int, elem_bytes: int, seed: int = SEED) -> np.ndarray:
    return values_np(np.arange(count * M * N, dtype=np.uint64), elem_bytes, seed)


def random_bits_np(n_elems: int, elem_bytes: int, seed: int = 0) -> np.ndarray:
    """Arbitrary bit patterns (NaN payloads, denormals, -0.0 when viewed as floats)."""
    rng = np.random.default_rng(seed)
    return np.frombuffer(rng.bytes(n_elems * elem_bytes), dtype=_DT[elem_bytes]).copy()


def fill_device_(buf, M: int, N: int, elem_bytes: int, t0: int = 0, count: int = 1,
                 seed: int = SEED):
    """Fill a flat torch CUDA tensor (int32/int64 storage of ``count`` matrices starting at
    matrix index t0) with the generator values, on the device.  Used by the bench and the
    large GPU tests so that full-size inputs never cross PCIe."""
    import torch

    n = count * M * N
    assert buf.numel() >= n
    if elem_bytes not in (4, 8):
        raise ValueError("device fill supports 4- and 8-byte elements")
    CH = 1 << 27   # bounded temporaries
    for c0 in range(0, n, CH):
        c1 = min(n, c0 + CH)
        lin = torch.arange(t0 * M * N + c0, t0 * M * N + c1, device=buf.device, dtype=torch.int64)
        buf[c0:c1].copy_(values_torch_sample(lin, elem_bytes, seed))
    return buf


def values_torch_sample(lin, elem_bytes: int, seed: int = SEED):
    """Expected generator values (as int32/int64 torch tensors on lin's device)."""
    import torch

    lin = lin.to(torch.int64)
    if elem_bytes == 8:
        return lin * (_MUL64 - (1 << 64)) + seed
    v = (lin * _MUL32 + seed) & 0xFFFFFFFF
    return torch.where(v >= 2 ** 31, v - 2 ** 32, v).to(torch.int32)
