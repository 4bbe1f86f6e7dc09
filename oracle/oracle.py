"""CPU oracle for in-place transposition -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this module.  The product package
(``paper_conf_ppopp_sunggggh14_b200``) never imports it, and it shares no code with the
CUDA path (see ``ipt_oracle.c`` for the paper passages each routine follows).

Thin ctypes wrapper around ``liboracle.so`` (plain single-threaded C).  Arrays are numpy
arrays of an unsigned integer dtype of the element width (raw bit moves, no FP).

Parity status: every routine here is pinned by ``tests/test_oracle.py`` against numpy's
out-of-place transpose (a library routine), the worked example of P:113
(``tests/golden/paper_5x3_cycles.txt``), closed-form cycle counts derived from number
theory (computed with sympy), and invariants (double transpose = identity, 1xN / Mx1
unchanged, square = pairwise swaps).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "ipt_oracle.c")
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None

_DTYPES = {1: np.uint8, 2: np.uint16, 4: np.uint32, 8: np.uint64}


def build(force: bool = False) -> str:
    """Compile liboracle.so in-tree with gcc (plain -O2, single thread)."""
    if force or not os.path.exists(_LIB_PATH) or (
        os.path.getmtime(_LIB_PATH) < os.path.getmtime(_SRC)
    ):
        tmp = _LIB_PATH + f".tmp{os.getpid()}"
        subprocess.check_call(
            ["gcc", "-O2", "-std=c11", "-shared", "-fPIC", "-o", tmp, _SRC]
        )
        os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB_PATH)
        i64 = ctypes.c_int64
        L.oracle_eq1_dest.argtypes = [i64, i64, i64]
        L.oracle_eq1_dest.restype = i64
        L.oracle_permute_inplace.argtypes = [ctypes.c_void_p, i64, i64, i64, i64, ctypes.c_int]
        L.oracle_permute_inplace.restype = ctypes.c_int
        L.oracle_transpose_inplace.argtypes = [ctypes.c_void_p, i64, i64, ctypes.c_int]
        L.oracle_transpose_inplace.restype = ctypes.c_int
        for f in (L.oracle_transpose_3stage, L.oracle_transpose_4stage):
            f.argtypes = [ctypes.c_void_p, i64, i64, i64, i64, ctypes.c_int]
            f.restype = ctypes.c_int
        L.oracle_cycle_stats.argtypes = [i64, i64] + [ctypes.POINTER(i64)] * 3
        L.oracle_cycle_stats.restype = ctypes.c_int
        L.oracle_cycles_list.argtypes = [i64, i64, ctypes.POINTER(i64), i64]
        L.oracle_cycles_list.restype = i64
        _lib = L
    return _lib


def _ptr(a: np.ndarray):
    assert a.flags.c_contiguous
    return ctypes.c_void_p(a.ctypes.data)


def _check(rc: int):
    if rc != 0:
        raise ValueError(f"oracle returned {rc}")


def eq1_dest(k: int, A: int, B: int) -> int:
    """Eq. (1): destination offset of offset k in an A x B row-major array."""
    return int(lib().oracle_eq1_dest(k, A, B))


def permute_inplace(a: np.ndarray, batch: int, A: int, B: int, s: int) -> np.ndarray:
    """P(batch, A, B, s) in place (the elementary transposition)."""
    assert a.size == batch * A * B * s, (a.size, batch, A, B, s)
    _check(lib().oracle_permute_inplace(_ptr(a), batch, A, B, s, a.itemsize))
    return a


def transpose_inplace(a: np.ndarray, M: int, N: int) -> np.ndarray:
    """Full in-place transpose by cycle following."""
    assert a.size == M * N
    _check(lib().oracle_transpose_inplace(_ptr(a), M, N, a.itemsize))
    return a


def transpose_3stage(a: np.ndarray, M: int, N: int, m: int, n: int) -> np.ndarray:
    """The paper's 3-stage algorithm (Sec. 4.2) with tiles (m, n)."""
    _check(lib().oracle_transpose_3stage(_ptr(a), M, N, m, n, a.itemsize))
    return a


def transpose_4stage(a: np.ndarray, M: int, N: int, m: int, n: int) -> np.ndarray:
    """The 4-stage Gustavson/Karlsson sequence (Fig. 2)."""
    _check(lib().oracle_transpose_4stage(_ptr(a), M, N, m, n, a.itemsize))
    return a


def cycle_stats(M: int, N: int):
    """(#cycles, #fixed points, longest cycle) of the M x N transposition."""
    c, f, L = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int64()
    _check(lib().oracle_cycle_stats(M, N, ctypes.byref(c), ctypes.byref(f), ctypes.byref(L)))
    return c.value, f.value, L.value


def cycles_list(M: int, N: int):
    """The cycles of the M x N transposition, each from its smallest offset."""
    cap = 2 * M * N + 2
    buf = (ctypes.c_int64 * cap)()
    w = lib().oracle_cycles_list(M, N, buf, cap)
    if w < 0:
        raise ValueError("oracle_cycles_list failed")
    out, cur = [], []
    for v in buf[:w]:
        if v == -1:
            out.append(tuple(cur))
            cur = []
        else:
            cur.append(int(v))
    return out


def dtype_for(elem_bytes: int):
    return _DTYPES[elem_bytes]
