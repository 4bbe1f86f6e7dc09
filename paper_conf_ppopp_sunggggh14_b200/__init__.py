"""paper_conf_ppopp_sunggggh14_b200 -- Python binding of libipt (B200-native in-place
transposition, Sung et al. PPoPP'14).

Argument marshalling only: every step of the transposition runs in libipt's CUDA kernels
(``csrc/``), called through the C ABI declared in ``include/ipt.h``.  PyTorch supplies
device memory and streams.  There is no CPU fallback: if ``libipt.so`` is missing the
import of ``lib()`` raises, and every call on a tensor that is not on a CUDA device
raises.

Function names follow the ABI (and the paper's factorial numbering):

    transpose_(t, M, N)                  A (M x N) -> A^T (N x M) in place, returns view
    transpose_batched_(t, count, M, N)   count independent matrices
    ipt_100_(t, batch, A, B, s)          100!  batch x [A x B x s] -> batch x [B x A x s]
    ipt_010_(t, batch, A, B)             010!  batch x [A x B]     -> batch x [B x A]
    ipt_0010_(t, d0, d1, d2, d3)         0010! d0 x d1 x d2 x d3   -> d0 x d1 x d3 x d2
    ipt_0100_(t, d0, d1, d2, d3)         0100! d0 x d1 x d2 x d3   -> d0 x d2 x d1 x d3
    ipt_1000_(t, d0, d1, d2, d3)         1000! d0 x d1 x d2 x d3   -> d1 x d0 x d2 x d3
    plan(M, N, elem_bytes, device)       the tile-size planner's choice (dict)
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libipt.so")

IPT_OK = 0
VARIANTS = {0: "identity", 1: "tile_onchip", 3: "cycle_global", 4: "square_swap"}   # 2: reserved


class IptError(RuntimeError):
    pass


class Plan(ctypes.Structure):
    _fields_ = [
        ("M", ctypes.c_int64), ("N", ctypes.c_int64),
        ("m", ctypes.c_int64), ("n", ctypes.c_int64),
        ("Mp", ctypes.c_int64), ("Np", ctypes.c_int64),
        ("elem_bytes", ctypes.c_int32), ("n_stages", ctypes.c_int32),
        ("variant", ctypes.c_int32 * 3), ("reserved", ctypes.c_int32),
        ("flag_bits", ctypes.c_int64 * 3),
        ("workspace_bytes", ctypes.c_uint64),
    ]

    def as_dict(self):
        return {
            "M": self.M, "N": self.N, "m": self.m, "n": self.n, "Mp": self.Mp, "Np": self.Np,
            "elem_bytes": self.elem_bytes, "n_stages": self.n_stages,
            "variant": [VARIANTS[v] for v in self.variant],
            "flag_bits": list(self.flag_bits), "workspace_bytes": self.workspace_bytes,
        }


_lib = None

# (name, restype, argtypes) of every symbol declared in include/ipt.h
_i64, _int, _vp, _sz = ctypes.c_int64, ctypes.c_int, ctypes.c_void_p, ctypes.c_size_t
ABI = [
    ("ipt_plan", _int, [_i64, _i64, _int, _int, ctypes.POINTER(Plan)]),
    ("ipt_plan_with_tiles", _int, [_i64, _i64, _i64, _i64, _int, _int, ctypes.POINTER(Plan)]),
    ("ipt_plan_autotune", _int, [_vp, _i64, _i64, _int, _int, _vp, ctypes.POINTER(Plan)]),
    ("ipt_plan_autotune_batched", _int, [_vp, _i64, _i64, _i64, _i64, _int, _int, _vp, ctypes.POINTER(Plan)]),
    ("ipt_workspace_bytes", _sz, [ctypes.POINTER(Plan), _i64]),
    ("ipt_transpose", _int, [_vp, _i64, _i64, _int, _vp]),
    ("ipt_transpose_plan", _int, [_vp, ctypes.POINTER(Plan), _vp, _sz, _vp]),
    ("ipt_transpose_plan_events", _int, [_vp, ctypes.POINTER(Plan), _vp, _sz, _vp, ctypes.POINTER(_vp)]),
    ("ipt_transpose_batched", _int, [_vp, _i64, _i64, _i64, _i64, _int, _vp]),
    ("ipt_transpose_batched_plan", _int, [_vp, _i64, _i64, ctypes.POINTER(Plan), _vp, _sz, _vp]),
    ("ipt_transpose_batched_plan_events", _int,
     [_vp, _i64, _i64, ctypes.POINTER(Plan), _vp, _sz, _vp, ctypes.POINTER(_vp)]),
    ("ipt_transpose_4stage", _int, [_vp, _i64, _i64, _i64, _i64, _int, _vp, _sz, _vp]),
    ("ipt_transpose_host", _int, [_vp, _i64, _i64, _int, _int, _vp, _sz, _vp]),
    ("ipt_transpose_host_async", _int, [_vp, _i64, _i64, _int, _int, _vp, _sz, _vp]),
    ("ipt_transpose_host_pipeline", _int,
     [ctypes.POINTER(_vp), ctypes.POINTER(_i64), ctypes.POINTER(_i64), _int, _int, _vp, _sz, _vp]),
    ("ipt_graph_create", _int, [_vp, _i64, _i64, ctypes.POINTER(Plan), _vp, _sz, ctypes.POINTER(_vp)]),
    ("ipt_graph_launch", _int, [_vp, _vp]),
    ("ipt_graph_destroy", _int, [_vp]),
    ("ipt_stage_workspace_bytes", _sz, [_i64, _i64, _i64, _i64, _int]),
    ("ipt_100", _int, [_vp, _i64, _i64, _i64, _i64, _int, _vp, _sz, _vp]),
    ("ipt_010", _int, [_vp, _i64, _i64, _i64, _int, _vp, _sz, _vp]),
    ("ipt_0010", _int, [_vp, _i64, _i64, _i64, _i64, _int, _vp, _sz, _vp]),
    ("ipt_0100", _int, [_vp, _i64, _i64, _i64, _i64, _int, _vp, _sz, _vp]),
    ("ipt_1000", _int, [_vp, _i64, _i64, _i64, _i64, _int, _vp, _sz, _vp]),
    ("ipt_aos_to_asta", _int, [_vp, _i64, _i64, _i64, _int, _vp, _sz, _vp]),
    ("ipt_asta_to_aos", _int, [_vp, _i64, _i64, _i64, _int, _vp, _sz, _vp]),
    ("ipt_soa_to_asta", _int, [_vp, _i64, _i64, _i64, _int, _vp, _sz, _vp]),
    ("ipt_asta_to_soa", _int, [_vp, _i64, _i64, _i64, _int, _vp, _sz, _vp]),
    ("ipt_status_string", ctypes.c_char_p, [_int]),
    ("ipt_kernel_launch_count", ctypes.c_uint64, []),
    ("ipt_last_cuda_error", ctypes.c_char_p, []),
    ("ipt_version", ctypes.c_char_p, []),
]


def lib():
    """Load libipt.so (in-tree).  Raises if it has not been built -- no fallback."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise IptError(
                f"{LIB_PATH} not found: build it with `python -m paper_conf_ppopp_sunggggh14_b200.build`"
            )
        L = ctypes.CDLL(LIB_PATH)
        for name, res, args in ABI:
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        L.ipt__stage_kernel.restype = ctypes.c_int
        L.ipt__stage_kernel.argtypes = [ctypes.POINTER(Plan), _i64, _vp, _int, ctypes.c_char_p, _int]
        L.ipt__fastdiv.restype = ctypes.c_uint64
        L.ipt__fastdiv.argtypes = [ctypes.c_uint64, ctypes.c_uint64]
        L.ipt__fastdiv32.restype = ctypes.c_uint32
        L.ipt__fastdiv32.argtypes = [ctypes.c_uint32, ctypes.c_uint32]
        _lib = L
    return _lib


def _check(rc: int, what: str):
    if rc != IPT_OK:
        msg = lib().ipt_status_string(rc).decode()
        if msg == "IPT_ERR_CUDA":
            msg += f" ({lib().ipt_last_cuda_error().decode()})"
        raise IptError(f"{what}: {msg}")


def _stream_ptr(stream):
    import torch

    if stream is None:
        stream = torch.cuda.current_stream()
    return ctypes.c_void_p(stream.cuda_stream)


def _dev_ptr(t):
    if not t.is_cuda:
        raise IptError("libipt operates on CUDA tensors only (no CPU fallback)")
    if not t.is_contiguous():
        raise IptError("tensor must be contiguous")
    return ctypes.c_void_p(t.data_ptr())


def _events_arr(events):
    arr = (ctypes.c_void_p * 4)()
    for i, e in enumerate(events or []):
        if e is not None and not e.cuda_event:
            e.record()   # torch creates the cudaEvent_t lazily, on its first record
        arr[i] = ctypes.c_void_p(e.cuda_event) if e is not None else None
    return arr


# ------------------------------------------------------------------------- planning
def plan(M: int, N: int, elem_bytes: int, device: int = -1, m: int | None = None,
         n: int | None = None) -> Plan:
    p = Plan()
    if m is None and n is None:
        _check(lib().ipt_plan(M, N, elem_bytes, device, ctypes.byref(p)), "ipt_plan")
    else:
        _check(lib().ipt_plan_with_tiles(M, N, m, n, elem_bytes, device, ctypes.byref(p)),
               "ipt_plan_with_tiles")
    return p


def plan_autotune(t, M: int, N: int, candidates: int = 4, stream=None,
                  elem_bytes: int | None = None) -> Plan:
    """Time the cost model's best candidate plans on t (data unchanged on return) and
    remember the fastest for (M, N, elem_bytes, device)."""
    eb = _eb(t, elem_bytes)
    p = Plan()
    _check(lib().ipt_plan_autotune(_dev_ptr(t), M, N, eb, candidates, _stream_ptr(stream),
                                   ctypes.byref(p)), "ipt_plan_autotune")
    return p


def plan_autotune_batched(t, count: int, M: int, N: int, candidates: int = 4,
                          stride_elems: int | None = None, stream=None,
                          elem_bytes: int | None = None) -> Plan:
    """plan_autotune for `count` matrices (data unchanged on return)."""
    eb = _eb(t, elem_bytes)
    stride = (stride_elems if stride_elems is not None else M * N) * eb
    p = Plan()
    _check(lib().ipt_plan_autotune_batched(_dev_ptr(t), count, stride, M, N, eb, candidates,
                                           _stream_ptr(stream), ctypes.byref(p)),
           "ipt_plan_autotune_batched")
    return p


def workspace_bytes(p: Plan, batch: int = 1) -> int:
    return int(lib().ipt_workspace_bytes(ctypes.byref(p), batch))


# ---------------------------------------------------------------- full transposition
def _eb(t, elem_bytes):
    return elem_bytes if elem_bytes else t.element_size()


def _nelem(t, eb):
    return t.numel() * t.element_size() // eb


def transpose_(t, M: int, N: int, plan_: Plan | None = None, workspace=None, stream=None,
               events=None, elem_bytes: int | None = None):
    """In-place A (M x N) -> A^T (N x M) on t's storage; returns t viewed as (N, M).
    elem_bytes defaults to t.element_size() (pass 16 for 16-byte elements)."""
    eb = _eb(t, elem_bytes)
    if _nelem(t, eb) != M * N:
        raise IptError(f"elements {_nelem(t, eb)} != M*N {M * N}")
    ptr, st = _dev_ptr(t), _stream_ptr(stream)
    ws = ctypes.c_void_p(workspace.data_ptr()) if workspace is not None else None
    wsb = workspace.numel() * workspace.element_size() if workspace is not None else 0
    if plan_ is None and events is None and workspace is None:
        _check(lib().ipt_transpose(ptr, M, N, eb, st), "ipt_transpose")
    else:
        p = plan_ if plan_ is not None else plan(M, N, eb, t.device.index)
        if events is None:
            _check(lib().ipt_transpose_plan(ptr, ctypes.byref(p), ws, wsb, st), "ipt_transpose_plan")
        else:
            _check(lib().ipt_transpose_plan_events(ptr, ctypes.byref(p), ws, wsb, st,
                                                   _events_arr(events)),
                   "ipt_transpose_plan_events")
    return t.view(N, M) if eb == t.element_size() else t


def transpose_batched_(t, count: int, M: int, N: int, stride_elems: int | None = None,
                       plan_: Plan | None = None, stream=None, elem_bytes: int | None = None,
                       events=None):
    """count matrices of M x N at t + i*stride (elements) -> their transposes in place.
    `events` (4 torch.cuda.Event or None) are recorded around the stages (needs plan_)."""
    eb = _eb(t, elem_bytes)
    stride = (stride_elems if stride_elems is not None else M * N) * eb
    if count and (count - 1) * (stride // eb) + M * N > _nelem(t, eb):
        raise IptError("tensor too small for the batch")
    ptr, st = _dev_ptr(t), _stream_ptr(stream)
    if events is not None:
        if plan_ is None:
            raise IptError("events need an explicit plan")
        _check(lib().ipt_transpose_batched_plan_events(ptr, count, stride, ctypes.byref(plan_),
                                                       None, 0, st, _events_arr(events)),
               "ipt_transpose_batched_plan_events")
    elif plan_ is None:
        _check(lib().ipt_transpose_batched(ptr, count, stride, M, N, eb, st),
               "ipt_transpose_batched")
    else:
        _check(lib().ipt_transpose_batched_plan(ptr, count, stride, ctypes.byref(plan_), None, 0, st),
               "ipt_transpose_batched_plan")
    return t


def transpose_4stage_(t, M: int, N: int, m: int = 0, n: int = 0, stream=None,
                      elem_bytes: int | None = None):
    """The paper's 4-stage Gustavson/Karlsson baseline on the GPU, in place."""
    eb = _eb(t, elem_bytes)
    if _nelem(t, eb) != M * N:
        raise IptError(f"elements {_nelem(t, eb)} != M*N {M * N}")
    _check(lib().ipt_transpose_4stage(_dev_ptr(t), M, N, m, n, eb, None, 0, _stream_ptr(stream)),
           "ipt_transpose_4stage")
    return t.view(N, M) if eb == t.element_size() else t


def transpose_host_(h, M: int, N: int, queues: int = 4, stream=None, elem_bytes: int | None = None):
    """Host-delegated in-place transpose (Sec. 6) of a CPU tensor (pinned for overlap):
    H2D, 3 stages on the GPU, D2H back into the same host storage.  Returns h viewed as
    (N, M)."""
    if h.is_cuda or not h.is_contiguous():
        raise IptError("transpose_host_ expects a contiguous host tensor")
    eb = _eb(h, elem_bytes)
    if _nelem(h, eb) != M * N:
        raise IptError(f"elements {_nelem(h, eb)} != M*N {M * N}")
    _check(lib().ipt_transpose_host(ctypes.c_void_p(h.data_ptr()), M, N, eb, queues, None, 0,
                                    _stream_ptr(stream)), "ipt_transpose_host")
    return h.view(N, M) if eb == h.element_size() else h


def transpose_host_async_(h, M: int, N: int, queues: int = 4, stream=None,
                          elem_bytes: int | None = None):
    """Asynchronous host-delegated transpose: enqueued on `stream` (pinned `h` required);
    synchronise the stream before reading `h`."""
    if h.is_cuda or not h.is_contiguous():
        raise IptError("transpose_host_async_ expects a contiguous host tensor")
    eb = _eb(h, elem_bytes)
    if _nelem(h, eb) != M * N:
        raise IptError(f"elements {_nelem(h, eb)} != M*N {M * N}")
    _check(lib().ipt_transpose_host_async(ctypes.c_void_p(h.data_ptr()), M, N, eb, queues, None, 0,
                                          _stream_ptr(stream)), "ipt_transpose_host_async")
    return h


def transpose_host_pipeline_(hs, shapes, stream=None, elem_bytes: int | None = None):
    """Host-delegated transposition of several host tensors (pinned for overlap) as one
    copy/compute pipeline: hs[i] holds a shapes[i] = (M, N) matrix and is overwritten with
    its transpose.  Asynchronous on `stream`; synchronise it before reading the tensors."""
    if len(hs) != len(shapes):
        raise IptError("one (M, N) per tensor")
    if not hs:
        return hs
    eb = _eb(hs[0], elem_bytes)
    for h, (M, N) in zip(hs, shapes):
        if h.is_cuda or not h.is_contiguous():
            raise IptError("transpose_host_pipeline_ expects contiguous host tensors")
        if _nelem(h, eb) != M * N:
            raise IptError(f"elements {_nelem(h, eb)} != M*N {M * N}")
    n = len(hs)
    ptrs = (ctypes.c_void_p * n)(*[h.data_ptr() for h in hs])
    Ms = (ctypes.c_int64 * n)(*[M for (M, _) in shapes])
    Ns = (ctypes.c_int64 * n)(*[N for (_, N) in shapes])
    _check(lib().ipt_transpose_host_pipeline(ptrs, Ms, Ns, n, eb, None, 0, _stream_ptr(stream)),
           "ipt_transpose_host_pipeline")
    return hs


class Graph:
    """A captured CUDA graph of one plan on fixed pointers (ipt_graph_create); launch() replays
    it on a stream.  Transpose once (uncaptured) before creating it to reuse the same
    kernels; an M x N graph pairs with an N x M one for repeated use."""

    def __init__(self, t, M: int, N: int, plan_: "Plan | None" = None, count: int = 1,
                 stride_elems: int | None = None, elem_bytes: int | None = None):
        eb = _eb(t, elem_bytes)
        p = plan_ if plan_ is not None else plan(M, N, eb, t.device.index)
        if (p.M, p.N, p.elem_bytes) != (M, N, eb):
            raise IptError(f"plan is for {p.M}x{p.N} ({p.elem_bytes} B), not {M}x{N} ({eb} B)")
        se = stride_elems if stride_elems is not None else M * N
        if count < 1 or (count > 1 and se < M * N) or (count - 1) * se + M * N > _nelem(t, eb):
            raise IptError("tensor too small for the batch (count, stride, M*N)")
        stride = se * eb
        h = ctypes.c_void_p()
        _check(lib().ipt_graph_create(_dev_ptr(t), count, stride, ctypes.byref(p), None, 0,
                                      ctypes.byref(h)), "ipt_graph_create")
        self._h, self._t, self._plan = h, t, p   # the graph records t's storage: keep it alive

    def launch(self, stream=None):
        _check(lib().ipt_graph_launch(self._h, _stream_ptr(stream)), "ipt_graph_launch")

    def __del__(self):
        try:
            if self._h:
                lib().ipt_graph_destroy(self._h)
        except Exception:
            pass


# ----------------------------------------------------------- elementary transpositions
def ipt_100_(t, batch: int, A: int, B: int, s: int, stream=None, elem_bytes: int | None = None):
    _check(lib().ipt_100(_dev_ptr(t), batch, A, B, s, _eb(t, elem_bytes), None, 0, _stream_ptr(stream)),
           "ipt_100")
    return t


def ipt_010_(t, batch: int, A: int, B: int, stream=None, elem_bytes: int | None = None):
    _check(lib().ipt_010(_dev_ptr(t), batch, A, B, _eb(t, elem_bytes), None, 0, _stream_ptr(stream)),
           "ipt_010")
    return t


def ipt_0010_(t, d0: int, d1: int, d2: int, d3: int, stream=None, elem_bytes: int | None = None):
    _check(lib().ipt_0010(_dev_ptr(t), d0, d1, d2, d3, _eb(t, elem_bytes), None, 0,
                          _stream_ptr(stream)), "ipt_0010")
    return t


def ipt_0100_(t, d0: int, d1: int, d2: int, d3: int, stream=None, elem_bytes: int | None = None):
    _check(lib().ipt_0100(_dev_ptr(t), d0, d1, d2, d3, _eb(t, elem_bytes), None, 0,
                          _stream_ptr(stream)), "ipt_0100")
    return t


def ipt_1000_(t, d0: int, d1: int, d2: int, d3: int, stream=None, elem_bytes: int | None = None):
    _check(lib().ipt_1000(_dev_ptr(t), d0, d1, d2, d3, _eb(t, elem_bytes), None, 0,
                          _stream_ptr(stream)), "ipt_1000")
    return t


# ------------------------------------------------ layout marshaling (NEXT-3)
def _marshal(name):
    def f(t, M: int, N: int, m: int, stream=None, elem_bytes: int | None = None):
        eb = _eb(t, elem_bytes)
        if _nelem(t, eb) != M * N:
            raise IptError(f"elements {_nelem(t, eb)} != M*N {M * N}")
        _check(getattr(lib(), name)(_dev_ptr(t), M, N, m, eb, None, 0, _stream_ptr(stream)), name)
        return t
    f.__name__ = name[4:] + "_"
    f.__doc__ = (f"{name}: M structures x N fields, tiles of m structures (P:140); in place.")
    return f


aos_to_asta_ = _marshal("ipt_aos_to_asta")
asta_to_aos_ = _marshal("ipt_asta_to_aos")
soa_to_asta_ = _marshal("ipt_soa_to_asta")
asta_to_soa_ = _marshal("ipt_asta_to_soa")


def stage_kernels(p: Plan, count: int = 1, t=None) -> list:
    """Names of the kernels the three stages of plan p launch for `count` packed matrices at
    t's storage (diagnostics: per-kernel attribution of stage times)."""
    out = []
    for st in range(3):
        buf = ctypes.create_string_buffer(64)
        ptr = ctypes.c_void_p(t.data_ptr()) if t is not None else None
        if lib().ipt__stage_kernel(ctypes.byref(p), count, ptr, st, buf, 64) != 0:
            raise IptError("ipt__stage_kernel: invalid plan")
        out.append(buf.value.decode())
    return out


def kernel_launch_count() -> int:
    return int(lib().ipt_kernel_launch_count())


def version() -> str:
    return lib().ipt_version().decode()
