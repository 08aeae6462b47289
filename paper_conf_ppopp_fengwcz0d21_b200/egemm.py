"""Thin Python binding of libegemm.so (include/egemm.h): argument marshalling only.

Every compute step runs in the CUDA kernels behind the C ABI.  PyTorch supplies device
memory, the current stream and (in ``distributed``) process groups.  There is no CPU
fallback: if the library is missing or the device is not an sm_100 GPU, calls raise.
"""
from __future__ import annotations

import ctypes
import os

import torch

_PKG = os.path.dirname(os.path.abspath(__file__))
# EGEMM_LIB_PATH: load another build of the same library (A/B experiments in tools/)
LIB_PATH = os.environ.get("EGEMM_LIB_PATH") or os.path.join(_PKG, "libegemm.so")

OK, ERR_INVALID_ARG, ERR_UNSUPPORTED, ERR_CUDA, ERR_WORKSPACE = 0, 1, 2, 3, 4


class EgemmError(RuntimeError):
    def __init__(self, status: int, fn: str, detail: str):
        super().__init__("%s -> %s: %s" % (fn, _STATUS.get(status, status), detail))
        self.status = status


_STATUS = {0: "EGEMM_OK", 1: "EGEMM_ERR_INVALID_ARG", 2: "EGEMM_ERR_UNSUPPORTED",
           3: "EGEMM_ERR_CUDA", 4: "EGEMM_ERR_WORKSPACE"}


class Operand(ctypes.Structure):
    """egemm_operand_t"""
    _fields_ = [("f32", ctypes.c_void_p), ("hi", ctypes.c_void_p), ("lo", ctypes.c_void_p),
                ("ld", ctypes.c_int64), ("trans", ctypes.c_int), ("ld_split", ctypes.c_int64)]


class Config(ctypes.Structure):
    """egemm_config_t (0 / -1 = not set, the tuning table's value)."""
    _fields_ = [(n, ctypes.c_int) for n in ("cg", "bn", "sep", "kc", "stages", "fused", "terms",
                                            "n_slices", "epi_warps", "a_resident", "pace",
                                            "max_clusters", "operand_format", "tail_peel", "ksplit",
                                            "tail_split")]


EXPORTS = ["egemm_status_string", "egemm_last_error", "egemm_version", "egemm_split",
           "egemm_split_trunc", "egemm_gemm",
           "egemm_gemm_workspace_size", "egemm_knn", "egemm_knn_workspace_size", "egemm_knn_index",
           "egemm_kmeans_step", "egemm_kmeans_workspace_size", "egemm_kmeans_finalize",
           "egemm_set_config", "egemm_num_sms", "egemm_debug_last_clock", "egemm_tune_table",
           "egemm_debug_clock_stats", "egemm_debug_counter", "egemm_debug_timeline", "egemm_tc_probe",
           "egemm_query_config", "egemm_gemm_host", "egemm_gemm_host_workspace_size",
           "egemm_set_config_ex", "egemm_query_config_ex", "egemm_knn_merge", "egemm_split_bf16",
           "egemm_kmeans_allreduce_finalize"]

_lib = None


def load(path: str = LIB_PATH):
    """Load libegemm.so (raises if it was not built: there is no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise RuntimeError("libegemm.so not built (run python -m paper_conf_ppopp_fengwcz0d21_b200.build)")
    L = ctypes.CDLL(path)
    P, I64, I, SZ = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int, ctypes.c_size_t
    L.egemm_status_string.argtypes = [I]
    L.egemm_status_string.restype = ctypes.c_char_p
    L.egemm_last_error.argtypes = []
    L.egemm_last_error.restype = ctypes.c_char_p
    L.egemm_version.restype = I
    L.egemm_split.argtypes = [P, I64, I64, I64, P, P, I64, I, P, P]
    L.egemm_split.restype = I
    L.egemm_split_trunc.argtypes = [P, I64, I64, I64, P, P, I64, I, P, P]
    L.egemm_split_trunc.restype = I
    L.egemm_split_bf16.argtypes = [P, I64, I64, I64, P, P, I64, I, P]
    L.egemm_split_bf16.restype = I
    L.egemm_gemm.argtypes = [I64, I64, I64, Operand, Operand, P, I64, P, I64, I, P, SZ, P]
    L.egemm_gemm.restype = I
    L.egemm_gemm_workspace_size.argtypes = [I64, I64, I64, I, I]
    L.egemm_gemm_workspace_size.restype = SZ
    L.egemm_knn.argtypes = [Operand, P, I64, Operand, I64, I64, I, P, P, P, SZ, P]
    L.egemm_knn.restype = I
    L.egemm_knn_workspace_size.argtypes = [I64, I64, I64, I, I]
    L.egemm_knn_workspace_size.restype = SZ
    L.egemm_knn_index.argtypes = [P, I64, I64, I64, P, P, I64, P, P]
    L.egemm_knn_index.restype = I
    L.egemm_kmeans_step.argtypes = [Operand, I64, I64, P, I64, P, P, P, P, P, SZ, P]
    L.egemm_kmeans_step.restype = I
    L.egemm_kmeans_workspace_size.argtypes = [I64, I64, I64, I]
    L.egemm_kmeans_workspace_size.restype = SZ
    L.egemm_kmeans_finalize.argtypes = [P, P, I64, I64, P, P]
    L.egemm_kmeans_finalize.restype = I
    L.egemm_set_config.argtypes = [I, I, I, I]
    L.egemm_set_config.restype = I
    L.egemm_num_sms.restype = I
    L.egemm_debug_last_clock.argtypes = [ctypes.POINTER(ctypes.c_double)]
    L.egemm_debug_last_clock.restype = I
    L.egemm_tc_probe.argtypes = [I, I, I, P, P, P, P, P]
    L.egemm_tc_probe.restype = I
    DP = ctypes.POINTER(ctypes.c_double)
    L.egemm_debug_clock_stats.argtypes = [DP, DP, DP, I]
    L.egemm_debug_clock_stats.restype = I
    L.egemm_debug_counter.argtypes = [ctypes.POINTER(ctypes.c_ulonglong), I]
    L.egemm_debug_counter.restype = I
    L.egemm_debug_timeline.argtypes = [ctypes.POINTER(ctypes.c_ulonglong), I]
    L.egemm_debug_timeline.restype = I
    L.egemm_gemm_host.argtypes = [I64, I64, I64, P, I64, P, I64, P, I64, I, P, SZ, P]
    L.egemm_gemm_host.restype = I
    L.egemm_gemm_host_workspace_size.argtypes = [I64, I64, I64]
    L.egemm_gemm_host_workspace_size.restype = SZ
    L.egemm_tune_table.argtypes = [ctypes.POINTER(ctypes.c_int)]
    L.egemm_tune_table.restype = ctypes.c_char_p
    IP = ctypes.POINTER(ctypes.c_int)
    L.egemm_query_config.argtypes = [I, I64, I64, I64, IP, IP, IP, IP, IP]
    L.egemm_query_config.restype = I
    L.egemm_set_config_ex.argtypes = [ctypes.POINTER(Config)]
    L.egemm_set_config_ex.restype = I
    L.egemm_query_config_ex.argtypes = [I, I64, I64, I64, ctypes.POINTER(Config)]
    L.egemm_query_config_ex.restype = I
    L.egemm_knn_merge.argtypes = [P, P, I, I64, I, I, P, P, P, P]
    L.egemm_knn_merge.restype = I
    L.egemm_kmeans_allreduce_finalize.argtypes = [ctypes.POINTER(ctypes.c_void_p),
                                                  ctypes.POINTER(ctypes.c_void_p), I, I64, I64, P,
                                                  P, P, P]
    L.egemm_kmeans_allreduce_finalize.restype = I
    _lib = L
    return L


def tune_table():
    """(path of the loaded tune_table.json or '', number of entries)."""
    n = ctypes.c_int(0)
    p = load().egemm_tune_table(ctypes.byref(n))
    return p.decode(), n.value


def query_config(op: str, M: int, N: int, K: int, with_fused: bool = False):
    """The (cg, bn, sep, kc) the library picks for op in {'gemm' (pre-split B), 'knn',
    'kmeans', 'gemm_b32' (fp32 B split inside the call)} (+ the fused-split flag when
    with_fused: 1 = A, 2 = B round-split inside the GEMM kernel, 0 = none)."""
    v = [ctypes.c_int(0) for _ in range(5)]
    _check(load().egemm_query_config({"gemm": 0, "knn": 1, "kmeans": 2, "gemm_b32": 3}[op], M, N, K,
                                     *[ctypes.byref(x) for x in v]), "egemm_query_config")
    out = tuple(x.value for x in v)
    return out if with_fused else out[:4]


OPS = {"gemm": 0, "knn": 1, "kmeans": 2, "gemm_b32": 3}


def query_config_ex(op: str, M: int, N: int, K: int) -> dict:
    """The full launch configuration (egemm_config_t as a dict) the library picks for op."""
    c = Config()
    _check(load().egemm_query_config_ex(OPS[op], M, N, K, ctypes.byref(c)), "egemm_query_config_ex")
    return {n: getattr(c, n) for n, _ in Config._fields_}


def set_config_ex(**fields):
    """Thread-local override of the tuning table: any egemm_config_t field (cg, bn, sep, kc,
    stages, fused, terms, n_slices, epi_warps, a_resident, pace, max_clusters); no arguments
    restores the table.  fused / a_resident / pace default to -1 (the table's)."""
    if not fields:
        _check(load().egemm_set_config_ex(None), "egemm_set_config_ex")
        return
    c = Config()
    c.fused = c.a_resident = c.pace = c.tail_peel = c.tail_split = -1
    c.operand_format = 0
    for k, v in fields.items():
        if k not in dict(Config._fields_):
            raise TypeError("unknown config field %r" % k)
        setattr(c, k, int(v))
    _check(load().egemm_set_config_ex(ctypes.byref(c)), "egemm_set_config_ex")


PROBE_KINDS = {"f16": 0, "bf16": 1, "tf32": 2}


def tc_probe(kind: str, A: torch.Tensor, B: torch.Tensor, C: torch.Tensor | None = None,
             stream=None) -> torch.Tensor:
    """One tcgen05.mma chain D = C + A @ B^T on a single CTA (M = 128) in the MMA's own
    arithmetic -- the precision-profiling probe of Sec. 3.1 (egemm_tc_probe).  A [128, K] and
    B [N, K] are fp16 / bf16 (kinds "f16" / "bf16") or fp32 holding tf32 values ("tf32")."""
    L = load()
    _need_cuda(A, B)
    k = PROBE_KINDS[kind]
    dt = {0: torch.float16, 1: torch.bfloat16, 2: torch.float32}[k]
    assert A.dtype == dt and B.dtype == dt and A.shape[0] == 128 and A.shape[1] == B.shape[1]
    A, B = A.contiguous(), B.contiguous()
    if C is not None:
        C = C.contiguous().float()
    N, K = B.shape
    D = torch.empty((128, N), dtype=torch.float32, device=A.device)
    _check(L.egemm_tc_probe(k, N, K, _ptr(A), _ptr(B), _ptr(C), _ptr(D), _stream(stream)),
           "egemm_tc_probe")
    return D


def debug_clock_stats(reset: bool = True):
    """(mean SM MHz, CTA-0 cycles per launch, launches) over the tensor-core launches since
    the last reset (synchronous; debug)."""
    v = [ctypes.c_double(0.0) for _ in range(3)]
    _check(load().egemm_debug_clock_stats(*[ctypes.byref(x) for x in v], int(reset)),
           "egemm_debug_clock_stats")
    return tuple(x.value for x in v)


def debug_counter(reset: bool = True) -> int:
    """The device debug event counter (EGEMM_DIAG builds, EGEMM_DEBUG_MODE bit 256: kNN
    candidate-path entries)."""
    v = ctypes.c_ulonglong(0)
    _check(load().egemm_debug_counter(ctypes.byref(v), int(reset)), "egemm_debug_counter")
    return int(v.value)


def debug_timeline(reset: bool = True) -> list:
    """CTA 0's phase timeline of the last tensor-core launch (16 SM-clock values; recorded
    only by an EGEMM_DIAG=1 build under EGEMM_DEBUG_MODE bit 2048; see egemm.h)."""
    v = (ctypes.c_ulonglong * 16)()
    _check(load().egemm_debug_timeline(v, int(reset)), "egemm_debug_timeline")
    return [int(x) for x in v]


def debug_last_clock() -> float:
    """Effective SM clock (MHz) of CTA 0 over the last tensor-core kernel (synchronous)."""
    v = ctypes.c_double(0.0)
    _check(load().egemm_debug_last_clock(ctypes.byref(v)), "egemm_debug_last_clock")
    return v.value


def _check(status: int, fn: str):
    if status != OK:
        raise EgemmError(status, fn, load().egemm_last_error().decode())


def _ptr(t):
    return None if t is None else ctypes.c_void_p(t.data_ptr())


def _stream(stream=None):
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


def _need_cuda(*ts):
    for t in ts:
        if t is not None and not t.is_cuda:
            raise ValueError("egemm expects CUDA tensors (no CPU path)")


def _f32_rows(name, t, shape=None):
    """An fp32 CUDA matrix with unit inner stride (the C ABI sees only base, ld, sizes)."""
    if t is None:
        return
    if t.dtype != torch.float32 or t.dim() != 2 or (t.shape[1] > 1 and t.stride(1) != 1):
        raise ValueError("%s must be a 2-D float32 tensor with stride(1) == 1" % name)
    if shape is not None and tuple(t.shape) != tuple(shape):
        raise ValueError("%s has shape %s, expected %s" % (name, tuple(t.shape), tuple(shape)))


def _split_pair(name, pair, rows, cols):
    if pair is None:
        return
    hi, lo = pair
    for t in (hi, lo):
        if t.dtype not in (torch.int16, torch.float16) or t.dim() != 2 or t.stride(1) != 1:
            raise ValueError("%s hi/lo must be 2-D int16/float16 with stride(1) == 1" % name)
        if tuple(t.shape) != (rows, cols):
            raise ValueError("%s hi/lo have shape %s, expected %s" % (name, tuple(t.shape), (rows, cols)))
    if hi.stride(0) != lo.stride(0):
        raise ValueError("%s hi and lo must share the row stride" % name)


def _workspace(nbytes: int, device, ws=None):
    if nbytes == 0:
        return None, 0
    if ws is not None and ws.numel() >= nbytes:
        return ws, ws.numel()
    return torch.empty(nbytes, dtype=torch.uint8, device=device), nbytes


# ---------------------------------------------------------------------------- split
def split(x: torch.Tensor, transpose: bool = False, range_flags: torch.Tensor | None = None,
          out: tuple | None = None, stream=None, mode: str = "round"):
    """Round-split fp32 x [rows, cols] -> (hi, lo) fp16 bit patterns as int16 tensors
    (viewable as torch.float16).  transpose=True returns the [cols, rows] transpose.
    mode="trunc": the Markidis truncate-split (egemm_split_trunc); mode="bf16": bf16 parts
    (egemm_split_bf16, NEXT-3)."""
    L = load()
    _need_cuda(x)
    assert x.dtype == torch.float32 and x.dim() == 2 and x.stride(1) == 1
    rows, cols = x.shape
    oshape = (cols, rows) if transpose else (rows, cols)
    if out is None:
        hi = torch.empty(oshape, dtype=torch.int16, device=x.device)
        lo = torch.empty(oshape, dtype=torch.int16, device=x.device)
    else:
        hi, lo = out
    if mode == "bf16":
        assert range_flags is None
        _check(L.egemm_split_bf16(_ptr(x), rows, cols, x.stride(0), _ptr(hi), _ptr(lo), hi.stride(0),
                                  1 if transpose else 0, _stream(stream)), "egemm_split_bf16")
        return hi, lo
    fn = {"round": L.egemm_split, "trunc": L.egemm_split_trunc}[mode]
    _check(fn(_ptr(x), rows, cols, x.stride(0), _ptr(hi), _ptr(lo), hi.stride(0),
              1 if transpose else 0, _ptr(range_flags), _stream(stream)), "egemm_split")
    return hi, lo


def operand(f32: torch.Tensor | None = None, hi=None, lo=None, trans: bool = False) -> Operand:
    op = Operand()
    op.f32 = f32.data_ptr() if f32 is not None else None
    op.hi = hi.data_ptr() if hi is not None else None
    op.lo = lo.data_ptr() if lo is not None else None
    op.ld = f32.stride(0) if f32 is not None else (hi.shape[1] if hi is not None else 0)
    op.trans = 1 if trans else 0
    op.ld_split = hi.stride(0) if hi is not None else 0
    return op


# ---------------------------------------------------------------------------- GEMM
def gemm_workspace_size(M, N, K, a_presplit=False, b_presplit=False) -> int:
    return int(load().egemm_gemm_workspace_size(M, N, K, int(a_presplit), int(b_presplit)))


def gemm(A: torch.Tensor | None, B: torch.Tensor | None, C: torch.Tensor | None = None,
         terms: int = 0, out: torch.Tensor | None = None, a_split=None, b_split=None,
         b_trans: bool = False, workspace: torch.Tensor | None = None, stream=None):
    """D = A @ B (+ C) with the EGEMM-TC emulation (Alg. 1).

    A: [M, K] fp32 (or a_split=(hi, lo) [M, K]); B: [K, N] fp32, or [N, K] with b_trans,
    or b_split=(hi, lo) [N, K] (K-major, e.g. split(B, transpose=True))."""
    L = load()
    if A is not None:
        M, K = A.shape
    else:
        M, K = a_split[0].shape
    if B is not None:
        N = B.shape[0] if b_trans else B.shape[1]
        KB = B.shape[1] if b_trans else B.shape[0]
    else:
        N, KB = b_split[0].shape
    if KB != K:
        raise ValueError("inner dimensions differ: A has K=%d, B has K=%d" % (K, KB))
    _f32_rows("A", A)
    _f32_rows("B", B)
    _split_pair("a_split", a_split, M, K)
    _split_pair("b_split", b_split, N, K)
    _f32_rows("C", C, (M, N))
    _f32_rows("out", out, (M, N))
    dev = (A if A is not None else a_split[0]).device
    _need_cuda(A, B, C, out)
    D = out if out is not None else torch.empty((M, N), dtype=torch.float32, device=dev)
    opA = operand(A, *(a_split or (None, None)))
    opB = operand(B, *(b_split or (None, None)), trans=b_trans)
    need = gemm_workspace_size(M, N, K, a_split is not None, b_split is not None)
    ws, wsn = _workspace(need, dev, workspace)
    _check(L.egemm_gemm(M, N, K, opA, opB, _ptr(C), C.stride(0) if C is not None else 0, _ptr(D),
                        D.stride(0), int(terms), _ptr(ws), wsn, _stream(stream)), "egemm_gemm")
    return D


def gemm_host_workspace_size(M, N, K) -> int:
    return int(load().egemm_gemm_host_workspace_size(M, N, K))


def gemm_host(A: torch.Tensor, B: torch.Tensor, out: torch.Tensor | None = None, terms: int = 0,
              workspace: torch.Tensor | None = None, device=None, stream=None):
    """D = A @ B on HOST (preferably pinned) fp32 tensors through egemm_gemm_host: the copies
    are pipelined against the GPU work inside the library.  Asynchronous: synchronise the
    stream before reading ``out``."""
    L = load()
    assert not A.is_cuda and not B.is_cuda
    _f32_rows("A", A)
    _f32_rows("B", B)
    M, K = A.shape
    N = B.shape[1]
    if B.shape[0] != K:
        raise ValueError("inner dimensions differ: A has K=%d, B has K=%d" % (K, B.shape[0]))
    if out is not None and (out.is_cuda or out.dtype != torch.float32 or tuple(out.shape) != (M, N)
                            or out.stride(1) != 1):
        raise ValueError("out must be a host float32 [M, N] tensor with stride(1) == 1")
    D = out if out is not None else torch.empty((M, N), dtype=torch.float32, pin_memory=True)
    dev = device or torch.device("cuda", torch.cuda.current_device())
    ws, wsn = _workspace(gemm_host_workspace_size(M, N, K), dev, workspace)
    _check(L.egemm_gemm_host(M, N, K, _ptr(A), A.stride(0), _ptr(B), B.stride(0), _ptr(D),
                             D.stride(0), int(terms), _ptr(ws), wsn, _stream(stream)),
           "egemm_gemm_host")
    return D


# ---------------------------------------------------------------------------- kNN
def knn_workspace_size(nx, nq, d, k, x_presplit=False) -> int:
    return int(load().egemm_knn_workspace_size(nx, nq, d, k, int(x_presplit)))


def knn_index(X: torch.Tensor, stream=None):
    """Index build for kNN: (hi, lo, norms) of the references X [nx, d] (done once)."""
    L = load()
    _need_cuda(X)
    nx, d = X.shape
    ld = (d + 7) // 8 * 8
    hi = torch.empty((nx, ld), dtype=torch.int16, device=X.device)[:, :d]
    lo = torch.empty((nx, ld), dtype=torch.int16, device=X.device)[:, :d]
    norms = torch.empty(nx, dtype=torch.float32, device=X.device)
    _check(L.egemm_knn_index(_ptr(X), nx, d, X.stride(0), _ptr(hi), _ptr(lo), ld, _ptr(norms),
                             _stream(stream)), "egemm_knn_index")
    return hi, lo, norms


def knn(X: torch.Tensor | None, Q: torch.Tensor, k: int, x_split=None, index=None, workspace=None,
        out=None, stream=None):
    """k nearest rows of X [nx, d] for each query row of Q [nq, d] (squared L2, ascending).
    Pass ``index=knn_index(X)`` to reuse the split references and their norms (X may then
    be None).  Returns (idx int32 [nq, k], dist fp32 [nq, k])."""
    L = load()
    _need_cuda(X, Q)
    _f32_rows("Q", Q)
    nq, d = Q.shape
    if index is not None:
        hi, lo, norms = index
        nx = hi.shape[0]
        _split_pair("index", (hi, lo), nx, d)
        if norms.dtype != torch.float32 or norms.numel() != nx:
            raise ValueError("index norms must be float32 [nx]")
        opX = operand(X, hi, lo)
    else:
        nx = X.shape[0]
        norms = None
        _split_pair("x_split", x_split, nx, d)
        opX = operand(X, *(x_split or (None, None)))
    if X is not None:
        _f32_rows("X", X, (nx, d))
    if out is None:
        idx = torch.empty((nq, k), dtype=torch.int32, device=Q.device)
        dist = torch.empty((nq, k), dtype=torch.float32, device=Q.device)
    else:
        idx, dist = out
        if idx.dtype != torch.int32 or dist.dtype != torch.float32 or tuple(idx.shape) != (nq, k) \
                or tuple(dist.shape) != (nq, k) or not idx.is_contiguous() or not dist.is_contiguous():
            raise ValueError("out must be contiguous (int32 [nq, k], float32 [nq, k])")
    need = knn_workspace_size(nx, nq, d, k, index is not None or x_split is not None)
    ws, wsn = _workspace(need, Q.device, workspace)
    _check(L.egemm_knn(opX, _ptr(norms), nx, operand(Q), nq, d, k, _ptr(idx), _ptr(dist), _ptr(ws),
                       wsn, _stream(stream)), "egemm_knn")
    return idx, dist


# ---------------------------------------------------------------------------- kMeans
def kmeans_workspace_size(n, d, kc, x_presplit=False) -> int:
    return int(load().egemm_kmeans_workspace_size(n, d, kc, int(x_presplit)))


def kmeans_step(X: torch.Tensor, centroids: torch.Tensor, x_split=None, want_inertia=True,
                workspace=None, out=None, stream=None):
    """One local Lloyd step: (assign int32 [n], sums fp64 [kc, d], counts int64 [kc],
    inertia fp64 [1] or None)."""
    L = load()
    _need_cuda(X, centroids)
    _f32_rows("X", X)
    n, d = X.shape
    kc = centroids.shape[0]
    _f32_rows("centroids", centroids, (kc, d))
    if not centroids.is_contiguous():
        raise ValueError("centroids must be contiguous")
    _split_pair("x_split", x_split, n, d)
    if out is None:
        assign = torch.empty(n, dtype=torch.int32, device=X.device)
        sums = torch.empty((kc, d), dtype=torch.float64, device=X.device)
        counts = torch.empty(kc, dtype=torch.int64, device=X.device)
        inertia = torch.empty(1, dtype=torch.float64, device=X.device) if want_inertia else None
    else:
        assign, sums, counts, inertia = out
        if assign.dtype != torch.int32 or assign.numel() != n or sums.dtype != torch.float64 or \
                tuple(sums.shape) != (kc, d) or counts.dtype != torch.int64 or counts.numel() != kc:
            raise ValueError("out must be (int32 [n], float64 [kc, d], int64 [kc], float64 [1] | None)")
    need = kmeans_workspace_size(n, d, kc, x_split is not None)
    ws, wsn = _workspace(need, X.device, workspace)
    _check(L.egemm_kmeans_step(operand(X, *(x_split or (None, None))), n, d, _ptr(centroids), kc,
                               _ptr(assign), _ptr(sums), _ptr(counts), _ptr(inertia), _ptr(ws),
                               wsn, _stream(stream)), "egemm_kmeans_step")
    return assign, sums, counts, inertia


def kmeans_finalize(sums: torch.Tensor, counts: torch.Tensor, centroids: torch.Tensor, stream=None):
    L = load()
    kc, d = centroids.shape
    if sums.dtype != torch.float64 or tuple(sums.shape) != (kc, d) or not sums.is_contiguous() or \
            counts.dtype != torch.int64 or counts.numel() != kc or not centroids.is_contiguous() or \
            centroids.dtype != torch.float32:
        raise ValueError("kmeans_finalize: sums float64 [kc, d], counts int64 [kc], centroids float32 [kc, d]")
    _check(L.egemm_kmeans_finalize(_ptr(sums), _ptr(counts), kc, d, _ptr(centroids),
                                   _stream(stream)), "egemm_kmeans_finalize")
    return centroids


def knn_merge(keys: torch.Tensor, idx: torch.Tensor, k: int, qnorm: torch.Tensor | None = None,
              stream=None):
    """Merge sorted partial lists keys / idx [n_lists, nq, k_in] (ascending (key, idx) per
    list, idx -1 = empty, indices distinct across lists) into the top k per query
    (egemm_knn_merge).  With qnorm [nq] the output keys become max(0, qnorm + key)."""
    L = load()
    _need_cuda(keys, idx, qnorm)
    if keys.dtype != torch.float32 or idx.dtype != torch.int32 or keys.dim() != 3 or \
            keys.shape != idx.shape or not keys.is_contiguous() or not idx.is_contiguous():
        raise ValueError("keys float32 / idx int32, contiguous [n_lists, nq, k_in]")
    nl, nq, k_in = keys.shape
    if qnorm is not None and (qnorm.dtype != torch.float32 or qnorm.numel() != nq):
        raise ValueError("qnorm must be float32 [nq]")
    oi = torch.empty((nq, k), dtype=torch.int32, device=keys.device)
    ok = torch.empty((nq, k), dtype=torch.float32, device=keys.device)
    _check(L.egemm_knn_merge(_ptr(keys), _ptr(idx), nl, nq, k_in, k, _ptr(qnorm), _ptr(oi), _ptr(ok),
                             _stream(stream)), "egemm_knn_merge")
    return oi, ok


def kmeans_allreduce_finalize(peer_sums, peer_counts, centroids: torch.Tensor, sums_out=None,
                              counts_out=None, stream=None):
    """The kMeans exchange step fused with the update over peer memory
    (egemm_kmeans_allreduce_finalize): peer_sums / peer_counts are lists of the ranks' partial
    (kc x d fp64, kc int64) tensors readable from this device (e.g. torch SymmetricMemory peer
    buffers); reduced in rank order (bitwise identical on every rank), then finalized."""
    L = load()
    kc, d = centroids.shape
    n = len(peer_sums)
    for t in list(peer_sums) + list(peer_counts):
        _need_cuda(t)
    if n != len(peer_counts) or any(t.dtype != torch.float64 or t.numel() != kc * d for t in peer_sums) or \
            any(t.dtype != torch.int64 or t.numel() != kc for t in peer_counts):
        raise ValueError("peer_sums: float64 [kc, d] each; peer_counts: int64 [kc] each")
    ps = (ctypes.c_void_p * n)(*[t.data_ptr() for t in peer_sums])
    pc = (ctypes.c_void_p * n)(*[t.data_ptr() for t in peer_counts])
    _check(L.egemm_kmeans_allreduce_finalize(ps, pc, n, kc, d, _ptr(sums_out), _ptr(counts_out),
                                             _ptr(centroids), _stream(stream)),
           "egemm_kmeans_allreduce_finalize")
    return centroids


def set_config(cg: int = 0, bn: int = 0, sep: int = 0, kc: int = 0):
    """Per-thread tile-config override (all zeros = tuning table)."""
    _check(load().egemm_set_config(cg, bn, sep, kc), "egemm_set_config")


def num_sms() -> int:
    return int(load().egemm_num_sms())
