"""Python face of the CPU oracle (ctypes over ``egemm_oracle.c``) plus the pieces that are
plain numpy / exact-rational code: error metrics, element error bounds, the parity gap
rules and the tensor-core accumulation candidate models of the precision probe.

TEST INFRASTRUCTURE ONLY (see ``oracle/__init__.py``).  Citations "P:a-b" are lines of
/root/reference/PAPER.md; "R<n>" are the readings listed in DESIGN.md.
"""
from __future__ import annotations

import ctypes
import math
import os
import subprocess
from fractions import Fraction

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "egemm_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

_lib = None


def build(force: bool = False) -> str:
    """Compile the C oracle (gcc, -O2 -fopenmp -ffp-contract=off, no fast-math)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + ".tmp%d" % os.getpid()
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fopenmp", "-ffp-contract=off",
                               "-fno-fast-math", "-fPIC", "-shared", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        P, I64, I = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int
        L.oracle_f32_to_f16_rne.argtypes = [ctypes.c_uint32]
        L.oracle_f32_to_f16_rne.restype = ctypes.c_uint16
        L.oracle_f16_to_f32.argtypes = [ctypes.c_uint16]
        L.oracle_f16_to_f32.restype = ctypes.c_uint32
        for f in ("oracle_split", "oracle_split_rha", "oracle_split_trunc"):
            getattr(L, f).argtypes = [P, I64, P, P]
            getattr(L, f).restype = I64
        for f in ("oracle_gemm64", "oracle_gemm32_naive"):
            getattr(L, f).argtypes = [I64, I64, I64, P, I64, P, I64, P, I64, P, I64]
            getattr(L, f).restype = None
        L.oracle_gemm_emu64.argtypes = [I64, I64, I64, P, I64, P, I64, P, I64, I, P, I64]
        L.oracle_gemm_emu64.restype = None
        L.oracle_knn.argtypes = [P, I64, P, I64, I64, I, P, P]
        L.oracle_knn.restype = None
        L.oracle_sqdist.argtypes = [P, I64, P, I64, I64, P]
        L.oracle_sqdist.restype = None
        L.oracle_kmeans_step.argtypes = [P, I64, I64, P, I64, P, P, P, P, P]
        L.oracle_kmeans_step.restype = None
        L.oracle_kmeans_finalize.argtypes = [P, P, I64, I64, P]
        L.oracle_kmeans_finalize.restype = None
        L.oracle_group_sums.argtypes = [P, I64, I64, P, I64, P, P]
        L.oracle_group_sums.restype = None
        L.oracle_tc_mma16.argtypes = [P, P, I, ctypes.c_float, I]
        L.oracle_tc_mma16.restype = ctypes.c_float
        L.oracle_gemm_alg1_tc.argtypes = [I64, I64, I64, P, P, P, I, I, I, P]
        L.oracle_gemm_alg1_tc.restype = None
        L.oracle_tf32_parts.argtypes = [ctypes.c_float, P, P, P]
        L.oracle_tf32_parts.restype = None
        L.oracle_norm_step.argtypes = [I64, I64, P, P, P]
        L.oracle_norm_step.restype = None
        L.oracle_num_threads.argtypes = []
        L.oracle_num_threads.restype = I
        _lib = L
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def _f32(a):
    return np.ascontiguousarray(a, dtype=np.float32)


def num_threads() -> int:
    return int(lib().oracle_num_threads())


# ---------------------------------------------------------------- split (Alg. 1 l.2-3)
def split(x, variant: str = "rne"):
    """Round-split x (fp32) -> (hi, lo) as uint16 fp16 bit patterns.  P:741-745.

    variant: "rne" (the parity reading R1), "rha" (literal round-half-away, R1),
    "trunc" (Markidis truncate-split, Fig. 4a)."""
    x = _f32(x)
    hi = np.empty(x.shape, np.uint16)
    lo = np.empty(x.shape, np.uint16)
    fn = {"rne": lib().oracle_split, "rha": lib().oracle_split_rha,
          "trunc": lib().oracle_split_trunc}[variant]
    inexact = fn(_p(x), x.size, _p(hi), _p(lo))
    if inexact:
        raise AssertionError("fp32 residual x - hi was inexact for %d elements" % inexact)
    return hi, lo


def f32_to_f16_bits(u32: int) -> int:
    return int(lib().oracle_f32_to_f16_rne(int(u32) & 0xFFFFFFFF))


def f16_bits_to_f32(h: int) -> float:
    return float(np.uint32(lib().oracle_f16_to_f32(int(h))).view(np.float32))


def h2f(bits: np.ndarray) -> np.ndarray:
    """fp16 bit patterns -> float64 values (numpy's IEEE binary16 decode)."""
    return np.asarray(bits, np.uint16).view(np.float16).astype(np.float64)


# ---------------------------------------------------------------- GEMMs (Alg. 1, Eq. 10)
def gemm64(A, B, C=None):
    """D = A @ B (+ C) in fp64, k ascending.  The exact reference (Alg. 1 semantics)."""
    A, B = _f32(A), _f32(B)
    M, K = A.shape
    K2, N = B.shape
    assert K == K2
    D = np.empty((M, N), np.float64)
    Cp = _f32(C) if C is not None else None
    lib().oracle_gemm64(M, N, K, _p(A), K, _p(B), N, _p(Cp) if Cp is not None else None, N,
                        _p(D), N)
    return D


def gemm32_naive(A, B, C=None):
    """Naive fp32 GEMM: float accumulator, k ascending, no FMA (R10; Eq. 10's V_single)."""
    A, B = _f32(A), _f32(B)
    M, K = A.shape
    _, N = B.shape
    D = np.empty((M, N), np.float32)
    Cp = _f32(C) if C is not None else None
    lib().oracle_gemm32_naive(M, N, K, _p(A), K, _p(B), N, _p(Cp) if Cp is not None else None,
                              N, _p(D), N)
    return D


def gemm_emu64(A, B, terms: int = 3, C=None):
    """sum_k of the split products (3 or 4 terms, Alg. 1 l.5-8) in fp64."""
    A, B = _f32(A), _f32(B)
    M, K = A.shape
    _, N = B.shape
    D = np.empty((M, N), np.float64)
    Cp = _f32(C) if C is not None else None
    lib().oracle_gemm_emu64(M, N, K, _p(A), K, _p(B), N, _p(Cp) if Cp is not None else None,
                            N, int(terms), _p(D), N)
    return D


# ---------------------------------------------------------------- metrics (BJ, Eq. 10)
def normwise_error(D, A, B, C64=None):
    """e = ||D - C64||_F / || |A| |B| ||_F  (BJ north_star; C64 = gemm64(A, B))."""
    if C64 is None:
        C64 = gemm64(A, B)
    absAB = np.abs(np.asarray(A, np.float64)) @ np.abs(np.asarray(B, np.float64))
    den = np.linalg.norm(absAB)
    if den == 0:
        return float(np.linalg.norm(np.asarray(D, np.float64) - C64))
    return float(np.linalg.norm(np.asarray(D, np.float64) - C64) / den)


def eq10_max_error(D, D32):
    """Eq. 10: MaxError = max |V_p - V_single|."""
    return float(np.max(np.abs(np.asarray(D, np.float64) - np.asarray(D32, np.float64))))


# ---------------------------------------------------------------- element bounds (R18)
U = 2.0 ** -24  # unit roundoff of fp32


def split_abs_bound(x):
    """|x - hi - lo| bound per element: max(2^-22 |x|, 2^-25) for |x| < 65504 (R4)."""
    return np.maximum(np.abs(np.asarray(x, np.float64)) * 2.0 ** -22, 2.0 ** -25)


def elem_bound(A, B, mma_ulps: float = 4.0, terms: int = 3):
    """Worst-case |D_gpu - (AB)_ij| (reading R18): split residuals of both operands, the
    dropped lo*lo term, and `mma_ulps` fp32 ulps of sum_k |a||b| per tensor-core MMA
    (3 MMAs per 16-wide k-step) plus the promotions and the final combine."""
    A = np.abs(np.asarray(A, np.float64))
    B = np.abs(np.asarray(B, np.float64))
    K = A.shape[1]
    eA, eB = split_abs_bound(A), split_abs_bound(B)
    absAB = A @ B
    t_split = eA @ B + A @ eB + eA @ eB
    t_lolo = 0.0 if terms == 4 else (A * 2.0 ** -11 + 2.0 ** -24) @ (B * 2.0 ** -11 + 2.0 ** -24)
    n_round = mma_ulps * (3 * math.ceil(K / 16) + 4)
    return t_split + t_lolo + n_round * 2.0 ** -23 * absAB


# ---------------------------------------------------------------- kNN / kMeans oracles
def knn(X, Q, k: int):
    """Exact kNN: fp64 direct squared distances, ascending (dist, idx)."""
    X, Q = _f32(X), _f32(Q)
    nx, d = X.shape
    nq = Q.shape[0]
    idx = np.empty((nq, k), np.int32)
    dist = np.empty((nq, k), np.float64)
    lib().oracle_knn(_p(X), nx, _p(Q), nq, d, int(k), _p(idx), _p(dist))
    return idx, dist


def sqdist(X, Q):
    X, Q = _f32(X), _f32(Q)
    out = np.empty((Q.shape[0], X.shape[0]), np.float64)
    lib().oracle_sqdist(_p(X), X.shape[0], _p(Q), Q.shape[0], X.shape[1], _p(out))
    return out


def kmeans_step(X, C):
    """One Lloyd step: (assign, sums fp64, counts int64, inertia, best_dist)."""
    X, C = _f32(X), _f32(C)
    n, d = X.shape
    kc = C.shape[0]
    assign = np.empty(n, np.int32)
    sums = np.empty((kc, d), np.float64)
    counts = np.empty(kc, np.int64)
    inertia = np.zeros(1, np.float64)
    best = np.empty(n, np.float64)
    lib().oracle_kmeans_step(_p(X), n, d, _p(C), kc, _p(assign), _p(sums), _p(counts),
                             _p(inertia), _p(best))
    return assign, sums, counts, float(inertia[0]), best


def kmeans_finalize(sums, counts, C):
    sums = np.ascontiguousarray(sums, np.float64)
    counts = np.ascontiguousarray(counts, np.int64)
    out = _f32(C).copy()
    lib().oracle_kmeans_finalize(_p(sums), _p(counts), out.shape[0], out.shape[1], _p(out))
    return out


def tc_mma16(a, b, c: float = 0.0, use_c: bool = True) -> float:
    """The profiled tcgen05 kind::f16 MMA step (C implementation) on <= 16 products."""
    a, b = _f32(a), _f32(b)
    return float(np.float32(lib().oracle_tc_mma16(_p(a), _p(b), int(a.size), float(c), int(use_c))))


def gemm_alg1_tc(A, B, C=None, terms: int = 3, sep: int = 0, kc: int = 64):
    """Alg. 1 step by step on the profiled tensor-core primitive with promotion every kc
    (reading R21): the bitwise model of what the kernel computes for (terms, sep, kc)."""
    A, B = _f32(A), _f32(B)
    M, K = A.shape
    N = B.shape[1]
    D = np.empty((M, N), np.float32)
    Cp = _f32(C) if C is not None else None
    lib().oracle_gemm_alg1_tc(M, N, K, _p(A), _p(B), _p(Cp) if Cp is not None else None,
                              int(terms), int(sep), int(kc), _p(D))
    return D


def rownorm_tree(X):
    """Squared row norms in the order reading R22 fixes (the paper is silent): in fp64,
    lane l of 32 sums x_t^2 for t = l, l+32, l+64, ... in order; the 32 lane sums are then
    combined by the butterfly s_l <- s_l + s_(l xor o) for o = 16, 8, 4, 2, 1; the result
    is rounded to fp32.  Every x^2 is exact in fp64."""
    X = np.asarray(X, np.float32).astype(np.float64)
    n, d = X.shape
    lanes = np.zeros((n, 32), np.float64)
    for t0 in range(0, d, 32):
        blk = X[:, t0:t0 + 32]
        lanes[:, :blk.shape[1]] += blk * blk  # one exact square added per lane and round
    idx = np.arange(32)
    for o in (16, 8, 4, 2, 1):
        lanes = lanes + lanes[:, idx ^ o]
    return lanes[:, 0].astype(np.float32)


def _kc_single(d: int) -> int:
    return ((d + 63) // 64) * 64  # one promotion chunk over the whole feature dimension


def tf32_parts(y: float):
    """(h, m, l) with y = h + m + l exactly, each part an exact tf32 value (reading R22)."""
    h, m, l = ctypes.c_float(), ctypes.c_float(), ctypes.c_float()
    lib().oracle_tf32_parts(float(np.float32(y)), ctypes.byref(h), ctypes.byref(m), ctypes.byref(l))
    return h.value, m.value, l.value


def norm_step(dot, nrm):
    """acc_ij = TC(dot_ij; 1*h_j + 1*m_j + 1*l_j), (h, m, l) = tf32_parts(-nrm_j / 2): the
    tensor-core step that adds -||x_j||^2 / 2 after the products (reading R22)."""
    dot, nrm = _f32(dot), _f32(nrm)
    M, N = dot.shape
    out = np.empty((M, N), np.float32)
    lib().oracle_norm_step(M, N, _p(dot), _p(nrm), _p(out))
    return out


def knn_alg1_tc(X, Q, k: int):
    """kNN with the distance GEMM done by Alg. 1 on the profiled tensor core (R21, R22):
    dot = gemm_alg1_tc(Q, X^T, kc = whole d); acc = norm_step(dot, ||x||^2) (one more
    tensor-core step adding -||x_j||^2 / 2); key_ij = -2 acc_ij (exact); the k smallest
    (key, j) ascending; dist = max(0, RN32(||q_i||^2 + key)).  The bitwise model of
    egemm_knn; the plain definition stays `knn` (exact distances, gap rule R18)."""
    X, Q = _f32(X), _f32(Q)
    nx, d = X.shape
    xn = rownorm_tree(X)
    qn = rownorm_tree(Q).astype(np.float64)
    dot = gemm_alg1_tc(Q, X.T, terms=3, sep=0, kc=_kc_single(d))
    key = np.float32(-2.0) * norm_step(dot, xn)
    order = np.lexsort((np.broadcast_to(np.arange(nx), key.shape), key), axis=1)[:, :k]
    kk = np.take_along_axis(key, order, 1)
    dist = (qn[:, None] + kk.astype(np.float64)).astype(np.float32)
    return order.astype(np.int32), np.maximum(dist, np.float32(0.0))


def kmeans_assign_alg1_tc(X, C):
    """kMeans assignment with Alg. 1 on the profiled tensor core (R21, R22): key_ij =
    -2 norm_step(x_i . c_j, ||c_j||^2), assign_i = the lowest j of minimal key.  Returns
    (assign int32, best key fp32)."""
    X, C = _f32(X), _f32(C)
    d = X.shape[1]
    cn = rownorm_tree(C)
    dot = gemm_alg1_tc(X, C.T, terms=3, sep=0, kc=_kc_single(d))
    key = np.float32(-2.0) * norm_step(dot, cn)
    a = np.argmin(key, axis=1)  # first occurrence: ties -> lowest j
    return a.astype(np.int32), key[np.arange(len(a)), a]


def group_sums(X, assign, kc: int):
    """R20-ordered fp64 sums and int64 counts of X's rows grouped by a given assignment."""
    X = _f32(X)
    a = np.ascontiguousarray(assign, np.int32)
    n, d = X.shape
    sums = np.empty((kc, d), np.float64)
    counts = np.empty(kc, np.int64)
    lib().oracle_group_sums(_p(X), n, d, _p(a), kc, _p(sums), _p(counts))
    return sums, counts


def dist_tolerance(Q, X, mma_ulps: float = 4.0):
    """tau_ij for a squared distance ||q||^2 + ||x||^2 - 2 q.x computed by the method
    (R18): 2 * elem_bound(q.x) + 12 * 2^-24 * (||q||^2 + ||x||^2).  The norm term covers
    the fp32 norms (1 ulp each), the R22 norm step (4 terms truncated onto 2^(E-25) with
    2^E <= max(|q.x|, ||x||^2/2), then RZ: < 2^-22 (||q||^2 + 1.5 ||x||^2) on the key) and
    the final RN of ||q||^2 + key (<= 2 ulps of the norms): <= 9 units, rounded up to 12."""
    Q = np.asarray(Q, np.float64)
    X = np.asarray(X, np.float64)
    eb = elem_bound(Q, X.T, mma_ulps)
    nq = (Q * Q).sum(1)[:, None]
    nx = (X * X).sum(1)[None, :]
    return 2.0 * eb + 12.0 * 2.0 ** -24 * (nq + nx) + 2.0 ** -20


# ---------------------------------------------------------------- tensor-core models
# Candidate models for one tensor-core MMA step d = c + sum_{t<16} a_t*b_t with fp16
# a, b and fp32 c (the paper's precision-profiling workflow, Sec. 3.1 P:596-629,
# profiling P:712-737).  All arithmetic is exact (fractions); only the final step rounds.
def _round_f32(v: Fraction, mode: str) -> float:
    if v == 0:
        return 0.0
    s = -1 if v < 0 else 1
    a = -v if v < 0 else v
    e = a.numerator.bit_length() - a.denominator.bit_length()
    if Fraction(2) ** e > a:
        e -= 1
    elif Fraction(2) ** (e + 1) <= a:
        e += 1
    e = max(e, -126)
    ulp = Fraction(2) ** (e - 23)
    q, r = divmod(a, ulp)  # q integer, r remainder
    q = int(q)
    if mode == "rn":
        if r * 2 > ulp or (r * 2 == ulp and q % 2 == 1):
            q += 1
    elif mode == "rz":
        pass
    else:
        raise ValueError(mode)
    val = Fraction(q) * ulp
    if val >= Fraction(2) ** 128:
        return s * math.inf
    return s * float(val)  # exact: val is an fp32 value


def tc_model(a, b, c: float, model: str, extra_bits: int = 0, anchor: str = "fields") -> float:
    """Candidate semantics of one MMA step.

    model "rn": exact sum, round to nearest-even fp32.
    model "rz": exact sum, truncate toward zero to fp32.
    model "align": every product and c is first truncated toward zero onto the grid
      2^(E-23-extra_bits), where E is the largest exponent estimate among the non-zero
      terms, the truncated terms are summed exactly, and the sum is truncated to fp32.
      anchor "fields": a product's estimate is the sum of the operands' exponents
        (e_a + e_b, the exponent-field sum before normalisation); c's is its exponent.
      anchor "value": the product's true exponent (e_a + e_b or e_a + e_b + 1).
    """
    terms = []
    ests = []
    for x, y in zip(a, b):
        x, y = float(x), float(y)
        if x == 0.0 or y == 0.0:
            continue
        terms.append(Fraction(x) * Fraction(y))
        if anchor == "fields":
            ests.append((math.frexp(abs(x))[1] - 1) + (math.frexp(abs(y))[1] - 1))
        else:
            ests.append(math.frexp(abs(x * y))[1] - 1)
    c = float(c)
    if c != 0.0:
        terms.append(Fraction(c))
        ests.append(math.frexp(abs(c))[1] - 1)
    if model in ("rn", "rz"):
        return _round_f32(sum(terms, Fraction(0)), model)
    if model == "align":
        if not terms:
            return 0.0
        g = Fraction(2) ** (max(ests) - 23 - extra_bits)
        tot = Fraction(0)
        for t in terms:
            q = abs(t) // g
            tot += (q * g) if t >= 0 else -(q * g)
        return _round_f32(tot, "rz")
    raise ValueError(model)
