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
        for f in ("oracle_split", "oracle_split_rha", "oracle_split_trunc", "oracle_split_bf16"):
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
        L.oracle_kmeans_sums.argtypes = [P, I64, I64, P, I64, P, P]
        L.oracle_kmeans_sums.restype = None
        L.oracle_rownorm.argtypes = [P, I64, I64, P]
        L.oracle_rownorm.restype = None
        L.oracle_tc_mma16.argtypes = [P, P, I, ctypes.c_float, I]
        L.oracle_tc_mma16.restype = ctypes.c_float
        L.oracle_gemm_alg1_tc.argtypes = [I64, I64, I64, P, P, P, I, I, I64, I, I64, P]
        L.oracle_gemm_alg1_tc.restype = None
        L.oracle_tc_rows.argtypes = [I64, I64, I, P, P, P, P]
        L.oracle_tc_rows.restype = None
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
    "trunc" (Markidis truncate-split, Fig. 4a), "bf16" (NEXT-3: bf16 parts, the
    upper halves of fp32 patterns, RNE)."""
    x = _f32(x)
    hi = np.empty(x.shape, np.uint16)
    lo = np.empty(x.shape, np.uint16)
    fn = {"rne": lib().oracle_split, "rha": lib().oracle_split_rha,
          "trunc": lib().oracle_split_trunc, "bf16": lib().oracle_split_bf16}[variant]
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


MMA_ULPS = 5.25  # per MMA step of the probed primitive: 17 terms truncated (< 17 g) + RZ (< 1 ulp)


def elem_bound(A, B, terms: int = 3, kc: int = 0, mma_ulps: float = MMA_ULPS):
    """Worst-case |D - (AB)_ij| of Alg. 1 on the profiled tensor core (reading R18), derived
    from the probed primitive: one MMA step truncates each of its <= 17 terms
    onto the grid g = 2^(E-25) with 2^E <= max |term| <= S (S = sum of |terms|), then rounds
    toward zero: error < 17 g + ulp(S) <= 5.25 * 2^-23 * S.  Inside a promotion chunk every
    step's S is at most the chunk's sum of |products| (<= 1.01 sum_k |a_k||b_k| over the
    chunk), so the chained steps of all chunks add <= 5.25 * 1.01 * terms * ceil(kc/16)
    * 2^-23 * sum_k |a||b|; each promotion add, the SEP combine and + C add half an ulp.
    Plus the split residuals of both operands and, for terms = 3, the dropped lo*lo term.
    kc <= 0 or kc >= K: one chain over all of K (the loosest case)."""
    A = np.abs(np.asarray(A, np.float64))
    B = np.abs(np.asarray(B, np.float64))
    K = A.shape[1]
    kce = K if (kc <= 0 or kc >= K) else kc
    eA, eB = split_abs_bound(A), split_abs_bound(B)
    absAB = A @ B
    t_split = eA @ B + A @ eB + eA @ eB
    t_lolo = 0.0 if terms == 4 else (A * 2.0 ** -11 + 2.0 ** -24) @ (B * 2.0 ** -11 + 2.0 ** -24)
    n_round = mma_ulps * 1.01 * terms * math.ceil(max(kce, 1) / 16) + 0.5 * (math.ceil(K / max(kce, 1)) + 2)
    return t_split + t_lolo + n_round * 2.0 ** -23 * absAB


NORM_UNITS = 9.0  # units of 2^-24 (||q||^2 + ||x||^2) in dist_tolerance (derivation below)


def dist_tolerance(Q, X):
    """tau_ij for a squared distance ||q||^2 + ||x||^2 - 2 q.x computed by the method
    (reading R18): 2 * elem_bound(q.x) + 9 * 2^-24 * (||q||^2 + ||x||^2).

    The norm term (derived; pinned against the exact-rational model in
    tests/test_kernel_model.py): the norm step adds y = -||x||^2/2 to the fp32 dot with one
    step of the probed primitive (4 terms dot, h, m, l truncated onto g = 2^(E-25), 2^E <=
    max(|dot|, |y|); result RZ with |result| < 2^(E+2), ulp <= 8 g): error < 12 g, doubled
    in key = -2 acc: < 24 * 2^-25 max(|dot|, |y|) <= 6 * 2^-24 (||q||^2 + ||x||^2) since
    |dot| <= ||q|| ||x|| <= (||q||^2 + ||x||^2)/2.  The fp32 norms add 1 unit (RN, 2^-24
    relative each) and the final RN of ||q||^2 + key (|dist| <= 2 (||q||^2 + ||x||^2))
    2 units: 9 units."""
    Q = np.asarray(Q, np.float64)
    X = np.asarray(X, np.float64)
    eb = elem_bound(Q, X.T, terms=3, kc=0)
    nq = (Q * Q).sum(1)[:, None]
    nx = (X * X).sum(1)[None, :]
    return 2.0 * eb + NORM_UNITS * 2.0 ** -24 * (nq + nx)


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


def kmeans_sums(X, assign, kc: int):
    """(sums fp64 [kc, d], counts int64 [kc]) of a given assignment: the plain definition,
    sums_j = sum of (double) x_i over a_i == j in ascending i (SURVEY c-6)."""
    X = _f32(X)
    a = np.ascontiguousarray(assign, np.int32)
    n, d = X.shape
    sums = np.empty((kc, d), np.float64)
    counts = np.empty(kc, np.int64)
    lib().oracle_kmeans_sums(_p(X), n, d, _p(a), kc, _p(sums), _p(counts))
    return sums, counts


def kmeans_sums_bound(X, assign, kc: int):
    """SURVEY c-20: any fp64 summation order of sums_j is within
    counts_j * 2^-52 * sum_{a_i = j} |x_i| of the plain ascending-i sum (both are within
    half that of the exact sum)."""
    X = np.abs(np.asarray(X, np.float64))
    a = np.asarray(assign, np.int64)
    absx = np.zeros((kc, X.shape[1]), np.float64)
    np.add.at(absx, a, X)
    cnt = np.bincount(a, minlength=kc)
    return cnt[:, None] * 2.0 ** -52 * absx


def kmeans_finalize(sums, counts, C):
    sums = np.ascontiguousarray(sums, np.float64)
    counts = np.ascontiguousarray(counts, np.int64)
    out = _f32(C).copy()
    lib().oracle_kmeans_finalize(_p(sums), _p(counts), out.shape[0], out.shape[1], _p(out))
    return out


def tc_mma16(a, b, c: float = 0.0, use_c: bool = True) -> float:
    """The profiled tcgen05 MMA step (C implementation) on <= 16 products."""
    a, b = _f32(a), _f32(b)
    return float(np.float32(lib().oracle_tc_mma16(_p(a), _p(b), int(a.size), float(c), int(use_c))))


def tc_rows(a, b, c=None):
    """The profiled MMA step in matrix form: out[i, j] = TC(c[i, j]; sum_t a[i, t] b[j, t])
    for a [M, n], b [N, n] with n <= 16 (c None: no addend)."""
    a, b = _f32(a), _f32(b)
    M, n = a.shape
    N = b.shape[0]
    assert b.shape[1] == n and n <= 16
    cp = _f32(c) if c is not None else None
    out = np.empty((M, N), np.float32)
    lib().oracle_tc_rows(M, N, n, _p(a), _p(b), _p(cp) if cp is not None else None, _p(out))
    return out


def bf16_bits_to_f64(bits):
    """bf16 bit patterns -> float64 (a bf16 is the top half of an fp32 pattern)."""
    return (np.asarray(bits, np.uint32) << 16).view(np.float32).astype(np.float64)


def gemm_alg1_tc(A, B, C=None, terms: int = 3, sep: int = 0, kc: int = 0, fmt: str = "f16",
                 kpart: int = 0):
    """Alg. 1 step by step on the profiled tensor-core primitive: per 16-wide
    k-slice in ascending k, [lo*lo,] lo*hi, hi*lo, hi*hi chained through one fp32
    accumulator; promotion into an fp32 total every kc k-elements (reading R21; kc = 0:
    the paper's single chain over K); sep = 1: hi*hi in its own chain; + C at the end (R7).
    fmt "bf16": the bf16 round-split variant (NEXT-3).  kpart > 0: split-K reading -- K in
    contiguous parts of kpart elements, each chained and promoted on its own, the part totals
    added in k order (then + C)."""
    A, B = _f32(A), _f32(B)
    M, K = A.shape
    N = B.shape[1]
    D = np.empty((M, N), np.float32)
    Cp = _f32(C) if C is not None else None
    lib().oracle_gemm_alg1_tc(M, N, K, _p(A), _p(B), _p(Cp) if Cp is not None else None,
                              int(terms), int(sep), int(kc), 1 if fmt == "bf16" else 0, int(kpart),
                              _p(D))
    return D


def rownorm(X):
    """||x_i||^2: fp64 sum of the (exact) squares in ascending t, rounded once to fp32."""
    X = _f32(X)
    out = np.empty(X.shape[0], np.float32)
    lib().oracle_rownorm(_p(X), X.shape[0], X.shape[1], _p(out))
    return out


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
