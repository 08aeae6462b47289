"""Pins for the oracle GEMMs (Alg. 1 semantics D = A x B + C, P:739-757, P:794-810;
naive fp32 = Eq. 10's V_single).

References used: exact rational arithmetic (fractions), exact integer matmul, scalar
numpy.float32 arithmetic, numpy's binary16 cast for the split, and Fig. 7.
"""
import math
from fractions import Fraction

import numpy as np
import pytest

from paper_conf_ppopp_fengwcz0d21_b200 import inputs


def _exact(A, B, C=None):
    M, K = A.shape
    N = B.shape[1]
    out = [[sum((Fraction(float(A[i, k])) * Fraction(float(B[k, j])) for k in range(K)),
                Fraction(0)) + (Fraction(float(C[i, j])) if C is not None else 0)
            for j in range(N)] for i in range(M)]
    return out


@pytest.mark.parametrize("gen", [inputs.uniform, inputs.stress, inputs.in_zone])
def test_gemm64_vs_exact_rationals(oracle_lib, gen):
    A, B, C = gen((4, 4), 1), gen((4, 4), 2), gen((4, 4), 3)
    D = oracle_lib.gemm64(A, B, C)
    ex = _exact(A, B, C)
    absAB = np.abs(A.astype(np.float64)) @ np.abs(B.astype(np.float64)) + np.abs(C)
    for i in range(4):
        for j in range(4):
            assert abs(Fraction(D[i, j]) - ex[i][j]) <= Fraction(5 * 2.0 ** -53) * Fraction(absAB[i, j])


def test_gemm64_integers_exact(oracle_lib):
    A = inputs.integers((37, 300), 4, lim=1000)
    B = inputs.integers((300, 29), 5, lim=1000)
    D = oracle_lib.gemm64(A, B)
    ref = A.astype(np.int64) @ B.astype(np.int64)
    assert np.array_equal(D, ref.astype(np.float64))


def test_gemm32_naive_vs_scalar_float32(oracle_lib):
    """Bitwise equal to a scalar np.float32 loop: acc = acc + a*b, k ascending, no FMA."""
    A, B = inputs.uniform((5, 37), 6), inputs.uniform((37, 7), 7)
    D = oracle_lib.gemm32_naive(A, B)
    for i in range(5):
        for j in range(7):
            acc = np.float32(0)
            for k in range(37):
                acc = np.float32(acc + np.float32(A[i, k] * B[k, j]))
            assert D[i, j].view(np.uint32) == acc.view(np.uint32)


def _np_split(x):
    hi = x.astype(np.float16)
    lo = (x - hi.astype(np.float32)).astype(np.float16)
    return hi.astype(np.float64), lo.astype(np.float64)


@pytest.mark.parametrize("terms", [3, 4])
@pytest.mark.parametrize("K", [4, 13, 16])
def test_emu64_vs_exact_split_products(oracle_lib, terms, K):
    """emu64 == the exact sum of the split products (split via numpy's binary16 cast),
    up to the fp64 accumulation rounding."""
    A, B = inputs.stress((4, K), 10 + K), inputs.uniform((K, 4), 20 + K)
    D = oracle_lib.gemm_emu64(A, B, terms)
    ah, al = _np_split(A)
    bh, bl = _np_split(B)
    for i in range(4):
        for j in range(4):
            ex = Fraction(0)
            mag = 0.0
            for k in range(K):
                t = [(ah[i, k], bh[k, j]), (ah[i, k], bl[k, j]), (al[i, k], bh[k, j])]
                if terms == 4:
                    t.append((al[i, k], bl[k, j]))
                for x, y in t:
                    ex += Fraction(x) * Fraction(y)
                    mag += abs(x * y)
            assert abs(Fraction(D[i, j]) - ex) <= Fraction(4 * K * 2.0 ** -53) * Fraction(mag)


def test_emu64_equals_gemm64_on_fp16_inputs(oracle_lib):
    """fp16-representable inputs: lo = 0, so the emulation is the plain product (bitwise
    in fp64: the same per-element k-ordered sum of the same exact products)."""
    A = inputs.uniform((33, 70), 30).astype(np.float16).astype(np.float32)
    B = inputs.uniform((70, 21), 31).astype(np.float16).astype(np.float32)
    assert np.array_equal(oracle_lib.gemm_emu64(A, B, 3), oracle_lib.gemm64(A, B))


def test_split_error_magnitudes(oracle_lib):
    """U[-1,1], M=N=64, K=1024: intrinsic split error (emu64 vs fp64) is ~1e-9 and far
    below naive fp32 (~2.4e-8); the 4th term changes it little (R5)."""
    A, B = inputs.uniform((64, 1024), 40), inputs.uniform((1024, 64), 41)
    C64 = oracle_lib.gemm64(A, B)
    e3 = oracle_lib.normwise_error(oracle_lib.gemm_emu64(A, B, 3), A, B, C64)
    e4 = oracle_lib.normwise_error(oracle_lib.gemm_emu64(A, B, 4), A, B, C64)
    en = oracle_lib.normwise_error(oracle_lib.gemm32_naive(A, B), A, B, C64)
    assert e3 < 1e-8 and e4 <= e3 * 1.05
    assert 5e-9 < en < 1e-7
    assert e3 < en / 5


def test_truncate_split_biased_on_nonnegative(oracle_lib):
    """Markidis truncate-split loses accuracy on non-negative data: its residual is
    one-signed (Fig. 4a; SURVEY [sim-spliterr])."""
    A, B = inputs.uniform((32, 512), 42, 0, 1), inputs.uniform((512, 32), 43, 0, 1)
    C64 = oracle_lib.gemm64(A, B)
    ahr, alr = oracle_lib.split(A, "trunc")
    bhr, blr = oracle_lib.split(B, "trunc")
    h = oracle_lib.h2f
    Dt = h(ahr) @ h(bhr) + h(ahr) @ h(blr) + h(alr) @ h(bhr)
    e_trunc = oracle_lib.normwise_error(Dt, A, B, C64)
    e_round = oracle_lib.normwise_error(oracle_lib.gemm_emu64(A, B, 3), A, B, C64)
    assert e_trunc > 10 * e_round


def test_fig7_sanity_ceiling(oracle_lib):
    """Eq. 10 error of the emulated products vs naive fp32 sits far under the paper's
    EGEMM-TC series of Fig. 7 at N=256 (1.9e-5, tests/golden/fig7_max_error.txt)."""
    N = 256
    A, B = inputs.uniform((N, N), 50), inputs.uniform((N, N), 51)
    e = oracle_lib.eq10_max_error(oracle_lib.gemm_emu64(A, B, 3), oracle_lib.gemm32_naive(A, B))
    assert e < 1.9e-5


def test_elem_bound_holds_for_emu(oracle_lib):
    """The element bound (R18) covers the split-only error with zero rounding ulps."""
    A, B = inputs.stress((16, 200), 60), inputs.uniform((200, 16), 61)
    err = np.abs(oracle_lib.gemm_emu64(A, B, 3) - oracle_lib.gemm64(A, B))
    assert np.all(err <= oracle_lib.elem_bound(A, B, mma_ulps=0.0))
    assert math.isfinite(float(oracle_lib.elem_bound(A, B).max()))


def test_gemm32_naive_closed_forms(oracle_lib):
    """Reading R10 pinned by hand-derived values, not by re-running the formula:
    * order: a = (2^24, 1, 1), b = (1, 1, 1): k ascending gives 2^24 + 1 -> 2^24 (an fp32 tie,
      to even) twice, so 2^24; the exact sum 2^24 + 2 (what any other order would give).
    * no FMA: a = (-1, 1 + 2^-12), b = (1, 1 + 2^-12): the product 1 + 2^-11 + 2^-24 rounds to
      1 + 2^-11 (a tie, to even) before the add, so -1 + that = 2^-11 exactly; a fused
      multiply-add would keep 2^-11 + 2^-24."""
    A = np.array([[2.0 ** 24, 1.0, 1.0]], np.float32)
    B = np.ones((3, 1), np.float32)
    assert oracle_lib.gemm32_naive(A, B)[0, 0] == np.float32(2.0 ** 24)
    assert oracle_lib.gemm64(A, B)[0, 0] == 2.0 ** 24 + 2
    t = np.float32(1.0 + 2.0 ** -12)
    A = np.array([[-1.0, t]], np.float32)
    B = np.array([[1.0], [t]], np.float32)
    assert oracle_lib.gemm32_naive(A, B)[0, 0] == np.float32(2.0 ** -11)
    assert oracle_lib.gemm64(A, B)[0, 0] == 2.0 ** -11 + 2.0 ** -24
