"""Pins for the Alg.-1-on-the-profiled-tensor-core oracle (oracle.gemm_alg1_tc, reading R21):
the C primitive against the exact-rational Python model of the same definition, closed
forms (integers, fp16-exact inputs, K <= 16), the element error bound, and the design's
promotion claim (shorter chunks -> smaller error)."""
import numpy as np
import pytest

from paper_conf_ppopp_fengwcz0d21_b200 import inputs


def _f16(x):
    return np.asarray(x, np.float32).astype(np.float16).astype(np.float32)


def test_tc_mma16_matches_rational_model(oracle_lib):
    """C primitive == oracle.tc_model('align', 2 extra bits, exponent-field anchor),
    computed with fractions -- two independent renderings of the probed definition."""
    g = inputs.rng(3)
    for trial in range(600):
        n = int(g.integers(1, 17))
        scale = 2.0 ** g.integers(-12, 4, size=n)
        a = _f16(g.uniform(-1, 1, n) * scale)
        b = _f16(g.uniform(-1, 1, n))
        if trial % 5 == 0:
            a[: n // 2] = 0.0
        if trial % 7 == 0:  # subnormal fp16 operands (lo parts of small values)
            a = _f16(g.integers(-1023, 1024, n) * 2.0 ** -24)
        c = float(np.float32(g.uniform(-4, 4) * 2.0 ** g.integers(-6, 6))) if trial % 3 else 0.0
        ref = oracle_lib.tc_model(a, b, c, "align", 2, "fields")
        got = oracle_lib.tc_mma16(a, b, c, True)
        assert np.float32(got) == np.float32(ref), (trial, got, ref)


def test_tc_mma16_exact_when_representable(oracle_lib):
    a = np.array([1, 2, 3, 0.5] + [0] * 12, np.float32)
    b = np.array([2, 0.25, -1, 4] + [0] * 12, np.float32)
    assert oracle_lib.tc_mma16(a, b, 1.5) == 2 + 0.5 - 3 + 2 + 1.5
    assert oracle_lib.tc_mma16(a, b, 7.0, use_c=False) == 2 + 0.5 - 3 + 2


@pytest.mark.parametrize("sep,kc", [(0, 64), (0, 128), (1, 256)])
def test_alg1_tc_integers_exact(oracle_lib, sep, kc):
    """Integer inputs |x| <= 32, K = 2048: every partial sum is an exact fp32 integer, so
    truncation never fires and the model equals the integer GEMM bitwise."""
    A, B = inputs.integers((9, 2048), 1), inputs.integers((2048, 11), 2)
    D = oracle_lib.gemm_alg1_tc(A, B, sep=sep, kc=kc)
    assert np.array_equal(D, (A.astype(np.int64) @ B.astype(np.int64)).astype(np.float32))


def test_alg1_tc_fp16_inputs_k16_is_one_mma(oracle_lib):
    """fp16-exact inputs (lo = 0) and K <= 16: the whole product is one profiled MMA on a
    zero accumulator (the cross MMAs add exact zeros)."""
    g = inputs.rng(4)
    A, B = _f16(g.uniform(-1, 1, (6, 13))), _f16(g.uniform(-1, 1, (13, 5)))
    D = oracle_lib.gemm_alg1_tc(A, B)
    for i in range(6):
        for j in range(5):
            assert D[i, j] == np.float32(oracle_lib.tc_model(A[i], B[:, j], 0.0, "align", 2))


@pytest.mark.parametrize("terms,sep,kc", [(3, 0, 64), (3, 0, 128), (3, 1, 256), (4, 0, 64)])
def test_alg1_tc_within_bounds(oracle_lib, terms, sep, kc):
    A, B = inputs.uniform((48, 1000), 5), inputs.uniform((1000, 40), 6)
    C = inputs.uniform((48, 40), 7)
    D = oracle_lib.gemm_alg1_tc(A, B, C, terms=terms, sep=sep, kc=kc)
    C64 = oracle_lib.gemm64(A, B, C)
    assert np.all(np.abs(D - C64) <= oracle_lib.elem_bound(A, B, terms=terms) + 2.0 ** -23 * np.abs(C))
    e = oracle_lib.normwise_error(D, A, B, C64)
    en = oracle_lib.normwise_error(oracle_lib.gemm32_naive(A, B, C), A, B, C64)
    assert e <= 2 * en


def test_alg1_tc_promotion_reduces_error(oracle_lib):
    """with the truncating primitive a single accumulator over all of K is
    several times worse than naive fp32; promotion every 64 k brings it below."""
    A, B = inputs.uniform((24, 4096), 8), inputs.uniform((4096, 24), 9)
    C64 = oracle_lib.gemm64(A, B)
    e_long = oracle_lib.normwise_error(oracle_lib.gemm_alg1_tc(A, B, kc=4096), A, B, C64)
    e_64 = oracle_lib.normwise_error(oracle_lib.gemm_alg1_tc(A, B, kc=64), A, B, C64)
    en = oracle_lib.normwise_error(oracle_lib.gemm32_naive(A, B), A, B, C64)
    assert e_long > 2 * en and e_64 < en
