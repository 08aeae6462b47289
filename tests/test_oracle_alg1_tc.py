"""Pins for the Alg.-1-on-the-profiled-tensor-core oracle (oracle.gemm_alg1_tc; Alg. 1
P:749-755 in the paper's step order, promotion reading R21): the C primitive against the
exact-rational Python model of the same definition, a worked example whose result depends
on Alg. 1's order (derived by hand below), closed forms (integers, A = signed permutation,
fp16-exact inputs, K <= 16), the element error bound, and the promotion claim."""
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


@pytest.mark.parametrize("sep,kc", [(0, 64), (0, 128), (1, 256), (0, 0), (1, 48)])
def test_alg1_tc_integers_exact(oracle_lib, sep, kc):
    """Integer inputs |x| <= 32, K = 2048: every partial sum is an exact fp32 integer, so
    truncation never fires and the model equals the integer GEMM bitwise."""
    A, B = inputs.integers((9, 2048), 1), inputs.integers((2048, 11), 2)
    D = oracle_lib.gemm_alg1_tc(A, B, sep=sep, kc=kc)
    assert np.array_equal(D, (A.astype(np.int64) @ B.astype(np.int64)).astype(np.float32))


def test_alg1_order_worked_example(oracle_lib):
    """Alg. 1's order decides the result.  a = b = 1.5 + 2^-22 (fp32-exact) split into
    hi = 1.5, lo = 2^-22 (an fp16 subnormal).  Products: hi*hi = 2.25, lo*hi = hi*lo =
    3 * 2^-23.  In the paper's order (l.6 lo*hi, l.7 hi*lo, l.8 hi*hi) the two cross terms
    meet first: 3*2^-23 + 3*2^-23 = 3*2^-22 exactly; the last step adds 2.25 with
    E = e(1.5) + e(1.5) = 0, grid 2^-25, on which 3*2^-22 lies, so D = 2.25 + 3*2^-22
    (representable: the fp32 ulp at 2.25 is 2^-22) = the exact 3-term sum.  hi*hi first
    would round toward zero after each cross term: 2.25 + 3*2^-23 -> 2.25 + 2^-22, then
    2.25 + 5*2^-23 -> 2.25 + 2*2^-22 -- one ulp lower.  terms = 4 puts lo*lo = 2^-44 first;
    it is dropped by the last step's 2^-25 grid: the same D."""
    x = np.float32(1.5 + 2.0 ** -22)
    A, B = np.array([[x]], np.float32), np.array([[x]], np.float32)
    want = np.float32(2.25 + 3 * 2.0 ** -22)
    assert float(want) == 2.25 + 3 * 2.0 ** -22
    for terms in (3, 4):
        assert oracle_lib.gemm_alg1_tc(A, B, terms=terms)[0, 0] == want
    # the same pair inside a longer K (zeros elsewhere) and with the promotion chunking
    Ak = np.zeros((1, 48), np.float32)
    Bk = np.zeros((48, 1), np.float32)
    Ak[0, 37], Bk[37, 0] = x, x
    for kc in (0, 16, 32):
        assert oracle_lib.gemm_alg1_tc(Ak, Bk, kc=kc)[0, 0] == want


def test_alg1_signed_permutation_reconstructs_hi_plus_lo(oracle_lib):
    """A = a signed permutation scaled by powers of two: every output is one product chain
    2^s * (lo_b ... ) with lo_a = 0, i.e. TC(TC(0; 2^s lo_b); 2^s hi_b) = 2^s (hi_b + lo_b)
    exactly (hi + lo has <= 22 significant bits), whatever the 16-wide slice it sits in."""
    g = inputs.rng(11)
    n = 40
    perm = g.permutation(n)
    sgn = g.choice([-1.0, 1.0], n)
    pw = 2.0 ** g.integers(-3, 4, n)
    A = np.zeros((n, n), np.float32)
    A[np.arange(n), perm] = sgn * pw
    B = inputs.uniform((n, 7), 12)
    hi, lo = oracle_lib.split(B)
    hl = (oracle_lib.h2f(hi) + oracle_lib.h2f(lo)).astype(np.float32)
    want = (sgn * pw)[:, None].astype(np.float32) * hl[perm]
    for kc in (0, 16):
        assert np.array_equal(oracle_lib.gemm_alg1_tc(A, B, kc=kc), want)


def test_alg1_tc_fp16_inputs_k16_is_one_mma(oracle_lib):
    """fp16-exact inputs (lo = 0) and K <= 16: the whole product is one profiled MMA on a
    zero accumulator (the cross MMAs add exact zeros)."""
    g = inputs.rng(4)
    A, B = _f16(g.uniform(-1, 1, (6, 13))), _f16(g.uniform(-1, 1, (13, 5)))
    D = oracle_lib.gemm_alg1_tc(A, B)
    for i in range(6):
        for j in range(5):
            assert D[i, j] == np.float32(oracle_lib.tc_model(A[i], B[:, j], 0.0, "align", 2))


@pytest.mark.parametrize("terms,sep,kc", [(3, 0, 64), (3, 0, 128), (3, 1, 256), (4, 0, 64), (3, 0, 0), (4, 1, 0)])
def test_alg1_tc_within_bounds(oracle_lib, terms, sep, kc):
    A, B = inputs.uniform((48, 1000), 5), inputs.uniform((1000, 40), 6)
    C = inputs.uniform((48, 40), 7)
    D = oracle_lib.gemm_alg1_tc(A, B, C, terms=terms, sep=sep, kc=kc)
    C64 = oracle_lib.gemm64(A, B, C)
    assert np.all(np.abs(D - C64) <= oracle_lib.elem_bound(A, B, terms=terms, kc=kc) + 2.0 ** -23 * np.abs(C))
    e = oracle_lib.normwise_error(D, A, B, C64)
    en = oracle_lib.normwise_error(oracle_lib.gemm32_naive(A, B, C), A, B, C64)
    if kc:  # the single chain (kc = 0) is the unpromoted paper design: bound only
        assert e <= 2 * en


def test_alg1_tc_promotion_reduces_error(oracle_lib):
    """with the truncating primitive the paper's single chain over all of K is
    several times worse than naive fp32; promotion every 64 k brings it below."""
    A, B = inputs.uniform((24, 4096), 8), inputs.uniform((4096, 24), 9)
    C64 = oracle_lib.gemm64(A, B)
    e_long = oracle_lib.normwise_error(oracle_lib.gemm_alg1_tc(A, B, kc=0), A, B, C64)
    e_64 = oracle_lib.normwise_error(oracle_lib.gemm_alg1_tc(A, B, kc=64), A, B, C64)
    en = oracle_lib.normwise_error(oracle_lib.gemm32_naive(A, B), A, B, C64)
    assert e_long > 2 * en and e_64 < en


def test_alg1_tc_bf16_variant_closed_forms(oracle_lib):
    """NEXT-3's bf16 round-split through the same Alg. 1: integer inputs (8 significant bits,
    partial sums < 2^24) are exact; A = signed permutation reconstructs fl32(hi_b + lo_b) of
    the bf16 parts; and at fp16-range inputs the bf16 parts (8 + 8 bits) are less accurate
    than the fp16 ones (11 + 11 bits), while at |x| ~ 2^40 (beyond fp16) only bf16 works."""
    A, B = inputs.integers((9, 1024), 1, lim=100), inputs.integers((1024, 11), 2, lim=100)
    D = oracle_lib.gemm_alg1_tc(A, B, kc=64, fmt="bf16")
    assert np.array_equal(D, (A.astype(np.int64) @ B.astype(np.int64)).astype(np.float32))
    n = 24
    g = inputs.rng(13)
    perm = g.permutation(n)
    A = np.zeros((n, n), np.float32)
    A[np.arange(n), perm] = g.choice([-2.0, -1.0, 0.5, 1.0], n)
    B = inputs.uniform((n, 5), 14)
    hi, lo = oracle_lib.split(B, "bf16")
    hl = (oracle_lib.bf16_bits_to_f64(hi) + oracle_lib.bf16_bits_to_f64(lo)).astype(np.float32)
    want = A[np.arange(n), perm][:, None] * hl[perm]
    assert np.array_equal(oracle_lib.gemm_alg1_tc(A, B, fmt="bf16"), want)
    A, B = inputs.uniform((32, 512), 15), inputs.uniform((512, 32), 16)
    C64 = oracle_lib.gemm64(A, B)
    e16 = oracle_lib.normwise_error(oracle_lib.gemm_alg1_tc(A, B, kc=64), A, B, C64)
    eb = oracle_lib.normwise_error(oracle_lib.gemm_alg1_tc(A, B, kc=64, fmt="bf16"), A, B, C64)
    assert eb > 10 * e16
    Aw, Bw = (A * 2.0 ** 40).astype(np.float32), (B * 2.0 ** 40).astype(np.float32)
    C64w = oracle_lib.gemm64(Aw, Bw)
    ebw = oracle_lib.normwise_error(oracle_lib.gemm_alg1_tc(Aw, Bw, kc=64, fmt="bf16"), Aw, Bw, C64w)
    assert np.isclose(ebw, eb, rtol=0.05)  # scale-invariant with the 8-bit exponent
    with np.errstate(all="ignore"):
        D16 = oracle_lib.gemm_alg1_tc(Aw, Bw, kc=64)
    assert not np.all(np.isfinite(D16))  # fp16 parts overflow


def test_alg1_tc_kparts_split_k_reading(oracle_lib):
    """Split-K reading (R21): kpart >= K is the single part; integer inputs stay exact for any
    split; and the parts compose as their own Alg. 1 runs: D(kpart) = RN(D(A[:, :p], B[:p]) +
    D(A[:, p:], B[p:])) with C added last -- checked against two independent oracle calls."""
    A, B = inputs.uniform((20, 500), 31), inputs.uniform((500, 17), 32)
    C = inputs.uniform((20, 17), 33)
    one = oracle_lib.gemm_alg1_tc(A, B, C, kc=128)
    assert np.array_equal(oracle_lib.gemm_alg1_tc(A, B, C, kc=128, kpart=500), one)
    assert np.array_equal(oracle_lib.gemm_alg1_tc(A, B, C, kc=128, kpart=1024), one)
    for sep in (0, 1):
        two = oracle_lib.gemm_alg1_tc(A, B, C, sep=sep, kc=128, kpart=256)
        lo = oracle_lib.gemm_alg1_tc(A[:, :256], B[:256], sep=sep, kc=128)
        hi = oracle_lib.gemm_alg1_tc(A[:, 256:], B[256:], sep=sep, kc=128)
        assert np.array_equal(two, ((lo + hi).astype(np.float32) + C).astype(np.float32))
    Ai, Bi = inputs.integers((9, 700), 34), inputs.integers((700, 5), 35)
    ref = (Ai.astype(np.int64) @ Bi.astype(np.int64)).astype(np.float32)
    for kp in (64, 192, 448):
        assert np.array_equal(oracle_lib.gemm_alg1_tc(Ai, Bi, kc=64, kpart=kp), ref)
