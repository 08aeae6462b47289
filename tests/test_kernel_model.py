"""CPU checks of tests/kernel_model.py (the bitwise models of the kernels' own choices for
the kNN / kMeans case studies, reading R22) and of the oracle's distance tolerance, whose
norm term is derived from the profiled primitive (oracle.dist_tolerance docstring) and
pinned here against the exact-rational model of that primitive."""
from fractions import Fraction

import numpy as np

import oracle
from paper_conf_ppopp_fengwcz0d21_b200 import inputs
from tests import kernel_model as km


def _low13_zero(x):
    return (np.asarray(x, np.float32).view(np.uint32) & 0x1FFF) == 0


def test_tf32_parts_exact_decomposition():
    """y = h + m + l exactly (checked in fp64), every part an exact tf32 value (13 low
    mantissa bits zero), |m| < 2^-10 |h| and |l| < 2^-20 |h|; tf32-exact y gives m = l = 0."""
    g = inputs.rng(2205)
    ys = np.concatenate([(g.uniform(-1, 1, 4000) * 2.0 ** g.integers(-30, 40, 4000)),
                         [0.0, -0.0, 1.0, -3.5, 65504.0, 1e30, -1e-30]]).astype(np.float32)
    h, m, l = km.tf32_parts(ys)
    assert np.array_equal(h.astype(np.float64) + m.astype(np.float64) + l.astype(np.float64),
                          ys.astype(np.float64))
    assert _low13_zero(h).all() and _low13_zero(m).all() and _low13_zero(l).all()
    nz = h != 0
    assert np.all(np.abs(m[nz]) < 2.0 ** -10 * np.abs(h[nz]))
    assert np.all(np.abs(l[nz]) < 2.0 ** -20 * np.abs(h[nz]))
    h, m, l = km.tf32_parts(np.float32([1.0, 0.75, -1024.0, 3.0 * 2 ** 20]))
    assert not m.any() and not l.any()


def test_norm_step_matches_rational_model_and_exact_cases(oracle_lib):
    """norm_step = one profiled tensor-core step on (1, 1, 1) x (h, m, l) with C = dot:
    checked against the exact-rational tc_model rendering, and exact (= dot - nrm / 2) when
    that value is representable on the step's grid (integers)."""
    g = inputs.rng(2206)
    dot = (g.uniform(-1, 1, (7, 50)) * 2.0 ** g.integers(-4, 12, (7, 50))).astype(np.float32)
    nrm = (g.uniform(0, 1, 50) * 2.0 ** g.integers(-6, 14, 50)).astype(np.float32)
    out = km.norm_step(dot, nrm)
    h, m, l = km.tf32_parts(np.float32(-0.5) * nrm)
    for i in range(7):
        for j in range(50):
            parts = np.float32([h[j], m[j], l[j]])
            ref = oracle_lib.tc_model(np.ones(3, np.float32), parts, float(dot[i, j]), "align", 2, "fields")
            assert out[i, j] == np.float32(ref), (i, j)
    di = g.integers(-5000, 5000, (9, 40)).astype(np.float32)
    ni = g.integers(0, 20000, 40).astype(np.float32)
    assert np.array_equal(km.norm_step(di, ni).astype(np.float64),
                          di.astype(np.float64) - 0.5 * ni.astype(np.float64))


def test_dist_tolerance_norm_term_derivation(oracle_lib):
    """The norm step's key error is < 12 * 2^-24 * max(|dot|, |y|) (y = -||x||^2 / 2), the
    bound oracle.dist_tolerance's 6 units of its 9 come from; checked with exact rationals on
    random and adversarial magnitudes (dot and y of equal or very different size, opposite
    signs: cancellation, y with a long tf32 tail)."""
    g = inputs.rng(2207)
    n = 3000
    mag_d = 2.0 ** g.integers(-20, 20, n)
    rel = 2.0 ** g.integers(-12, 12, n)
    dot = (g.uniform(-1, 1, n) * mag_d).astype(np.float32)
    nrm = (g.uniform(0, 1, n) * mag_d * rel).astype(np.float32)
    nrm[::7] = np.float32(2.0) * np.abs(dot[::7])  # dot ~= ||x||^2 / 2: acc cancels to ~0
    h, m, l = km.tf32_parts(np.float32(-0.5) * nrm)
    worst = 0.0
    for t in range(n):
        parts = np.float32([h[t], m[t], l[t]])
        acc = oracle_lib.tc_model(np.ones(3, np.float32), parts, float(dot[t]), "align", 2, "fields")
        exact = Fraction(float(dot[t])) - Fraction(float(nrm[t])) / 2
        err = abs(Fraction(-2.0 * acc) - (-2 * exact))
        scale = max(abs(float(dot[t])), float(nrm[t]) / 2)
        if scale:
            assert err < Fraction(12) * Fraction(2.0 ** -24) * Fraction(scale), t
            worst = max(worst, float(err) / scale / 2.0 ** -24)
    assert worst > 1.0  # the bound is not vacuous: the step does lose bits
    assert oracle_lib.oracle.NORM_UNITS >= 6 + 1 + 2


def test_knn_model_integer_data_is_exact(oracle_lib):
    """On small integers every step is exact, so the kernel model kNN equals the exact kNN."""
    g = inputs.rng(2202)
    X = g.integers(-4, 5, (400, 20)).astype(np.float32)
    Q = g.integers(-4, 5, (37, 20)).astype(np.float32)
    i1, d1 = km.knn_model(X, Q, 9)
    i0, d0 = oracle_lib.knn(X, Q, 9)
    assert np.array_equal(i1, i0) and np.array_equal(d1.astype(np.float64), d0)


def test_knn_model_agrees_with_exact_where_gap(oracle_lib):
    g = inputs.rng(2203)
    X, Q = g.uniform(-1, 1, (600, 48)), g.uniform(-1, 1, (40, 48))
    i1, d1 = km.knn_model(X, Q, 8)
    D = oracle_lib.sqdist(X, Q)
    tau = oracle_lib.dist_tolerance(Q, X)
    for r in range(Q.shape[0]):
        o = np.argsort(D[r], kind="stable")
        if D[r, o[8]] - D[r, o[7]] > tau[r, o[7]] + tau[r, o[8]]:
            assert set(i1[r]) == set(o[:8])
        assert np.all(np.abs(d1[r] - D[r, i1[r]]) <= tau[r, i1[r]])


def test_kmeans_assign_model_integer_and_ties(oracle_lib):
    g = inputs.rng(2204)
    X = g.integers(-3, 4, (500, 12)).astype(np.float32)
    C = g.integers(-3, 4, (17, 12)).astype(np.float32)
    C[9] = C[4]  # duplicate centroid: ties must go to the lower index
    a, best = km.kmeans_assign_model(X, C)
    D = ((X[:, None, :].astype(np.int64) - C[None].astype(np.int64)) ** 2).sum(2)
    assert np.array_equal(a, np.argmin(D, 1))
    assert not np.any(a == 9)
    cn = (C.astype(np.int64) ** 2).sum(1)
    assert np.all(cn[a] - 2 * (X.astype(np.int64) * C[a].astype(np.int64)).sum(1) == best)


def test_group_sums_chunked_within_bound_of_plain(oracle_lib):
    """The kernels' chunked fp64 order vs the oracle's plain ascending sums: counts equal,
    sums within SURVEY c-20's n 2^-52 sum |x|; integer data: bitwise equal."""
    X, _, cent = inputs.mixture(5000, 6, 3, 10, sigma=0.3)
    a, sums, counts, _, _ = oracle_lib.kmeans_step(X, cent)
    s2, c2 = km.group_sums_chunked(X, a, 3)
    assert np.array_equal(c2, counts)
    absx = np.zeros_like(sums)
    np.add.at(absx, a, np.abs(X.astype(np.float64)))
    assert np.all(np.abs(s2 - sums) <= counts[:, None] * 2.0 ** -52 * absx)
    Xi = inputs.integers((3000, 5), 11, lim=100)
    ai = (np.arange(3000) * 7) % 4
    s3, _ = km.group_sums_chunked(Xi, ai, 4)
    ref = np.zeros((4, 5), np.int64)
    np.add.at(ref, ai, Xi.astype(np.int64))
    assert np.array_equal(s3, ref.astype(np.float64))
