"""Pins for the kNN / kMeans oracles (the GEMM-based case studies [9], [2] the paper
plugs EGEMM-TC into: P:142-145) and for the tensor-core
candidate models of the precision probe (Sec. 3.1; artifact P:2874-2908)."""
import os

import numpy as np
import pytest

from paper_conf_ppopp_fengwcz0d21_b200 import inputs

HERE = os.path.dirname(os.path.abspath(__file__))


def test_knn_brute_force_tiny(oracle_lib):
    X, Q = inputs.uniform((50, 3), 1), inputs.uniform((7, 3), 2)
    idx, dist = oracle_lib.knn(X, Q, 5)
    for i in range(7):
        d = [(sum((float(Q[i, t]) - float(X[j, t])) ** 2 for t in range(3)), j) for j in range(50)]
        d.sort()
        assert [j for _, j in d[:5]] == list(idx[i])
        assert np.allclose([v for v, _ in d[:5]], dist[i], rtol=1e-15, atol=0)


def test_knn_d1_is_sorting(oracle_lib):
    X = inputs.integers((40, 1), 3, lim=10)  # many equal distances: ties -> lower index
    Q = np.array([[0.0], [3.0], [-10.0]], np.float32)
    idx, dist = oracle_lib.knn(X, Q, 40)
    for i in range(3):
        key = sorted(range(40), key=lambda j: ((float(Q[i, 0]) - float(X[j, 0])) ** 2, j))
        assert list(idx[i]) == key


def test_knn_planted_duplicates(oracle_lib):
    X = inputs.uniform((30, 8), 4)
    X[17] = X[3]
    Q = X[3:4].copy()
    idx, dist = oracle_lib.knn(X, Q, 2)
    assert list(idx[0]) == [3, 17] and dist[0, 0] == 0 and dist[0, 1] == 0


def test_kmeans_single_cluster_mean(oracle_lib):
    X = inputs.uniform((1000, 5), 5)
    C = np.zeros((1, 5), np.float32)
    a, sums, counts, inertia, best = oracle_lib.kmeans_step(X, C)
    assert np.all(a == 0) and counts[0] == 1000
    newc = oracle_lib.kmeans_finalize(sums, counts, C)
    assert np.allclose(newc[0], X.astype(np.float64).mean(0), rtol=0, atol=1e-7)
    assert np.isclose(inertia, float((X.astype(np.float64) ** 2).sum()), rtol=1e-12)


def test_kmeans_separated_mixture_recovers_labels(oracle_lib):
    X, lab, centres = inputs.mixture(4000, 16, 8, 6, sigma=0.02)
    a, *_ = oracle_lib.kmeans_step(X, centres)
    assert np.array_equal(a, lab)


def test_kmeans_integer_sums_exact_and_empty_cluster(oracle_lib):
    X = inputs.integers((500, 4), 7, lim=20)
    C = np.array([[0, 0, 0, 0], [1000, 1000, 1000, 1000], [5, 5, 5, 5]], np.float32)
    a, sums, counts, _, _ = oracle_lib.kmeans_step(X, C)
    assert counts[1] == 0 and counts.sum() == 500
    for j in (0, 2):
        ref = X[a == j].astype(np.int64).sum(0)
        assert np.array_equal(sums[j], ref.astype(np.float64))
    newc = oracle_lib.kmeans_finalize(sums, counts, C)
    assert np.array_equal(newc[1], C[1])  # empty cluster keeps its centroid (R12)


def test_kmeans_sums_plain_order(oracle_lib):
    """SURVEY c-6: sums_j = sum of (double) x_i over the members of j in ascending i.
    Closed form: members 2^53, 1, -2^53 (all fp32) in that order give (2^53 + 1) - 2^53 = 0
    (2^53 + 1 rounds to the even 2^53), where any order adding the 1 last would give 1.
    And on mixed data the sums are within n 2^-52 sum |x| of the exact rational sums."""
    from fractions import Fraction
    X = np.array([[2.0 ** 53], [1.0], [-2.0 ** 53]], np.float32)
    _, sums, counts, _, _ = oracle_lib.kmeans_step(X, np.zeros((1, 1), np.float32))
    assert counts[0] == 3 and sums[0, 0] == 0.0
    X, lab, cent = inputs.mixture(3000, 3, 2, 9, sigma=0.5)
    a, sums, counts, _, _ = oracle_lib.kmeans_step(X, cent)
    for j in range(2):
        mem = [i for i in range(3000) if a[i] == j]
        assert counts[j] == len(mem) and len(mem) > 600
        for t in range(3):
            exact = sum(Fraction(float(X[i, t])) for i in mem)
            mag = sum(abs(float(X[i, t])) for i in mem)
            assert abs(Fraction(sums[j, t]) - exact) <= Fraction(len(mem) * 2.0 ** -52 * mag)


def test_rownorm_plain_definition(oracle_lib):
    """||x||^2 = fp32(fp64 sum of squares in ascending t).  Closed form for the order:
    (2^12, 1, 2^-15 x 4): in ascending t the fp64 sum is 2^24 + 1 (each 2^-30 falls below
    half an fp64 ulp of 2^24), an fp32 tie that rounds to the even 2^24; the reverse order
    keeps 4 * 2^-30 = 2^-28 and would round up to 2^24 + 2.  Integer rows are exact; random
    rows equal the correctly rounded exact value (the fp64 error, <= d 2^-53 of the sum,
    cannot move an fp32 rounding except within that distance of a midpoint)."""
    from fractions import Fraction
    x = np.array([[2.0 ** 12, 1.0] + [2.0 ** -15] * 4], np.float32)
    assert oracle_lib.rownorm(x)[0] == np.float32(2.0 ** 24)
    assert oracle_lib.rownorm(x[:, ::-1])[0] == np.float32(2.0 ** 24 + 2)
    g = inputs.rng(2201)
    Xi = g.integers(-40, 41, (50, 300)).astype(np.float32)
    assert np.array_equal(oracle_lib.rownorm(Xi), (Xi.astype(np.int64) ** 2).sum(1).astype(np.float32))
    for d in (1, 33, 128, 257):
        X = g.uniform(-2, 2, (200, d)).astype(np.float32)
        got = oracle_lib.rownorm(X)
        for r in range(X.shape[0]):
            ex = sum(Fraction(float(v)) ** 2 for v in X[r])
            want = np.float32(oracle_lib.oracle._round_f32(ex, "rn"))  # correctly rounded
            w = Fraction(float(want))
            mids = [(w + Fraction(float(np.nextafter(want, np.float32(t))))) / 2 for t in (0, np.inf)]
            if min(abs(ex - m) for m in mids) > Fraction(d) * Fraction(2.0 ** -52) * ex:
                assert got[r] == want, (d, r)


def test_sqdist_closed_forms(oracle_lib):
    """Integer rows: exact integer distances; d = 1: (q - x)^2; symmetric in its arguments."""
    g = inputs.rng(2210)
    X = g.integers(-50, 51, (30, 17)).astype(np.float32)
    Q = g.integers(-50, 51, (9, 17)).astype(np.float32)
    D = oracle_lib.sqdist(X, Q)
    ref = ((Q[:, None, :].astype(np.int64) - X[None].astype(np.int64)) ** 2).sum(2)
    assert np.array_equal(D, ref.astype(np.float64))
    x1, q1 = np.float32([[0.1], [-3.5]]), np.float32([[2.25]])
    assert np.array_equal(oracle_lib.sqdist(x1, q1)[0],
                          [(2.25 - float(np.float32(0.1))) ** 2, (2.25 + 3.5) ** 2])
    U, V = inputs.uniform((12, 8), 2211), inputs.uniform((7, 8), 2212)
    assert np.array_equal(oracle_lib.sqdist(U, V), oracle_lib.sqdist(V, U).T)


def test_kmeans_ties_lowest_index(oracle_lib):
    X = np.array([[0.0, 0.0]], np.float32)
    C = np.array([[1.0, 0.0], [0.0, 1.0], [-1.0, 0.0]], np.float32)
    a, *_ = oracle_lib.kmeans_step(X, C)
    assert a[0] == 0


# ------------------------------------------------------------ tensor-core models
def test_round_f32_matches_numpy_cast(oracle_lib):
    """RN rounding of exact dyadic values == numpy's correctly rounded double->float cast."""
    from fractions import Fraction
    g = inputs.rng(8)
    v = g.standard_normal(2000) * np.exp2(g.integers(-30, 30, 2000))
    for x in v:
        assert oracle_lib.oracle._round_f32(Fraction(float(x)), "rn") == float(np.float32(x))
        rz = oracle_lib.oracle._round_f32(Fraction(float(x)), "rz")
        assert abs(rz) <= abs(float(x)) and abs(float(x) - rz) < abs(float(np.spacing(np.float32(x)))) * 1.0000001


def _golden_example():
    rows = {}
    for line in open(os.path.join(HERE, "golden", "paper_profiling_example.txt")):
        if line.startswith("#") or not line.strip():
            continue
        name, val, hx = line.split()
        le = bytes.fromhex(hx[2:])
        rows[name] = (float(val), np.frombuffer(le, "<u4")[0])
    return rows


def test_paper_profiling_example_decodes():
    """the hex strings are little-endian fp32 dumps; the tensor-core result
    is exactly 1 ulp below the fp32 round-to-nearest result (truncation on T4)."""
    rows = _golden_example()
    for name, (val, bits) in rows.items():
        f = np.uint32(bits).view(np.float32)
        assert abs(float(f) - val) < 1e-5, name
    assert rows["single_result"][1] - rows["tensor_core"][1] == 1


def test_tc_models_reduce_to_textbook_cases(oracle_lib):
    """Exactly representable sums: every model returns the exact value.  A sum that lies
    strictly between two fp32 neighbours: RZ picks the lower magnitude (as the paper's
    T4 example), RN the nearer."""
    m = oracle_lib.tc_model
    a = [1.0, 2.0, 0.5] + [0.0] * 13
    b = [3.0, 0.25, 4.0] + [0.0] * 13
    for model in ("rn", "rz", "align"):
        assert m(a, b, 1.5, model) == 3.0 + 0.5 + 2.0 + 1.5
    c = float(np.float32(934.40625))  # fp32 grid at 934 is 2^-14
    a2 = [2.0 ** -8] + [0.0] * 15
    b2 = [2.0 ** -7 * 1.5] + [0.0] * 15  # adds 0.75 * 2^-14: between two fp32 values
    assert m(a2, b2, c, "rz") == c
    assert m(a2, b2, c, "rn") == c + 2.0 ** -14
    # alignment truncation loses the small product entirely when it sits below the grid
    a3 = [2.0 ** -14] + [0.0] * 15
    b3 = [2.0 ** -14] + [0.0] * 15
    assert m(a3, b3, 1.0, "align", 3) == 1.0 and m(a3, b3, 1.0, "rn") == 1.0
