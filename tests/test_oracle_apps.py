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


def test_kmeans_sums_fixed_order_r20(oracle_lib):
    """Reading R20: group members in ascending i, chunks of 256 summed sequentially, then
    the chunk sums sequentially -- checked against a pure-Python rendering of that order
    and against the exact rational sum (fp64 rounding bound)."""
    from fractions import Fraction
    X, lab, cent = inputs.mixture(3000, 3, 2, 9, sigma=0.5)
    a, sums, counts, _, _ = oracle_lib.kmeans_step(X, cent)
    for j in range(2):
        mem = [i for i in range(3000) if a[i] == j]
        assert counts[j] == len(mem) and len(mem) > 600
        for t in range(3):
            tot = 0.0
            for c0 in range(0, len(mem), 256):
                part = 0.0
                for i in mem[c0:c0 + 256]:
                    part = part + float(X[i, t])
                tot = tot + part
            assert sums[j, t] == tot
            exact = sum(Fraction(float(X[i, t])) for i in mem)
            mag = sum(abs(float(X[i, t])) for i in mem)
            assert abs(Fraction(sums[j, t]) - exact) <= Fraction(len(mem) * 2.0 ** -52 * mag)


def test_group_sums_equals_step_sums(oracle_lib):
    X, _, cent = inputs.mixture(5000, 6, 3, 10, sigma=0.3)
    a, sums, counts, _, _ = oracle_lib.kmeans_step(X, cent)
    s2, c2 = oracle_lib.group_sums(X, a, 3)
    assert np.array_equal(s2, sums) and np.array_equal(c2, counts)


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


# ------------------------------------------------------------------ R22 bitwise app models
def test_rownorm_tree_vs_exact(oracle_lib):
    """rownorm_tree (R22) is within 1 fp32 ulp of the correctly rounded exact sum of squares
    and equal to it for nearly all rows; integer rows are exact."""
    from fractions import Fraction
    g = inputs.rng(2201)
    for d in (1, 33, 100, 128, 257):
        X = g.uniform(-2, 2, (300, d)).astype(np.float32)
        tree = oracle_lib.rownorm_tree(X)
        exact = np.array([float(sum(Fraction(float(v)) ** 2 for v in row)) for row in X],
                         np.float64).astype(np.float32)
        ulp = np.spacing(exact)
        assert np.all(np.abs(tree.astype(np.float64) - exact) <= ulp)
        assert np.mean(tree == exact) >= 0.97
    Xi = g.integers(-40, 41, (50, 300)).astype(np.float32)
    assert np.array_equal(oracle_lib.rownorm_tree(Xi), (Xi.astype(np.int64) ** 2).sum(1).astype(np.float32))


def test_knn_alg1_tc_integer_data_is_exact(oracle_lib):
    """On small integers every step is exact, so the TC model kNN equals the exact kNN."""
    g = inputs.rng(2202)
    X = g.integers(-4, 5, (400, 20)).astype(np.float32)
    Q = g.integers(-4, 5, (37, 20)).astype(np.float32)
    i1, d1 = oracle_lib.knn_alg1_tc(X, Q, 9)
    i0, d0 = oracle_lib.knn(X, Q, 9)
    assert np.array_equal(i1, i0) and np.array_equal(d1.astype(np.float64), d0)


def test_knn_alg1_tc_agrees_with_exact_where_gap(oracle_lib):
    g = inputs.rng(2203)
    X, Q = g.uniform(-1, 1, (600, 48)), g.uniform(-1, 1, (40, 48))
    i1, _ = oracle_lib.knn_alg1_tc(X, Q, 8)
    D = oracle_lib.sqdist(X, Q)
    for r in range(Q.shape[0]):
        o = np.argsort(D[r], kind="stable")
        if D[r, o[8]] - D[r, o[7]] > 1e-5:  # far above the method's error bound here
            assert set(i1[r]) == set(o[:8])


def test_kmeans_assign_alg1_tc_integer_and_ties(oracle_lib):
    g = inputs.rng(2204)
    X = g.integers(-3, 4, (500, 12)).astype(np.float32)
    C = g.integers(-3, 4, (17, 12)).astype(np.float32)
    C[9] = C[4]  # duplicate centroid: ties must go to the lower index
    a, best = oracle_lib.kmeans_assign_alg1_tc(X, C)
    D = ((X[:, None, :].astype(np.int64) - C[None].astype(np.int64)) ** 2).sum(2)
    assert np.array_equal(a, np.argmin(D, 1))
    assert not np.any(a == 9)
    cn = (C.astype(np.int64) ** 2).sum(1)
    assert np.array_equal(best.astype(np.int64), (D - (X.astype(np.int64) ** 2).sum(1)[:, None])[np.arange(500), a])
    assert np.all(cn[a] - 2 * (X.astype(np.int64) * C[a].astype(np.int64)).sum(1) == best)


def _low13_zero(x):
    return (np.asarray(x, np.float32).view(np.uint32) & 0x1FFF) == 0


def test_tf32_parts_exact_decomposition(oracle_lib):
    """R22 norm parts: y = h + m + l exactly (checked in fp64), every part an exact tf32
    value (13 low mantissa bits zero), |m| < 2^-10 |h| and |l| < 2^-20 |h|; tf32-exact y
    gives m = l = 0."""
    g = inputs.rng(2205)
    ys = np.concatenate([(g.uniform(-1, 1, 4000) * 2.0 ** g.integers(-30, 40, 4000)),
                         [0.0, -0.0, 1.0, -3.5, 65504.0, 1e30, -1e-30]]).astype(np.float32)
    for y in ys:
        h, m, l = oracle_lib.tf32_parts(y)
        assert float(h) + float(m) + float(l) == float(y)
        assert _low13_zero([h, m, l]).all()
        if h != 0:
            assert abs(m) < 2.0 ** -10 * abs(h) and abs(l) < 2.0 ** -20 * abs(h)
    for y in np.float32([1.0, 0.75, -1024.0, 3.0 * 2 ** 20]):
        assert oracle_lib.tf32_parts(y)[1:] == (0.0, 0.0)


def test_norm_step_matches_rational_model_and_exact_cases(oracle_lib):
    """norm_step = one profiled tensor-core step on (1, 1, 1) x (h, m, l) with C = dot:
    checked against the exact-rational tc_model rendering, and exact (= dot - nrm / 2) when
    that value is representable on the step's grid (integers)."""
    g = inputs.rng(2206)
    dot = (g.uniform(-1, 1, (7, 50)) * 2.0 ** g.integers(-4, 12, (7, 50))).astype(np.float32)
    nrm = (g.uniform(0, 1, 50) * 2.0 ** g.integers(-6, 14, 50)).astype(np.float32)
    out = oracle_lib.norm_step(dot, nrm)
    for i in range(7):
        for j in range(50):
            parts = np.float32(oracle_lib.tf32_parts(np.float32(-0.5) * nrm[j]))
            ref = oracle_lib.tc_model(np.ones(3, np.float32), parts, float(dot[i, j]), "align", 2, "fields")
            assert out[i, j] == np.float32(ref), (i, j)
    di = g.integers(-5000, 5000, (9, 40)).astype(np.float32)
    ni = g.integers(0, 20000, 40).astype(np.float32)
    assert np.array_equal(oracle_lib.norm_step(di, ni).astype(np.float64),
                          di.astype(np.float64) - 0.5 * ni.astype(np.float64))
