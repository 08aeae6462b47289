"""GPU parity of egemm_knn / egemm_kmeans_step against the oracles.

Two bars.  (1) Against the exact fp64 definitions (BASELINE north_star; reading R18):
neighbour sets / assignments identical wherever the oracle's distance gap exceeds the
method's error bound tau; rows within tau are exempt and only checked for validity.
(2) Against the bitwise models of the method on the profiled tensor core (R21, R22):
indices, distances and assignments identical bit for bit, no exemptions.
"""
import numpy as np
import pytest
import torch

from paper_conf_ppopp_fengwcz0d21_b200 import inputs
from tests.gpu_util import require_gpu, to_dev, to_host

pytestmark = pytest.mark.gpu


def _knn_check(oracle_lib, X, Q, k, gidx, gdist):
    D = oracle_lib.sqdist(X, Q)  # fp64 [nq, nx]
    tau = oracle_lib.dist_tolerance(Q, X)
    order = np.lexsort((np.broadcast_to(np.arange(X.shape[0]), D.shape), D), axis=1)
    exempt = 0
    for i in range(Q.shape[0]):
        o = order[i]
        dk, dk1 = D[i, o[k - 1]], D[i, o[k]] if k < X.shape[0] else np.inf
        gap_ok = (dk1 - dk) > tau[i, o[k - 1]] + (tau[i, o[k]] if k < X.shape[0] else 0)
        # returned distances must match the oracle's within tau
        assert np.all(np.abs(gdist[i] - D[i, gidx[i]]) <= tau[i, gidx[i]] + 1e-6)
        assert len(set(gidx[i].tolist())) == k
        if gap_ok:
            assert set(gidx[i].tolist()) == set(o[:k].tolist()), i
        else:
            exempt += 1
            # validity: every returned distance is within tau of the true k-th distance
            assert np.all(D[i, gidx[i]] <= dk + tau[i, gidx[i]] + tau[i, o[k - 1]])
    return exempt


@pytest.mark.parametrize("nx,nq,d,k", [(5000, 600, 128, 16), (777, 300, 64, 5), (40, 33, 16, 16),
                                       (3000, 256, 100, 8)])
def test_knn_uniform(oracle_lib, nx, nq, d, k):
    eg = require_gpu()
    X, Q = inputs.uniform((nx, d), 30 + d), inputs.uniform((nq, d), 31 + d)
    idx, dist = eg.knn(to_dev(X), to_dev(Q), k)
    ex = _knn_check(oracle_lib, X, Q, k, to_host(idx), to_host(dist))
    assert ex <= nq // 50


def test_knn_clustered_and_presplit(oracle_lib):
    eg = require_gpu()
    X = inputs.clustered(8000, 128, 40, n_centres=64)
    Q = inputs.clustered(500, 128, 41, n_centres=64, centres_seed=40)
    Xd = to_dev(X)
    idx, dist = eg.knn(Xd, to_dev(Q), 16, x_split=eg.split(Xd))
    _knn_check(oracle_lib, X, Q, 16, to_host(idx), to_host(dist))
    idx2, dist2 = eg.knn(Xd, to_dev(Q), 16)
    assert torch.equal(idx, idx2) and torch.equal(dist, dist2)
    idx3, dist3 = eg.knn(None, to_dev(Q), 16, index=eg.knn_index(Xd))  # the index build path
    assert torch.equal(idx, idx3) and torch.equal(dist, dist3)


def test_knn_references_sharded(oracle_lib):
    """NEXT-4: references split into 3 shards (egemm_knn per shard, ids offset) merged by
    (dist, id) == the kNN rule against the fp64 oracle over all of X."""
    from paper_conf_ppopp_fengwcz0d21_b200 import distributed as edist
    eg = require_gpu()
    X, Q = inputs.uniform((4100, 96), 60), inputs.uniform((300, 96), 61)
    Xd, Qd = to_dev(X), to_dev(Q)
    cuts = [0, 1000, 1010, 4100]  # a shard with fewer than k rows included
    keys, ids = [], []
    for a, b in zip(cuts[:-1], cuts[1:]):
        i, d = edist.knn_references_sharded(Xd[a:b], a, Qd, 16, world=1)
        ids.append(i)
        keys.append(d)
    mk, mi = edist.merge_topk(torch.stack(keys), torch.where(torch.stack(ids) < 0, 1 << 62,
                                                            torch.stack(ids)), 16)
    ex = _knn_check(oracle_lib, X, Q, 16, to_host(mi), to_host(mk))
    assert ex <= 300 // 50


def test_knn_self_match_and_duplicates():
    eg = require_gpu()
    X = inputs.uniform((1000, 32), 42)
    X[500] = X[10]
    idx, dist = eg.knn(to_dev(X), to_dev(X[[10, 20]]), 3)
    i = to_host(idx)
    assert list(i[0][:2]) == [10, 500] and i[1][0] == 20
    # ||q||^2 + ||x||^2 - 2 q.x of identical rows cancels to within the fp32 rounding (R18)
    assert 0.0 <= to_host(dist)[1][0] <= 1e-5


def _kmeans_check(oracle_lib, X, C, ga, gsums, gcounts):
    oa, osums, ocounts, oin, best = oracle_lib.kmeans_step(X, C)
    D = oracle_lib.sqdist(C, X)  # [n, kc]
    tau = oracle_lib.dist_tolerance(X, C)
    part = np.partition(D, 1, axis=1)
    gap = part[:, 1] - part[:, 0]
    tol = 2 * tau.max(axis=1)
    strict = gap > tol
    assert np.array_equal(ga[strict], oa[strict])
    # exempt points: the GPU choice is within tau of the best
    ne = ~strict
    assert np.all(D[ne, ga[ne]] <= part[ne, 0] + tol[ne])
    # sums / counts: recompute from the GPU's own assignment in fp64 and compare
    kc, d = C.shape
    cnt = np.bincount(ga, minlength=kc)
    assert np.array_equal(gcounts, cnt)
    # the GPU sums each group in the fixed order of reading R20, like the oracle: the fp64
    # sums are bitwise equal to the oracle's for the same assignment
    ref, rcnt = oracle_lib.group_sums(X, ga, kc)
    assert np.array_equal(gsums, ref) and np.array_equal(gcounts, rcnt)
    if np.array_equal(ga, oa):
        assert np.array_equal(gsums, osums) and np.array_equal(gcounts, ocounts)
    return int(ne.sum())


@pytest.mark.parametrize("n,d,kc", [(20000, 64, 1024), (3001, 64, 100), (5000, 32, 7), (999, 130, 300)])
def test_kmeans_step(oracle_lib, n, d, kc):
    eg = require_gpu()
    X, lab, cent = inputs.mixture(n, d, min(kc, 1024), 50 + d, sigma=0.2)
    C = X[:kc].copy()  # Forgy init: the first kc points (reading R12)
    a, sums, counts, inertia = eg.kmeans_step(to_dev(X), to_dev(C))
    _kmeans_check(oracle_lib, X, C, to_host(a), to_host(sums), to_host(counts))
    oa, osums, ocounts, oin, _ = oracle_lib.kmeans_step(X, C)
    assert abs(float(to_host(inertia)[0]) - oin) <= 1e-5 * abs(oin)


def test_kmeans_finalize_and_empty_cluster(oracle_lib):
    eg = require_gpu()
    X = inputs.integers((4000, 64), 60, lim=20)
    C = np.concatenate([X[:31], np.full((1, 64), 1e4, np.float32)])
    Xd, Cd = to_dev(X), to_dev(C)
    a, sums, counts, _ = eg.kmeans_step(Xd, Cd)
    assert int(to_host(counts)[31]) == 0
    eg.kmeans_finalize(sums, counts, Cd)
    newc = to_host(Cd)
    ref = oracle_lib.kmeans_finalize(to_host(sums), to_host(counts), C)
    assert np.array_equal(newc, ref)
    assert np.array_equal(newc[31], C[31])


# ------------------------------------------------------------------ bitwise (R21 + R22)
@pytest.mark.parametrize("nx,nq,d,k,path", [(5000, 64, 128, 16, "index"), (777, 50, 100, 5, "f32"),
                                            (40, 33, 16, 16, "split"), (32768, 24, 128, 16, "index"),
                                            (3000, 300, 64, 8, "f32"),
                                            # d > 128: the streaming-A kernel variant (4+ k-blocks)
                                            (2000, 100, 200, 16, "index"), (1000, 40, 520, 8, "f32")])
def test_knn_bitexact_vs_alg1_model(oracle_lib, nx, nq, d, k, path):
    """egemm_knn equals the kNN-on-the-profiled-tensor-core model bitwise: indices AND
    distances (oracle.knn_alg1_tc: Alg. 1 dot products, R22 norms / key / ordering) -- no
    gap exemptions."""
    eg = require_gpu()
    X, Q = inputs.uniform((nx, d), 70 + d), inputs.uniform((nq, d), 71 + d)
    Xd, Qd = to_dev(X), to_dev(Q)
    if path == "index":
        idx, dist = eg.knn(None, Qd, k, index=eg.knn_index(Xd))
    elif path == "split":
        idx, dist = eg.knn(Xd, Qd, k, x_split=eg.split(Xd))
    else:
        idx, dist = eg.knn(Xd, Qd, k)
    ri, rd = oracle_lib.knn_alg1_tc(X, Q, k)
    assert np.array_equal(to_host(idx), ri)
    assert np.array_equal(to_host(dist).view(np.uint32), rd.view(np.uint32))


@pytest.mark.parametrize("nx,d,dup,nq", [(6000, 64, 700, 300), (9000, 128, 37, 200), (4096, 32, 256, 64)])
def test_knn_ties_lowest_index_bitexact(oracle_lib, nx, d, dup, nq):
    """Exact key ties on integer data: the references are `dup` distinct rows repeated down
    the index (copies in other 32-column groups, column halves and 256-column tiles), so the
    16 nearest keys are shared by several columns and the lower indices must win.  This is
    where the filter bound of the kNN epilogue (the 16th key of the union of a row's two
    column-group lists, kept inclusive) could drop a tied column; bitwise vs the model."""
    eg = require_gpu()
    base = inputs.integers((dup, d), 95 + d, lim=4)
    X = np.tile(base, (-(-nx // dup), 1))[:nx].copy()
    Q = inputs.integers((nq, d), 96 + d, lim=4)
    idx, dist = eg.knn(None, to_dev(Q), 16, index=eg.knn_index(to_dev(X)))
    ri, rd = oracle_lib.knn_alg1_tc(X, Q, 16)
    assert np.array_equal(to_host(idx), ri)
    assert np.array_equal(to_host(dist).view(np.uint32), rd.view(np.uint32))


@pytest.mark.parametrize("n,d,kc", [(20000, 64, 1024), (3001, 64, 100), (5000, 32, 7), (999, 130, 300),
                                    (9000, 16, 2000), (7000, 8, 7000), (3000, 4, 50), (5000, 128, 300)])
def test_kmeans_assign_bitexact_vs_alg1_model(oracle_lib, n, d, kc):
    """egemm_kmeans_step's assignment equals the profiled-tensor-core model bitwise, so its
    fp64 sums equal the oracle's R20 sums of that assignment bitwise: the whole step is
    exact against the oracle (no gap exemptions)."""
    eg = require_gpu()
    X, _, _ = inputs.mixture(n, d, min(kc, 1024), 50 + d, sigma=0.2)
    C = X[:kc].copy()
    a, sums, counts, _ = eg.kmeans_step(to_dev(X), to_dev(C))
    ra, _ = oracle_lib.kmeans_assign_alg1_tc(X, C)
    assert np.array_equal(to_host(a), ra)
    rs, rc = oracle_lib.group_sums(X, ra, kc)
    assert np.array_equal(to_host(sums), rs) and np.array_equal(to_host(counts), rc)


@pytest.mark.parametrize("n,d,kc,dup", [(4096, 64, 1024, 512), (3000, 64, 600, 300), (2000, 32, 97, 5)])
def test_kmeans_ties_lowest_index_bitexact(oracle_lib, n, d, kc, dup):
    """Exact ties on integer data: every centroid appears twice (columns j and j + dup, i.e.
    in other 16-column halves, 32-column groups and 256-column tiles), so the minimal key
    is always shared; the assignment must be the lower index (R12/R22), bitwise equal to
    the profiled-tensor-core model."""
    eg = require_gpu()
    X = inputs.integers((n, d), 90 + kc, lim=6)
    base = inputs.integers((dup, d), 91 + kc, lim=6)
    C = np.tile(base, (-(-kc // dup), 1))[:kc].copy()
    a, sums, counts, _ = eg.kmeans_step(to_dev(X), to_dev(C))
    ra, _ = oracle_lib.kmeans_assign_alg1_tc(X, C)
    ga = to_host(a)
    assert np.array_equal(ga, ra)
    assert ga.max() < dup  # the first copy always wins
    rs, rc = oracle_lib.group_sums(X, ra, kc)
    assert np.array_equal(to_host(sums), rs) and np.array_equal(to_host(counts), rc)


@pytest.mark.parametrize("scale", [2.0 ** 12, 2.0 ** -9])
def test_knn_kmeans_norm_step_extreme_magnitudes(oracle_lib, scale):
    """The R22 norm step on large (||x||^2 ~ 2^30) and tiny (~2^-12) norms: the tf32 parts
    keep the full fp32 value at any magnitude, and the GPU still equals the model bitwise."""
    eg = require_gpu()
    X = (inputs.uniform((3000, 64), 95) * scale).astype(np.float32)
    Q = (inputs.uniform((70, 64), 96) * scale).astype(np.float32)
    idx, dist = eg.knn(to_dev(X), to_dev(Q), 8)
    ri, rd = oracle_lib.knn_alg1_tc(X, Q, 8)
    assert np.array_equal(to_host(idx), ri)
    assert np.array_equal(to_host(dist).view(np.uint32), rd.view(np.uint32))
    C = X[:100].copy()
    a, _, _, _ = eg.kmeans_step(to_dev(X), to_dev(C))
    ra, _ = oracle_lib.kmeans_assign_alg1_tc(X, C)
    assert np.array_equal(to_host(a), ra)
