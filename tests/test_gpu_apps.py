"""GPU parity of egemm_knn / egemm_kmeans_step against the oracles.

Parity bars (against the plain oracle): (1) the exact fp64 definitions (BASELINE
north_star; reading R18): neighbour sets / assignments identical wherever the oracle's
distance gap exceeds the method's error bound tau; rows within tau are exempt and only
checked for validity; returned distances within tau; (2) kMeans sums within SURVEY c-20's
bound of the oracle's plain ascending-i fp64 sums, counts exact, finalized centroids
within 1 ulp.  Regression checks (bit for bit, no exemptions) against tests/kernel_model.py,
the model of the kernels' own arithmetic (Alg. 1 from the oracle + the R22 norm step +
the kernels' chunked sum order).
"""
import numpy as np
import pytest
import torch

from paper_conf_ppopp_fengwcz0d21_b200 import inputs
from tests import kernel_model as km
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
        assert np.all(np.abs(gdist[i] - D[i, gidx[i]]) <= tau[i, gidx[i]])
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
    (dist, id) in egemm_knn_merge (C ABI) == the kNN rule against the fp64 oracle over all
    of X, and == the unsharded egemm_knn wherever the split does not change the candidates."""
    from paper_conf_ppopp_fengwcz0d21_b200 import distributed as edist
    eg = require_gpu()
    X, Q = inputs.uniform((4100, 96), 60), inputs.uniform((300, 96), 61)
    Xd, Qd = to_dev(X), to_dev(Q)
    cuts = [0, 1000, 1010, 4100]  # a shard with fewer than k rows included
    keys, ids = [], []
    for a, b in zip(cuts[:-1], cuts[1:]):
        i, d = edist.knn_references_sharded(Xd[a:b], a, Qd, 16, world=1)
        ids.append(i.to(torch.int32))
        keys.append(d)
    mi, mk = eg.knn_merge(torch.stack(keys).contiguous(), torch.stack(ids).contiguous(), 16)
    ex = _knn_check(oracle_lib, X, Q, 16, to_host(mi), to_host(mk))
    assert ex <= 300 // 50
    # the distances of a row do not depend on which shard computed them (same arithmetic)
    fi, fd = eg.knn(Xd, Qd, 16)
    same = (to_host(fi) == to_host(mi)).all(1)
    assert same.mean() > 0.95
    assert np.array_equal(to_host(fd)[same], to_host(mk)[same])


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
    # sums / counts of the GPU's own assignment: counts exact; sums within SURVEY c-20's
    # bound of the oracle's plain ascending-i fp64 sums (bitwise against the kernels'
    # chunked order, kernel_model)
    kc, d = C.shape
    ref, rcnt = oracle_lib.kmeans_sums(X, ga, kc)
    assert np.array_equal(gcounts, rcnt)
    assert np.all(np.abs(gsums - ref) <= oracle_lib.kmeans_sums_bound(X, ga, kc))
    ks, _ = km.group_sums_chunked(X, ga, kc)
    assert np.array_equal(gsums, ks)
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
    ga = to_host(a)
    osums, ocnt = oracle_lib.kmeans_sums(X, ga, 32)
    ref = oracle_lib.kmeans_finalize(osums, ocnt, C)
    # integer data: the fp64 sums are exact in any order, so the centroids are bitwise equal
    assert np.array_equal(newc, ref)
    assert np.array_equal(newc[31], C[31])


def test_kmeans_finalize_within_one_ulp(oracle_lib):
    """Non-integer data: the finalized centroids are within 1 fp32 ulp of the oracle's
    finalize of its plain sums for the same assignment (SURVEY c-20)."""
    eg = require_gpu()
    X, _, _ = inputs.mixture(30000, 64, 64, 61, sigma=0.3)
    C = X[:64].copy()
    Xd, Cd = to_dev(X), to_dev(C)
    a, sums, counts, _ = eg.kmeans_step(Xd, Cd)
    eg.kmeans_finalize(sums, counts, Cd)
    osums, ocnt = oracle_lib.kmeans_sums(X, to_host(a), 64)
    ref = oracle_lib.kmeans_finalize(osums, ocnt, C)
    newc = to_host(Cd)
    assert np.all(np.abs(newc.astype(np.float64) - ref) <= np.spacing(np.abs(ref)))


# ------------------------------------------------------------------ regression: kernel model
@pytest.mark.parametrize("nx,nq,d,k,path", [(5000, 64, 128, 16, "index"), (777, 50, 100, 5, "f32"),
                                            (40, 33, 16, 16, "split"), (32768, 24, 128, 16, "index"),
                                            (3000, 300, 64, 8, "f32"),
                                            # d > 128: the streaming-A kernel variant (4+ k-blocks)
                                            (2000, 100, 200, 16, "index"), (1000, 40, 520, 8, "f32")])
def test_knn_bitexact_vs_alg1_model(oracle_lib, nx, nq, d, k, path):
    """egemm_knn equals the kernel model bitwise: indices AND distances (kernel_model.
    knn_model: the oracle's Alg. 1 dot products and plain norms, the R22 norm step, key and
    ordering) -- no gap exemptions."""
    eg = require_gpu()
    X, Q = inputs.uniform((nx, d), 70 + d), inputs.uniform((nq, d), 71 + d)
    Xd, Qd = to_dev(X), to_dev(Q)
    if path == "index":
        idx, dist = eg.knn(None, Qd, k, index=eg.knn_index(Xd))
    elif path == "split":
        idx, dist = eg.knn(Xd, Qd, k, x_split=eg.split(Xd))
    else:
        idx, dist = eg.knn(Xd, Qd, k)
    ri, rd = km.knn_model(X, Q, k)
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
    ri, rd = km.knn_model(X, Q, 16)
    assert np.array_equal(to_host(idx), ri)
    assert np.array_equal(to_host(dist).view(np.uint32), rd.view(np.uint32))


@pytest.mark.parametrize("n,d,kc", [(20000, 64, 1024), (3001, 64, 100), (5000, 32, 7), (999, 130, 300),
                                    (9000, 16, 2000), (7000, 8, 7000), (3000, 4, 50), (5000, 128, 300)])
def test_kmeans_assign_bitexact_vs_alg1_model(oracle_lib, n, d, kc):
    """egemm_kmeans_step's assignment and fp64 sums equal the kernel model bitwise (no gap
    exemptions)."""
    eg = require_gpu()
    X, _, _ = inputs.mixture(n, d, min(kc, 1024), 50 + d, sigma=0.2)
    C = X[:kc].copy()
    a, sums, counts, _ = eg.kmeans_step(to_dev(X), to_dev(C))
    ra, _ = km.kmeans_assign_model(X, C)
    assert np.array_equal(to_host(a), ra)
    rs, rc = km.group_sums_chunked(X, ra, kc)
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
    ra, _ = km.kmeans_assign_model(X, C)
    ga = to_host(a)
    assert np.array_equal(ga, ra)
    assert ga.max() < dup  # the first copy always wins
    rs, rc = km.group_sums_chunked(X, ra, kc)
    assert np.array_equal(to_host(sums), rs) and np.array_equal(to_host(counts), rc)


@pytest.mark.parametrize("scale", [2.0 ** 12, 2.0 ** -9])
def test_knn_kmeans_norm_step_extreme_magnitudes(oracle_lib, scale):
    """The R22 norm step on large (||x||^2 ~ 2^30) and tiny (~2^-12) norms: the tf32 parts
    keep the full fp32 value at any magnitude, and the GPU still equals the model bitwise."""
    eg = require_gpu()
    X = (inputs.uniform((3000, 64), 95) * scale).astype(np.float32)
    Q = (inputs.uniform((70, 64), 96) * scale).astype(np.float32)
    idx, dist = eg.knn(to_dev(X), to_dev(Q), 8)
    ri, rd = km.knn_model(X, Q, 8)
    assert np.array_equal(to_host(idx), ri)
    assert np.array_equal(to_host(dist).view(np.uint32), rd.view(np.uint32))
    C = X[:100].copy()
    a, _, _, _ = eg.kmeans_step(to_dev(X), to_dev(C))
    ra, _ = km.kmeans_assign_model(X, C)
    assert np.array_equal(to_host(a), ra)



@pytest.mark.parametrize("k", [17, 32, 33, 64])
@pytest.mark.parametrize("nx,nq,d", [(5000, 300, 128), (3000, 150, 200)])
def test_knn_long_lists(oracle_lib, k, nx, nq, d):
    """k in (16, 64]: the 32- and 64-entry register lists, query tile resident
    (d <= 128) or streamed; the gap rule against the exact fp64 kNN and bitwise against the
    kernel model."""
    eg = require_gpu()
    X, Q = inputs.uniform((nx, d), 80 + k), inputs.uniform((nq, d), 81 + k)
    idx, dist = eg.knn(None, to_dev(Q), k, index=eg.knn_index(to_dev(X)))
    gi, gd = to_host(idx), to_host(dist)
    ex = _knn_check(oracle_lib, X, Q, k, gi, gd)
    # (the 64th/65th neighbours of 3000 uniform points in d = 200 are often closer than tau:
    # such rows are exempt from set equality but still checked for validity in _knn_check)
    assert ex <= nq // 4
    ri, rd = km.knn_model(X, Q, k)
    assert np.array_equal(gi, ri)
    assert np.array_equal(gd.view(np.uint32), rd.view(np.uint32))


@pytest.mark.parametrize("k,slices", [(16, 1), (16, 7), (64, 3), (40, 16)])
def test_knn_slices_override_same_bits(k, slices):
    """The N-slice count (a tuning-table value) changes only the work split, never the result:
    every slice count gives the same indices and distances (the merge ranks (key, idx))."""
    eg = require_gpu()
    X, Q = inputs.uniform((20000, 64), 85), inputs.uniform((400, 64), 86)
    Xd, Qd = to_dev(X), to_dev(Q)
    ref = eg.knn(Xd, Qd, k)
    eg.set_config_ex(n_slices=slices)
    try:
        got = eg.knn(Xd, Qd, k)
    finally:
        eg.set_config_ex()
    assert torch.equal(ref[0], got[0]) and torch.equal(ref[1], got[1])


def test_knn_merge_call_vs_sort():
    """egemm_knn_merge (NEXT-4's merge through the C ABI) == a full lexicographic sort of the
    union of the lists, with empty slots, equal keys across lists and k > one list's length."""
    eg = require_gpu()
    g = inputs.rng(87)
    nl, nq, kin, k = 5, 300, 12, 40
    keys = np.sort(g.integers(0, 50, (nl, nq, kin)).astype(np.float32), axis=2)
    ids = np.stack([g.permutation(100000)[: nq * kin].reshape(nq, kin) + 100000 * l for l in range(nl)])
    ids = ids.astype(np.int32)
    # sort each list by (key, id)
    for l in range(nl):
        o = np.lexsort((ids[l], keys[l]), axis=1)
        keys[l] = np.take_along_axis(keys[l], o, 1)
        ids[l] = np.take_along_axis(ids[l], o, 1)
    keys[2, :, 8:] = np.inf  # empty tails
    ids[2, :, 8:] = -1
    qn = g.uniform(0, 5, nq).astype(np.float32)
    oi, ok = eg.knn_merge(to_dev(keys), to_dev(ids), k)
    oi2, od2 = eg.knn_merge(to_dev(keys), to_dev(ids), k, qnorm=to_dev(qn))
    oi, ok, oi2, od2 = to_host(oi), to_host(ok), to_host(oi2), to_host(od2)
    for q in range(nq):
        ak = keys[:, q, :].ravel()
        ai = ids[:, q, :].ravel()
        valid = ai >= 0
        o = np.lexsort((ai[valid], ak[valid]))[:k]
        assert np.array_equal(oi[q], ai[valid][o]) and np.array_equal(ok[q], ak[valid][o])
        assert np.array_equal(oi2[q], oi[q])
        assert np.array_equal(od2[q], np.maximum(np.float32(0), qn[q] + ak[valid][o]))
    # fewer valid entries than k: padded with (-1, +inf)
    oi3, ok3 = eg.knn_merge(to_dev(np.full((1, 2, 4), np.inf, np.float32)),
                            to_dev(np.full((1, 2, 4), -1, np.int32)), 3)
    assert np.all(to_host(oi3) == -1) and np.all(np.isinf(to_host(ok3)))


def test_kmeans_allreduce_finalize_peer_buffers(oracle_lib):
    """egemm_kmeans_allreduce_finalize (the exchange step fused with the update over peer
    memory): 3 "ranks" (shards of the points, their partials in separate device buffers, as
    SymmetricMemory peers would be) reduced in rank order == the fp64 rank-order sum of the
    partials + finalize, bitwise; counts exact; sums within SURVEY c-20's bound of the
    oracle's plain sums over all points."""
    eg = require_gpu()
    X, _, _ = inputs.mixture(9000, 32, 40, 65, sigma=0.3)
    C = X[:40].copy()
    Xd, Cd = to_dev(X), to_dev(C)
    cuts = [0, 2500, 6100, 9000]
    ps, pc = [], []
    assign = []
    for a, b in zip(cuts[:-1], cuts[1:]):
        ga, s, c, _ = eg.kmeans_step(Xd[a:b].contiguous(), Cd)
        ps.append(s.clone())
        pc.append(c.clone())
        assign.append(to_host(ga))
    sums_out = torch.empty_like(ps[0])
    cnt_out = torch.empty_like(pc[0])
    newc = Cd.clone()
    eg.kmeans_allreduce_finalize(ps, pc, newc, sums_out, cnt_out)
    ref_s = to_host(ps[0]).copy()
    for t in ps[1:]:
        ref_s = ref_s + to_host(t)  # fp64, rank order
    ref_c = sum(to_host(t) for t in pc)
    assert np.array_equal(to_host(sums_out), ref_s) and np.array_equal(to_host(cnt_out), ref_c)
    assert np.array_equal(to_host(newc), oracle_lib.kmeans_finalize(ref_s, ref_c, C))
    ga = np.concatenate(assign)
    os_, oc = oracle_lib.kmeans_sums(X, ga, 40)
    assert np.array_equal(ref_c, oc)
    assert np.all(np.abs(ref_s - os_) <= oracle_lib.kmeans_sums_bound(X, ga, 40))


@pytest.mark.parametrize("n,d,kc,epi", [(20000, 64, 1024, 16), (5000, 128, 300, 8), (3001, 64, 100, 16)])
def test_kmeans_resident_points_same_bits(oracle_lib, n, d, kc, epi):
    """The point tile resident in smem across the centroid tiles (a_resident, d <= 128) or
    streamed with every centroid tile: the same arithmetic, so the same bits (assignment,
    fp64 sums, counts, inertia)."""
    eg = require_gpu()
    X, _, _ = inputs.mixture(n, d, min(kc, 1024), 70 + d, sigma=0.2)
    C = X[:kc].copy()
    out = {}
    for ar in (0, 1):
        eg.set_config_ex(a_resident=ar, epi_warps=epi)
        try:
            out[ar] = [to_host(t) for t in eg.kmeans_step(to_dev(X), to_dev(C))]
            assert eg.query_config_ex("kmeans", n, kc, d)["a_resident"] == ar
        finally:
            eg.set_config_ex()
    for u, v in zip(out[0], out[1]):
        assert np.array_equal(u.view(np.uint8), v.view(np.uint8))
