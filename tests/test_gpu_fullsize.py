"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times
(default tuning table), on outputs the oracle can compute one by one (sampled rows /
queries / points).  Inputs are the bench's seeded recipes."""
import numpy as np
import pytest
import torch

from paper_conf_ppopp_fengwcz0d21_b200 import inputs
from tests import kernel_model as km
from tests.gpu_util import alg1_rows_with_tail, require_gpu, tail_split_tiles, to_dev, to_host

pytestmark = pytest.mark.gpu


def _gemm_sampled(oracle_lib, M, N, K, seed_a, seed_b, n_rows, presplit=False):
    eg = require_gpu()
    A, B = inputs.uniform((M, K), seed_a), inputs.uniform((K, N), seed_b)
    Ad, Bd = to_dev(A), to_dev(B)
    if presplit:  # the bench's step: split(A), split(B^T), GEMM on the pre-split operands
        D = eg.gemm(None, None, a_split=eg.split(Ad), b_split=eg.split(Bd, transpose=True))
    else:
        D = eg.gemm(Ad, Bd)
    D = to_host(D)
    rows = np.sort(inputs.rng(seed_a + 7).choice(M, size=min(n_rows, M), replace=False))
    As = A[rows]
    C64 = oracle_lib.gemm64(As, B)
    e = oracle_lib.normwise_error(D[rows], As, B, C64)
    en = oracle_lib.normwise_error(oracle_lib.gemm32_naive(As, B), As, B, C64)
    assert e <= 1e-6 and e <= 2 * en, (e, en)
    # bitwise: the sampled rows equal the oracle's Alg. 1 on the profiled tensor core (R21)
    # for the (terms, sep, Kc) the tuning table picked for this launch
    # (an fp32-B call looks up the "gemm_b32" rows, a pre-split call the "gemm" rows)
    cg, bn, sep, kc = eg.query_config("gemm" if presplit else "gemm_b32", M, N, K)
    bound = oracle_lib.elem_bound(As, B, kc=kc)
    assert np.all(np.abs(D[rows].astype(np.float64) - C64) <= bound)
    # (plus the last rows: with a tail-split last wave (R21 k-parts) they are split tiles')
    sched = tail_split_tiles(eg, "gemm" if presplit else "gemm_b32", M, N, K)
    br = np.unique(np.concatenate([rows[: min(len(rows), 8)], rows[-4:]]))
    ref = alg1_rows_with_tail(oracle_lib, A, B, br, sched, sep=sep, kc=kc)
    assert np.array_equal(D[br].view(np.uint32), ref.view(np.uint32))
    return e, en


@pytest.mark.parametrize("n", [1024, 4096])
def test_square_sweep_sampled(oracle_lib, n):
    """configs[1] square sweep points (full rows sampled)."""
    _gemm_sampled(oracle_lib, n, n, n, 100 + n.bit_length(), 200 + n.bit_length(), 128)


def test_8192_cube_bench_launch(oracle_lib):
    """configs[1] at 8192^3, exactly the bench step (pre-split operands), 48 sampled rows."""
    e, en = _gemm_sampled(oracle_lib, 8192, 8192, 8192, 101, 102, 48, presplit=True)
    print("8192^3 sampled normwise error %.3e (naive fp32 %.3e)" % (e, en))


def test_16384_cube_sampled(oracle_lib):
    _gemm_sampled(oracle_lib, 16384, 16384, 16384, 115, 215, 16)


@pytest.mark.parametrize("shape", [(4096, 4096, 8192), (16384, 4096, 4096), (2048, 2048, 4096),
                                   (8192, 2048, 2048)])
def test_skewed_fig9_sampled(oracle_lib, shape):
    """NEXT-2: Fig. 9's skewed shapes (N, N, 2N) and (4N, N, N), public call."""
    M, N, K = shape
    _gemm_sampled(oracle_lib, M, N, K, 300 + M.bit_length(), 400 + K.bit_length(), 32)


def test_tall_skinny_full(oracle_lib):
    """configs[2]: M=65536 N=256 K=1024, all rows against the fp64 oracle."""
    _gemm_sampled(oracle_lib, 65536, 256, 1024, 200, 201, 65536)


def test_knn_full_size_sampled_queries(oracle_lib):
    """configs[3]: 1M references x 64K queries, d=128, k=16 (the bench's index path);
    48 sampled queries checked against the exact fp64 kNN under the gap rule (R18)."""
    eg = require_gpu()
    nx, nq, d, k = 1 << 20, 1 << 16, 128, 16
    X, Q = inputs.uniform((nx, d), 300), inputs.uniform((nq, d), 301)
    Xd, Qd = to_dev(X), to_dev(Q)
    idx, dist = eg.knn(Xd, Qd, k, index=eg.knn_index(Xd))
    idx, dist = to_host(idx), to_host(dist)
    qs = np.sort(inputs.rng(302).choice(nq, size=48, replace=False))
    oidx, odist = oracle_lib.knn(X, Q[qs], k + 1)
    exempt = 0
    for t, i in enumerate(qs):
        cand = np.unique(np.concatenate([oidx[t], idx[i]]))
        tau = oracle_lib.dist_tolerance(Q[i:i + 1], X[cand])[0]
        tau_of = dict(zip(cand.tolist(), tau.tolist()))
        gap = odist[t, k] - odist[t, k - 1]
        if gap > tau_of[int(oidx[t, k - 1])] + tau_of[int(oidx[t, k])]:
            assert set(idx[i].tolist()) == set(oidx[t, :k].tolist()), i
        else:
            exempt += 1
        dd = oracle_lib.sqdist(X[idx[i]], Q[i:i + 1])[0]
        assert np.all(np.abs(dist[i] - dd) <= np.array([tau_of[int(j)] for j in idx[i]]))
    assert exempt <= 2
    # and bitwise against the kernel model (regression) on 2 of the sampled queries
    bi, bd = km.knn_model(X, Q[qs[:2]], k)
    assert np.array_equal(idx[qs[:2]], bi)
    assert np.array_equal(dist[qs[:2]].view(np.uint32), bd.view(np.uint32))


def test_kmeans_full_size_step_sampled(oracle_lib):
    """configs[4]: 4M points, d=64, 1024 centroids (Forgy init): one step; 32768 sampled
    points checked against the fp64 argmin under the gap rule; counts exact and the fp64
    sums within SURVEY c-20's bound of the oracle's plain sums of the GPU's assignment."""
    eg = require_gpu()
    n, d, kc = 1 << 22, 64, 1024
    X, _, _ = inputs.mixture(n, d, kc, 400)
    C = X[:kc].copy()
    Xd = to_dev(X)
    a, sums, counts, inertia = eg.kmeans_step(Xd, to_dev(C), x_split=eg.split(Xd))
    a, sums, counts = to_host(a), to_host(sums), to_host(counts)
    ps = np.sort(inputs.rng(401).choice(n, size=32768, replace=False))
    oa, _, _, _, _ = oracle_lib.kmeans_step(X[ps], C)
    D = oracle_lib.sqdist(C, X[ps])
    tau = oracle_lib.dist_tolerance(X[ps], C)
    part = np.partition(D, 1, axis=1)
    strict = (part[:, 1] - part[:, 0]) > 2 * tau.max(axis=1)
    assert np.array_equal(a[ps][strict], oa[strict])
    assert (~strict).sum() <= 0.01 * len(ps)
    ref, rcnt = oracle_lib.kmeans_sums(X, a, kc)
    assert np.array_equal(counts, rcnt)
    assert np.all(np.abs(sums - ref) <= oracle_lib.kmeans_sums_bound(X, a, kc))
    # regression: bitwise against the kernel model on 4096 of the sampled points
    ba, _ = km.kmeans_assign_model(X[ps[:4096]], C)
    assert np.array_equal(a[ps[:4096]], ba)
