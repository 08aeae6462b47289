"""Bitwise models of choices the KERNELS make where the paper is silent -- regression checks,
not the oracle.

The oracle (``oracle/``) holds the paper's definitions and Alg. 1 in the paper's order.  The
functions here compose oracle primitives with the arithmetic the product kernels chose for
the kNN / kMeans case studies (reading R22, the "norm MMA") and for the kMeans
fp64 sums (the kernels' chunked summation order).  GPU tests compare the kernels with them
bit for bit to catch regressions; parity with the paper is judged against the plain oracle
(exact fp64 kNN / kMeans under the gap rule R18, plain ascending-i sums under the bound of
SURVEY c-20).  Test infrastructure only.
"""
from __future__ import annotations

import numpy as np

import oracle

# ------------------------------------------------------------------ the norm MMA (R22)
def tf32_parts(y):
    """(h, m, l) with y = h + m + l exactly, each an exact tf32 value (13 low fp32 mantissa
    bits zero): h = y with those bits cleared, r = y - h (exact), m = r cleared, l = r - m.
    The kernel feeds them to one kind::tf32 MMA against a tile of ones."""
    y = np.asarray(y, np.float32)
    mask = np.uint32(0xFFFFE000)
    h = (y.view(np.uint32) & mask).view(np.float32)
    r = (y - h).astype(np.float32)
    m = (r.view(np.uint32) & mask).view(np.float32)
    l = (r - m).astype(np.float32)
    return h, m, l


def norm_step(dot, nrm):
    """acc_ij = TC(dot_ij; 1*h_j + 1*m_j + 1*l_j), (h, m, l) = tf32_parts(-nrm_j / 2): the
    tensor-core step (the oracle's profiled primitive) that adds -||x_j||^2 / 2."""
    dot = np.asarray(dot, np.float32)
    nrm = np.asarray(nrm, np.float32)
    h, m, l = tf32_parts(np.float32(-0.5) * nrm)
    parts = np.stack([h, m, l], axis=1)
    ones = np.ones((dot.shape[0], 3), np.float32)
    return oracle.tc_rows(ones, parts, dot)


def knn_model(X, Q, k: int):
    """kNN as the kernel computes it: dot = Alg. 1 over d in one chain (the oracle's
    gemm_alg1_tc, kc = 0), acc = norm_step(dot, ||x||^2), key = -2 acc (exact); the k
    smallest (key, j) ascending; dist = max(0, RN32(||q||^2 + key))."""
    X = np.asarray(X, np.float32)
    Q = np.asarray(Q, np.float32)
    nx = X.shape[0]
    xn = oracle.rownorm(X)
    qn = oracle.rownorm(Q).astype(np.float64)
    dot = oracle.gemm_alg1_tc(Q, X.T, terms=3, sep=0, kc=0)
    key = np.float32(-2.0) * norm_step(dot, xn)
    order = np.lexsort((np.broadcast_to(np.arange(nx), key.shape), key), axis=1)[:, :k]
    kk = np.take_along_axis(key, order, 1)
    dist = (qn[:, None] + kk.astype(np.float64)).astype(np.float32)
    return order.astype(np.int32), np.maximum(dist, np.float32(0.0))


def kmeans_assign_model(X, C):
    """kMeans assignment as the kernel computes it: key_ij = -2 norm_step(x_i . c_j,
    ||c_j||^2), assign_i = the lowest j of minimal key.  Returns (assign, best key)."""
    X = np.asarray(X, np.float32)
    C = np.asarray(C, np.float32)
    cn = oracle.rownorm(C)
    dot = oracle.gemm_alg1_tc(X, C.T, terms=3, sep=0, kc=0)
    key = np.float32(-2.0) * norm_step(dot, cn)
    a = np.argmin(key, axis=1)
    return a.astype(np.int32), key[np.arange(len(a)), a]


# ------------------------------------------------------------------ kMeans fp64 sums
KM_CHUNK = 256  # the kernels' chunk length (csrc/kmeans.cu kKmChunk)


def group_sums_chunked(X, assign, kc: int):
    """The kernels' summation order: members of j in ascending i, cut into chunks of
    KM_CHUNK rows; each chunk summed sequentially from 0.0; the chunk sums added
    sequentially from 0.0 (np.cumsum is a sequential scan)."""
    X = np.asarray(X, np.float32).astype(np.float64)
    a = np.asarray(assign, np.int64)
    d = X.shape[1]
    counts = np.bincount(a, minlength=kc).astype(np.int64)
    order = np.argsort(a, kind="stable")
    starts = np.concatenate([[0], np.cumsum(counts)])
    sums = np.zeros((kc, d), np.float64)
    for j in np.nonzero(counts)[0]:
        rows = X[order[starts[j]:starts[j + 1]]]
        parts = [np.cumsum(rows[c0:c0 + KM_CHUNK], axis=0)[-1] for c0 in range(0, len(rows), KM_CHUNK)]
        sums[j] = np.cumsum(np.stack(parts), axis=0)[-1]
    return sums, counts
