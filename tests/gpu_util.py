"""Helpers for the -m gpu parity tests (test infrastructure)."""
import numpy as np
import pytest
import torch


def require_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ppopp_fengwcz0d21_b200 import egemm
    egemm.load()  # raises if the library is missing: no silent fallback
    return egemm


def to_dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def to_host(t):
    torch.cuda.synchronize()
    return t.cpu().numpy()


def u16(t):
    return to_host(t).view(np.uint16)


def tail_split_tiles(eg, op, M, N, K):
    """The tiles of a STORE launch that the library runs as tail-split k-parts, and their k-part
    length: a mirror of gemm_tc.cu tail_geometry() and the kernel's band-order unit decode
    (decode_unit, 8 m-tiles per band) for the configuration the library reports for
    (op, M, N, K) -- schedule bookkeeping for the parity tests, no arithmetic.
    Returns (set of (m_tile, n_tile), kpart in k elements, tile height, bn); empty set = none."""
    c = eg.query_config_ex(op, M, N, K)
    cg, bn = c["cg"], c["bn"]
    th = 128 * cg
    none = (set(), 0, th, bn)
    if not c["tail_split"] or c["ksplit"] > 1 or c["tail_peel"] > 0 or min(M, N, K) <= 0:
        return none
    num_kb = -(-K // 64)
    if num_kb < 4:
        return none
    clusters = eg.num_sms() // cg
    if 0 < c["max_clusters"] < clusters:
        clusters = c["max_clusters"]
    mt, nt = -(-M // th), -(-N // bn)
    tiles = mt * nt
    if clusters < 2:
        return none
    rem = tiles % clusters
    if rem == 0 or 2 * rem > clusters:
        return none
    parts = min(4, clusters // rem, num_kb // 2)
    kbpp = -(-num_kb // parts)
    parts = -(-num_kb // kbpp)
    if parts < 2:
        return none
    out = set()
    for u in range(tiles - rem, tiles):
        band = u // (8 * nt)
        m0 = band * 8
        gm = min(8, mt - m0)
        idx = u - band * 8 * nt
        out.add((m0 + idx % gm, idx // gm))
    return out, 64 * kbpp, th, bn


def alg1_rows_with_tail(oracle_lib, A, B, rows, sched, C=None, terms=3, sep=0, kc=0):
    """oracle.gemm_alg1_tc on the given rows of A, with the columns of tail-split tiles taken
    from the same model with kpart (R21's k-parts) -- the reference for a launch whose
    schedule `sched` (tail_split_tiles) split its last wave."""
    tiles, kpart, th, bn = sched
    Cr = None if C is None else C[rows]
    ref = oracle_lib.gemm_alg1_tc(A[rows], B, Cr, terms=terms, sep=sep, kc=kc)
    hit = [(i, n) for i, r in enumerate(rows) for (m, n) in tiles if m == r // th]
    if hit:
        refp = oracle_lib.gemm_alg1_tc(A[rows], B, Cr, terms=terms, sep=sep, kc=kc, kpart=kpart)
        for i, n in hit:
            ref[i, n * bn:(n + 1) * bn] = refp[i, n * bn:(n + 1) * bn]
    return ref
