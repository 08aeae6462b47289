"""World-size-2 gloo tests (CPU) of the data-parallel composition in
paper_conf_ppopp_fengwcz0d21_b200/distributed.py: shard bounds, broadcast, row gather,
kNN candidate merge and the kMeans loop (local step -> all_reduce -> finalize).  The
per-rank compute is injected (the CPU oracle, test-only): on the GPU box it is the C ABI."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ppopp_fengwcz0d21_b200 import distributed as edist
from paper_conf_ppopp_fengwcz0d21_b200 import inputs


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, fn, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        q.put((rank, fn(rank, world)))
    except Exception as ex:  # pragma: no cover
        q.put((rank, ex))
    finally:
        dist.destroy_process_group()


def _run(fn, world=2):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, fn, q)) for r in range(world)]
    for p in ps:
        p.start()
    out = dict(q.get(timeout=120) for _ in ps)
    for p in ps:
        p.join(timeout=60)
    for r, v in out.items():
        if isinstance(v, Exception):
            raise v
    return out


def test_shard_bounds_cover_and_align():
    for n in (0, 1, 7, 256, 1000, 8192, 8193):
        for world in (1, 2, 3, 8):
            for align in (1, 256):
                b = [edist.shard_bounds(n, world, r, align) for r in range(world)]
                assert b[0][0] == 0 and b[-1][1] == n
                assert all(b[i][1] == b[i + 1][0] for i in range(world - 1))
                if n % align == 0:
                    assert all(lo % align == 0 for lo, _ in b)
    assert edist.shard_bounds(8192, 8, 3, 256) == (3072, 4096)


def _bcast_gather(rank, world):
    t = torch.arange(12, dtype=torch.float32).reshape(3, 4) if rank == 0 else torch.zeros(3, 4)
    edist.broadcast_(t, world)
    lo, hi = edist.shard_bounds(11, world, rank)
    local = torch.arange(lo, hi, dtype=torch.float32)[:, None].repeat(1, 2)
    full = edist.gather_rows(local, 11, world)
    return t.numpy(), full.numpy()


def test_broadcast_and_gather_rows():
    out = _run(_bcast_gather)
    for r in range(2):
        t, full = out[r]
        assert np.array_equal(t, np.arange(12).reshape(3, 4))
        assert np.array_equal(full[:, 0], np.arange(11))


def cpu_merge(keys, ids, k):
    """Host reference of egemm_knn_merge for the gloo tests: per query, the k smallest
    (key, id) of the union of the lists (id -1 = empty slot, padded back with (-1, +inf))."""
    P, nq, kk = keys.shape
    out_i = torch.full((nq, k), -1, dtype=torch.int64)
    out_k = torch.full((nq, k), float("inf"), dtype=keys.dtype)
    for q in range(nq):
        pairs = sorted((float(keys[p, q, t]), int(ids[p, q, t])) for p in range(P) for t in range(kk)
                       if int(ids[p, q, t]) >= 0)[:k]
        for t, (kv, iv) in enumerate(pairs):
            out_i[q, t], out_k[q, t] = iv, kv
    return out_i, out_k


def test_cpu_merge_reference_ties_and_padding():
    keys = torch.tensor([[[0.5, 1.0, float("inf")]], [[0.5, 0.7, 2.0]]])
    ids = torch.tensor([[[9, 4, -1]], [[3, 8, 1]]], dtype=torch.int32)
    i, kk = cpu_merge(keys, ids, 4)
    assert i.tolist() == [[3, 9, 8, 4]]
    assert kk.tolist() == torch.tensor([[0.5, 0.5, 0.7, 1.0]]).tolist()


def _kmeans_ranks(rank, world):
    import oracle
    X, _, _ = inputs.mixture(6000, 8, 16, 3, sigma=0.1)
    C = torch.from_numpy(X[:16].copy())
    lo, hi = edist.shard_bounds(6000, world, rank)
    Xl = torch.from_numpy(X[lo:hi].copy())

    def step(X_, C_, out):
        a, s, c, _, _ = oracle.kmeans_step(X_.numpy(), C_.numpy())
        return torch.from_numpy(a), torch.from_numpy(s), torch.from_numpy(c), None

    def finalize(s, c, C_):
        C_.copy_(torch.from_numpy(oracle.kmeans_finalize(s.numpy(), c.numpy(), C_.numpy())))

    edist.kmeans_fit(Xl, C, 3, world=world, step=step, finalize=finalize)
    return C.numpy()


def test_kmeans_fit_allreduce_equals_single_process(oracle_lib):
    out = _run(_kmeans_ranks)
    assert np.array_equal(out[0], out[1])  # every rank runs the same finalize
    X, _, _ = inputs.mixture(6000, 8, 16, 3, sigma=0.1)
    C = X[:16].copy()
    for _ in range(3):
        a, s, c, _, _ = oracle_lib.kmeans_step(X, C)
        C = oracle_lib.kmeans_finalize(s, c, C)
    # sums were reduced across ranks in another fp64 order: <= 1 ulp of fp32 (R20 note)
    assert np.allclose(out[0], C, rtol=2.0 ** -23, atol=2.0 ** -30)


def _knn_sharded_ranks(rank, world):
    import oracle
    X, _, _ = inputs.mixture(3001, 16, 12, 21, sigma=0.2)
    Q = torch.from_numpy(inputs.uniform((40, 16), 22))
    lo, hi = edist.shard_bounds(3001, world, rank)

    def knn_fn(X_, Q_, k_):
        i, d = oracle.knn(X_.numpy(), Q_.numpy(), k_)
        return torch.from_numpy(i), torch.from_numpy(d)

    i, d = edist.knn_references_sharded(torch.from_numpy(X[lo:hi].copy()), lo, Q, 16,
                                        world=world, knn_fn=knn_fn, merge_fn=cpu_merge)
    return i.numpy(), d.numpy()


def test_knn_references_sharded_equals_single_process(oracle_lib):
    """NEXT-4: references sharded over 2 ranks + all_gather merge == unsharded exact kNN
    (fp64 keys: (dist, id) is a total order, so the result is unique)."""
    out = _run(_knn_sharded_ranks)
    assert np.array_equal(out[0][0], out[1][0]) and np.array_equal(out[0][1], out[1][1])
    X, _, _ = inputs.mixture(3001, 16, 12, 21, sigma=0.2)
    ri, rd = oracle_lib.knn(X, inputs.uniform((40, 16), 22), 16)
    assert np.array_equal(out[0][0], ri) and np.array_equal(out[0][1], rd)


def test_knn_references_sharded_small_shards():
    """Shards with fewer than k rows pad with (+inf, -1) and never displace real rows."""
    X = torch.tensor([[0.0], [1.0], [2.0]])
    Q = torch.tensor([[0.9]])

    def knn_fn(X_, Q_, k_):
        d = ((X_[None, :, 0] - Q_[:, None, 0]) ** 2).double()
        dd, ii = torch.sort(d, dim=1, stable=True)
        return ii[:, :k_], dd[:, :k_]

    parts = [edist.knn_references_sharded(X[a:b], a, Q, 2, world=1, knn_fn=knn_fn,
                                          merge_fn=cpu_merge)
             for a, b in ((0, 1), (1, 3))]
    i0, d0 = parts[0]
    assert i0.tolist() == [[0, -1]] and d0[0, 1].item() == float("inf")
    i1, _ = parts[1]
    assert i1.tolist() == [[1, 2]]


class _GlooPeers:
    """CPU stand-in for distributed.SymmPeers: this rank's partial buffers, and the other
    ranks' gathered at barrier() (gloo all_gather emulates the peer reads)."""

    def __init__(self, kc, d, world, rank):
        self.world, self.rank = world, rank
        self.sums = [torch.zeros(kc, d, dtype=torch.float64) for _ in range(world)]
        self.counts = [torch.zeros(kc, dtype=torch.int64) for _ in range(world)]
        self.phase = 0

    def local(self):
        return self.sums[self.rank], self.counts[self.rank]

    def barrier(self):
        if self.phase == 0:  # first barrier of an iteration: publish the own partials
            gs = [torch.empty_like(self.sums[0]) for _ in range(self.world)]
            gc = [torch.empty_like(self.counts[0]) for _ in range(self.world)]
            dist.all_gather(gs, self.sums[self.rank])
            dist.all_gather(gc, self.counts[self.rank])
            for r in range(self.world):
                if r != self.rank:
                    self.sums[r].copy_(gs[r])
                    self.counts[r].copy_(gc[r])
        else:
            dist.barrier()
        self.phase ^= 1


def _kmeans_peer_ranks(rank, world):
    import oracle
    X, _, _ = inputs.mixture(6000, 8, 16, 3, sigma=0.1)
    C = torch.from_numpy(X[:16].copy())
    lo, hi = edist.shard_bounds(6000, world, rank)
    Xl = torch.from_numpy(X[lo:hi].copy())

    def step(X_, C_, out):
        a, s, c, _, _ = oracle.kmeans_step(X_.numpy(), C_.numpy())
        out[1].copy_(torch.from_numpy(s))
        out[2].copy_(torch.from_numpy(c))
        return torch.from_numpy(a), out[1], out[2], None

    def peer_finalize(P, C_):  # rank-order reduction, as egemm_kmeans_allreduce_finalize
        s = P.sums[0].clone()
        c = P.counts[0].clone()
        for r in range(1, P.world):
            s += P.sums[r]
            c += P.counts[r]
        C_.copy_(torch.from_numpy(oracle.kmeans_finalize(s.numpy(), c.numpy(), C_.numpy())))

    peers = _GlooPeers(16, 8, world, rank)
    edist.kmeans_fit(Xl, C, 3, world=world, step=step, reduce="peer", peers=peers,
                     peer_finalize=peer_finalize)
    return C.numpy()


def test_kmeans_fit_peer_reduce_composition(oracle_lib):
    """reduce='peer' (partials in per-rank buffers, barrier, rank-order reduction + update,
    barrier): identical centroids on every rank, equal to the NCCL-style path's within 1 ulp
    (another fp64 summation order) and to the single process."""
    out = _run(_kmeans_peer_ranks)
    assert np.array_equal(out[0], out[1])
    ref = _run(_kmeans_ranks)[0]
    assert np.allclose(out[0], ref, rtol=2.0 ** -23, atol=2.0 ** -30)
