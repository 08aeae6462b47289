"""Data parallelism over torch.distributed (NCCL over NVLink / NVSwitch on the B200 box).

The hot path shards naturally: rows of C for the GEMM, query rows for kNN, and
points for kMeans, with the operand that every rank needs (B, the kNN references X, the
kMeans centroids) replicated by one ``broadcast`` before the timed loop.  The only
collective inside a loop is kMeans' per-iteration ``all_reduce`` of the fp64 centroid sums
and int64 counts (the real exchange step of Lloyd's algorithm); every rank then runs the
identical egemm_kmeans_finalize, so the centroids stay bitwise identical across ranks.

The per-rank compute is the C ABI (``egemm``).  ``step``/``finalize`` hooks exist so the
host-side composition can be exercised by gloo tests on CPU.
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def world_size() -> int:
    return dist.get_world_size() if dist.is_available() and dist.is_initialized() else 1


def rank() -> int:
    return dist.get_rank() if dist.is_available() and dist.is_initialized() else 0


def shard_bounds(n: int, world: int, r: int, align: int = 1):
    """Contiguous, balanced [lo, hi) of n items for rank r; shard edges fall on multiples
    of `align` (e.g. the 256-row cluster tile) whenever n allows it."""
    if world <= 1:
        return 0, n
    units = (n + align - 1) // align
    base, rem = divmod(units, world)
    lo_u = r * base + min(r, rem)
    hi_u = lo_u + base + (1 if r < rem else 0)
    return min(n, lo_u * align), min(n, hi_u * align)


def broadcast_(t: torch.Tensor, world: int | None = None, src: int = 0) -> torch.Tensor:
    if (world if world is not None else world_size()) > 1:
        dist.broadcast(t, src)
    return t


def allreduce_sum_(t: torch.Tensor, world: int | None = None) -> torch.Tensor:
    if (world if world is not None else world_size()) > 1:
        dist.all_reduce(t, op=dist.ReduceOp.SUM)
    return t


def gather_rows(local: torch.Tensor, n_total: int, world: int | None = None, align: int = 1):
    """all_gather of row shards (possibly uneven) into a [n_total, ...] tensor."""
    world = world if world is not None else world_size()
    if world <= 1:
        return local
    bounds = [shard_bounds(n_total, world, r, align) for r in range(world)]
    mx = max(b - a for a, b in bounds)
    pad = torch.zeros((mx,) + tuple(local.shape[1:]), dtype=local.dtype, device=local.device)
    pad[: local.shape[0]] = local
    parts = [torch.empty_like(pad) for _ in range(world)]
    dist.all_gather(parts, pad)
    return torch.cat([p[: b - a] for p, (a, b) in zip(parts, bounds)], 0)


def gemm_rows(A_local: torch.Tensor, B: torch.Tensor, terms: int = 0, **kw):
    """This rank's rows of D = A @ B (B replicated): the row-sharded EGEMM."""
    from . import egemm
    return egemm.gemm(A_local, B, terms=terms, **kw)


def knn_queries(X: torch.Tensor, Q_local: torch.Tensor, k: int, **kw):
    """kNN of this rank's query rows against the replicated references X."""
    from . import egemm
    return egemm.knn(X, Q_local, k, **kw)


def knn_references_sharded(X_local: torch.Tensor, x_offset: int, Q: torch.Tensor, k: int,
                           world: int | None = None, knn_fn=None, merge_fn=None, **kw):
    """NEXT-4: kNN with the REFERENCES sharded over ranks (X too big for one GPU); every
    rank holds all queries Q.  Local top-k of this rank's rows X_local (global row ids
    x_offset + j) -> all_gather of the [nq, k] (dist, id) lists -> merge by (dist, id) in
    egemm_knn_merge (the library's exact rank-counting merge, C ABI).  Exchange: 8 * nq * k
    bytes per rank (tiny next to the GEMM).  ``knn_fn(X, Q, k)`` -> (idx, dist) defaults to
    egemm.knn and ``merge_fn(keys [P, nq, k], ids [P, nq, k], k)`` -> (ids, keys) to
    egemm.knn_merge (both injectable for the CPU gloo tests); shards with fewer than k rows
    pad with (+inf, -1).  Returns (idx int64 [nq, k], dist [nq, k]), identical on every rank."""
    world = world if world is not None else world_size()
    nq = Q.shape[0]
    if knn_fn is None or merge_fn is None:
        from . import egemm
        if knn_fn is None:
            knn_fn = lambda X_, Q_, k_: egemm.knn(X_, Q_, k_, **kw)  # noqa: E731
        if merge_fn is None:
            merge_fn = egemm.knn_merge
    kl = min(k, X_local.shape[0])
    idx, dst = knn_fn(X_local, Q, kl) if kl > 0 else (None, None)
    keys = torch.full((nq, k), float("inf"), dtype=dst.dtype if kl > 0 else torch.float32,
                      device=Q.device)
    ids = torch.full((nq, k), -1, dtype=torch.int32, device=Q.device)
    if kl > 0:
        keys[:, :kl] = dst
        ids[:, :kl] = (idx.long() + x_offset).to(torch.int32)
    if world > 1:
        kp = [torch.empty_like(keys) for _ in range(world)]
        ip = [torch.empty_like(ids) for _ in range(world)]
        dist.all_gather(kp, keys)
        dist.all_gather(ip, ids)
        keys, ids = torch.stack(kp), torch.stack(ip)
    else:
        keys, ids = keys[None].contiguous(), ids[None].contiguous()
    mi, mk = merge_fn(keys, ids, k)
    return mi.long(), mk


class SymmPeers:
    """Per-rank kMeans partial buffers in torch SymmetricMemory (NVLink peer-mapped): rank r
    writes its partial sums / counts into its own buffer; every rank can then read all of
    them (``sums[r]`` / ``counts[r]`` are this device's views of rank r's buffer).  Used by
    kmeans_fit(reduce="peer") with egemm_kmeans_allreduce_finalize."""

    def __init__(self, kc: int, d: int, device, group=None):
        import torch.distributed._symmetric_memory as symm_mem
        grp = group or dist.group.WORLD
        self.world, self.rank = dist.get_world_size(grp), dist.get_rank(grp)
        nb = kc * d * 8 + kc * 8
        self.buf = symm_mem.empty(nb, dtype=torch.uint8, device=device)
        self.handle = symm_mem.rendezvous(self.buf, grp.group_name)
        self.sums, self.counts = [], []
        for r in range(self.world):
            b = self.handle.get_buffer(r, (nb,), torch.uint8)
            self.sums.append(b[: kc * d * 8].view(torch.float64).view(kc, d))
            self.counts.append(b[kc * d * 8:].view(torch.int64))

    def local(self):
        return self.sums[self.rank], self.counts[self.rank]

    def barrier(self):
        self.handle.barrier()


def kmeans_fit(X: torch.Tensor, C: torch.Tensor, iters: int, x_split=None, workspace=None,
               bufs=None, world: int | None = None, step=None, finalize=None, reduce: str = "nccl",
               peers=None, peer_finalize=None):
    """Lloyd iterations on this rank's points X with replicated centroids C (updated in
    place).  reduce="nccl": local egemm_kmeans_step -> all_reduce(sums, counts) ->
    egemm_kmeans_finalize.  reduce="peer": the step writes its partials into this rank's
    SymmetricMemory buffer (``peers``, a SymmPeers), a symmetric barrier, then
    egemm_kmeans_allreduce_finalize reads every rank's partials over NVLink, reduces them in
    rank order and updates C (bitwise identical on every rank), and a second barrier keeps
    the next step from overwriting partials a peer is still reading.  The step / finalize
    hooks let the gloo tests drive the same host composition on CPU.
    Returns the last iteration's local assignment."""
    from . import egemm
    world = world if world is not None else world_size()
    step = step or (lambda X_, C_, out: egemm.kmeans_step(
        X_, C_, x_split=x_split, want_inertia=False, workspace=workspace, out=out))
    finalize = finalize or egemm.kmeans_finalize
    assign = None
    packed = None
    if reduce == "peer":
        if peers is None:
            raise ValueError("reduce='peer' needs the SymmPeers buffers")
        peer_finalize = peer_finalize or (lambda P, C_: egemm.kmeans_allreduce_finalize(P.sums, P.counts, C_))
        ls, lc = peers.local()
        abuf = bufs[0] if bufs else torch.empty(X.shape[0], dtype=torch.int32, device=X.device)
        for _ in range(iters):
            assign, _, _, _ = step(X, C, (abuf, ls, lc, None))  # partials into the own buffer
            peers.barrier()          # every rank's partials are written
            peer_finalize(peers, C)  # reduce over peer memory (rank order) + update
            peers.barrier()          # every rank has read them: the next step may overwrite
        return assign
    for _ in range(iters):
        assign, sums, counts, _ = step(X, C, bufs)
        if world > 1:
            # one collective per iteration: the fp64 sums and the counts (as fp64: exact below
            # 2^53) travel in one buffer -- a single NCCL launch / latency instead of two
            ns, nc = sums.numel(), counts.numel()
            if packed is None or packed.numel() != ns + nc or packed.device != sums.device:
                packed = torch.empty(ns + nc, dtype=torch.float64, device=sums.device)
            packed[:ns].copy_(sums.reshape(-1))
            packed[ns:].copy_(counts)
            dist.all_reduce(packed, op=dist.ReduceOp.SUM)
            sums.copy_(packed[:ns].view_as(sums))
            counts.copy_(packed[ns:])
        finalize(sums, counts, C)
    return assign
