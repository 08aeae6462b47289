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


def merge_topk(keys: torch.Tensor, idx: torch.Tensor, k: int):
    """Merge per-rank candidate lists [P, nq, k] -> [nq, k] ascending by (key, idx).
    Used when the REFERENCES are sharded (NEXT-4); host-side composition only."""
    P, nq, kk = keys.shape
    kcat = keys.permute(1, 0, 2).reshape(nq, P * kk)
    icat = idx.permute(1, 0, 2).reshape(nq, P * kk)
    # lexicographic (key, idx): stable sort by idx, then stable sort by key
    o1 = torch.argsort(icat, dim=1, stable=True)
    kcat, icat = torch.gather(kcat, 1, o1), torch.gather(icat, 1, o1)
    o2 = torch.argsort(kcat, dim=1, stable=True)
    return torch.gather(kcat, 1, o2)[:, :k], torch.gather(icat, 1, o2)[:, :k]


def kmeans_fit(X: torch.Tensor, C: torch.Tensor, iters: int, x_split=None, workspace=None,
               bufs=None, world: int | None = None, step=None, finalize=None):
    """Lloyd iterations on this rank's points X with replicated centroids C (updated in
    place): local egemm_kmeans_step -> all_reduce(sums, counts) -> egemm_kmeans_finalize.
    Returns the last iteration's local assignment."""
    from . import egemm
    world = world if world is not None else world_size()
    step = step or (lambda X_, C_, out: egemm.kmeans_step(
        X_, C_, x_split=x_split, want_inertia=False, workspace=workspace, out=out))
    finalize = finalize or egemm.kmeans_finalize
    assign = None
    for _ in range(iters):
        assign, sums, counts, _ = step(X, C, bufs)
        allreduce_sum_(sums, world)
        allreduce_sum_(counts, world)
        finalize(sums, counts, C)
    return assign
