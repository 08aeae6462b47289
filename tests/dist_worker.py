"""Worker of tests/test_gpu_distributed.py, launched by torchrun with EGEMM_BENCH_SHARE_GPU-style
placement: every rank on cuda:0, gloo for the collectives (the product runs NCCL, one GPU per
rank).  Runs the library's sharded compositions (distributed.py) on the seeded inputs and
has rank 0 save the gathered results to argv[1] (.npz).  Test infrastructure."""
import os
import sys

import numpy as np
import torch
import torch.distributed as dist

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_fengwcz0d21_b200 import distributed as edist  # noqa: E402
from paper_conf_ppopp_fengwcz0d21_b200 import egemm, inputs  # noqa: E402

# shapes shared with the test (single-process references use the same seeds)
GEMM = (1000, 300, 700)
KNN = (5000, 333, 64, 16)       # nx, nq, d, k
KMEANS = (6000, 32, 50, 3)      # n, d, kc, iterations
CFG = dict(cg=2, bn=256, sep=0, kc=128, fused=0, ksplit=1, tail_split=0)


def gemm_inputs():
    M, N, K = GEMM
    return inputs.uniform((M, K), 501), inputs.uniform((K, N), 502)


def knn_inputs():
    nx, nq, d, _ = KNN
    return inputs.uniform((nx, d), 503), inputs.uniform((nq, d), 504)


def kmeans_inputs():
    n, d, kc, _ = KMEANS
    X, _, _ = inputs.mixture(n, d, kc, 505, sigma=0.2)
    return X, X[:kc].copy()


def main(out_path):
    dist.init_process_group("gloo")
    world, rank = dist.get_world_size(), dist.get_rank()
    dev = torch.device("cuda:0")
    torch.cuda.set_device(dev)
    res = {}
    # GEMM: rows of C sharded on 256-row boundaries, B replicated (broadcast from rank 0)
    A, B = gemm_inputs()
    M = A.shape[0]
    r0, r1 = edist.shard_bounds(M, world, rank, align=256)
    Bd = torch.from_numpy(B).to(dev) if rank == 0 else torch.empty(B.shape, device=dev)
    Bc = Bd.cpu()
    edist.broadcast_(Bc, world)  # (gloo: host staging of the broadcast)
    Bd = Bc.to(dev)
    egemm.set_config_ex(**CFG)
    try:
        D_local = edist.gemm_rows(torch.from_numpy(A[r0:r1]).to(dev), Bd)
    finally:
        egemm.set_config_ex()
    res["gemm"] = edist.gather_rows(D_local.cpu(), M, world, align=256).numpy()
    # kNN: query rows sharded, references replicated
    X, Q = knn_inputs()
    nq, k = Q.shape[0], KNN[3]
    q0, q1 = edist.shard_bounds(nq, world, rank)
    idx, dst = edist.knn_queries(torch.from_numpy(X).to(dev), torch.from_numpy(Q[q0:q1]).to(dev), k)
    res["knn_idx"] = edist.gather_rows(idx.cpu(), nq, world).numpy()
    res["knn_dist"] = edist.gather_rows(dst.cpu(), nq, world).numpy()
    # kNN with the references sharded (NEXT-4): local top-k + egemm_knn_merge of all lists
    x0, x1 = edist.shard_bounds(X.shape[0], world, rank)
    si, sd = edist.knn_references_sharded(torch.from_numpy(X[x0:x1]).to(dev), x0,
                                          torch.from_numpy(Q).to(dev), k, world=world)
    res["knn_ref_idx"], res["knn_ref_dist"] = si.cpu().numpy(), sd.cpu().numpy()
    # kMeans: points sharded, one all_reduce of (sums, counts) per iteration
    Xk, C0 = kmeans_inputs()
    n, _, _, iters = KMEANS
    p0, p1 = edist.shard_bounds(n, world, rank)
    C = torch.from_numpy(C0).to(dev)
    a = edist.kmeans_fit(torch.from_numpy(Xk[p0:p1]).to(dev), C, iters, world=world)
    res["kmeans_assign"] = edist.gather_rows(a.cpu(), n, world).numpy()
    res["kmeans_C"] = C.cpu().numpy()
    if rank == 0:
        np.savez(out_path, **res)
    dist.barrier()
    dist.destroy_process_group()


if __name__ == "__main__":
    main(sys.argv[1])
