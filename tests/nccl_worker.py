"""Worker of tests/test_gpu_nccl.py: ONE rank on cuda:0 with the real NCCL backend (the
pool gives one GPU per box, so the multi-rank data plane cannot run here; this exercises the
NCCL and SymmetricMemory code paths of distributed.py on hardware).  kmeans_fit is driven
with world=2 so its packed fp64 all_reduce really goes through NCCL (identity on one rank).
Writes results to argv[1] (.npz).  Test infrastructure."""
import os
import sys

import numpy as np
import torch
import torch.distributed as dist

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_fengwcz0d21_b200 import distributed as edist  # noqa: E402
from paper_conf_ppopp_fengwcz0d21_b200 import egemm, inputs  # noqa: E402


def main(out_path):
    dev = torch.device("cuda:0")
    torch.cuda.set_device(dev)
    dist.init_process_group("nccl", device_id=dev)
    res = {"backend": np.array([dist.get_backend()])}
    # broadcast / all_reduce / gather through NCCL on CUDA tensors
    B = torch.from_numpy(inputs.uniform((300, 200), 601)).to(dev)
    Bc = B.clone()
    edist.broadcast_(Bc, 2)  # world=2 forces the collective; the group has one rank
    res["bcast_same"] = np.array([bool(torch.equal(Bc, B))])
    t = torch.arange(10, dtype=torch.float64, device=dev)
    edist.allreduce_sum_(t, 2)
    res["allreduce"] = t.cpu().numpy()
    # kMeans: the packed NCCL all_reduce path vs no collective
    X, _, _ = inputs.mixture(4000, 16, 20, 602, sigma=0.2)
    Xd = torch.from_numpy(X).to(dev)
    C1 = torch.from_numpy(X[:20].copy()).to(dev)
    C2 = C1.clone()
    a1 = edist.kmeans_fit(Xd, C1, 3, world=1)
    a2 = edist.kmeans_fit(Xd, C2, 3, world=2)
    res["km_assign1"], res["km_assign2"] = a1.cpu().numpy(), a2.cpu().numpy()
    res["km_C1"], res["km_C2"] = C1.cpu().numpy(), C2.cpu().numpy()
    # SymmetricMemory peer reduce (egemm_kmeans_allreduce_finalize over one peer)
    try:
        peers = edist.SymmPeers(20, 16, dev)
        C3 = torch.from_numpy(X[:20].copy()).to(dev)
        a3 = edist.kmeans_fit(Xd, C3, 3, reduce="peer", peers=peers)
        res["km_assign3"], res["km_C3"] = a3.cpu().numpy(), C3.cpu().numpy()
        res["symm"] = np.array(["ok"])
    except Exception as ex:  # reported, the test decides
        res["symm"] = np.array(["error: %s" % str(ex)[:300]])
    torch.cuda.synchronize()
    np.savez(out_path, **res)
    dist.barrier()
    dist.destroy_process_group()


if __name__ == "__main__":
    main(sys.argv[1])
