"""kNN candidate-path statistics: how many (warp, 32-column group) steps enter the top-k
insertion branch, with and without the cross-slice row bound, per query count.  Tool code
(EGEMM_DEBUG_MODE bit 256 counts; bit 512 disables the row-bound exchange)."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_fengwcz0d21_b200 import egemm, inputs  # noqa: E402


def main():
    nx = 1 << 20
    X = torch.from_numpy(inputs.uniform((nx, 128), 300)).cuda()
    index = egemm.knn_index(X)
    for nq in (8192, 16384, 65536):
        Q = torch.from_numpy(inputs.uniform((nq, 128), 301)).cuda()
        groups = nq * nx / 32 / 32  # warp x 32-column group steps
        for tag, mode in (("row bound", 256), ("no row bound", 256 | 512)):
            os.environ["EGEMM_DEBUG_MODE"] = str(mode)
            egemm.knn(None, Q, 16, index=index)
            torch.cuda.synchronize()
            egemm.debug_counter(reset=True)
            egemm.debug_clock_stats(reset=True)
            egemm.knn(None, Q, 16, index=index)
            torch.cuda.synchronize()
            n = egemm.debug_counter(reset=True)
            _, cyc, _ = egemm.debug_clock_stats(reset=True)
            print("nq=%6d %-13s candidate-path entries %11d = %.3f of the group steps, %.0f kcyc"
                  % (nq, tag, n, n / groups, cyc / 1e3), flush=True)
        os.environ.pop("EGEMM_DEBUG_MODE", None)


if __name__ == "__main__":
    main()
