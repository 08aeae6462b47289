"""Ceiling of reference-operand traffic savings in the kNN kernel (configs[3]: 1M x 64K,
d=128, k=16): steady-state batches with the references loaded normally vs not at all after
the ring's first fill (EGEMM_DEBUG_MODE=1024 in an EGEMM_DIAG build; results wrong by
design).  Run twice: EGEMM_DEBUG_MODE unset / 1024.  Tool code."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_fengwcz0d21_b200 import egemm, inputs  # noqa: E402


def main():
    nx, nq, d, k = 1 << 20, 1 << 16, 128, 16
    X = torch.from_numpy(inputs.uniform((nx, d), 300)).cuda()
    Q = torch.from_numpy(inputs.uniform((nq, d), 301)).cuda()
    index = egemm.knn_index(X)
    for _ in range(2):
        egemm.knn(None, Q, k, index=index)
    torch.cuda.synchronize()
    egemm.debug_clock_stats(reset=True)
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    for _ in range(5):
        egemm.knn(None, Q, k, index=index)
    e.record()
    e.synchronize()
    mhz, cyc, _ = egemm.debug_clock_stats(reset=True)
    print("mode=%s knn %.3f ms/batch  %.0f MHz  %.0f cycles" % (
        os.environ.get("EGEMM_DEBUG_MODE", "0"), s.elapsed_time(e) / 5, mhz, cyc), flush=True)


if __name__ == "__main__":
    main()
