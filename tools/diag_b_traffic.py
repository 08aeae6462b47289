"""Ceiling of B-operand traffic savings (what multicasting B across clusters could buy at
most): the fused-A GEMM at 8192^3 (the bench's launch) and at configs[2] 65536 x 256 x 1024,
steady state, with B loaded normally vs not at all after the ring's first fill
(EGEMM_DEBUG_MODE=1024 in an EGEMM_DIAG build; results are wrong by design).  Time, in-kernel
clock and CTA-0 cycles.  Run twice: EGEMM_DEBUG_MODE unset / 1024.  Tool code."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from paper_conf_ppopp_fengwcz0d21_b200 import egemm, inputs  # noqa: E402
from tune_sweep import timeit  # noqa: E402


def main():
    for (M, N, K) in ((8192, 8192, 8192), (65536, 256, 1024)):
        A = torch.from_numpy(inputs.uniform((M, K), 200)).cuda()
        B = torch.from_numpy(inputs.uniform((K, N), 201)).cuda()
        b_s = egemm.split(B, transpose=True)
        D = torch.empty((M, N), device="cuda")
        ws = torch.empty(egemm.gemm_workspace_size(M, N, K, False, True), dtype=torch.uint8, device="cuda")
        egemm.set_config_ex(cg=2, bn=256, sep=0, kc=256 if K > 1024 else 64, fused=1)
        try:
            egemm.debug_clock_stats(reset=True)
            t = timeit(lambda: egemm.gemm(A, None, b_split=b_s, out=D, workspace=ws), reps=5)
            mhz, cyc, _ = egemm.debug_clock_stats(reset=True)
        finally:
            egemm.set_config_ex()
        print("mode=%s %dx%dx%d  %.4f ms  %.0f MHz  %.0f cycles" % (
            os.environ.get("EGEMM_DEBUG_MODE", "0"), M, N, K, t, mhz, cyc), flush=True)
        del A, B, b_s, D, ws
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
