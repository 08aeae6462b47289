"""Fused-A staged GEMM: coupled ring (3 stages of A + B) vs decoupled rings (stages = 4: four
fp32-A slots, two B slots) on the tall-skinny and square shapes, public call (fp32 A and B),
alternating rounds; CTA-0 cycles per launch.  Tool code."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_fengwcz0d21_b200 import egemm, inputs  # noqa: E402
from tools.tune_sweep import timeit  # noqa: E402


def main():
    shapes = [(65536, 256, 1024, 128), (18944, 256, 1024, 128), (131072, 256, 1024, 128),
              (65536, 512, 1024, 128), (2048, 2048, 2048, 128), (8192, 8192, 8192, 256),
              (4096, 4096, 4096, 128)]
    for M, N, K, kc in shapes:
        A = torch.from_numpy(inputs.uniform((M, K), 1)).cuda()
        B = torch.from_numpy(inputs.uniform((K, N), 2)).cuda()
        D = torch.empty(M, N, device="cuda")
        ws = torch.empty(egemm.gemm_workspace_size(M, N, K), dtype=torch.uint8, device="cuda")
        ref = None
        for rnd in range(2):
            for st in (3, 4):
                egemm.set_config_ex(cg=2, bn=256, sep=0, kc=kc, fused=1, stages=st)
                egemm.debug_clock_stats(reset=True)
                ms = timeit(lambda: egemm.gemm(A, B, out=D, workspace=ws))
                mhz, cyc, _ = egemm.debug_clock_stats(reset=True)
                torch.cuda.synchronize()
                if ref is None:
                    ref = D.clone()
                same = bool(torch.equal(D.view(torch.int32), ref.view(torch.int32)))
                print("%6d x %5d x %5d kc=%d stages=%d  %.4f ms  %.1f TF/s  %4.0f MHz  %7.0f cyc  bitwise-same=%s"
                      % (M, N, K, kc, st, ms, 2.0 * M * N * K / ms / 1e9, mhz, cyc, same), flush=True)
        egemm.set_config_ex()
        del A, B, D, ws


if __name__ == "__main__":
    main()
