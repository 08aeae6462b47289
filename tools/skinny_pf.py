"""Tall-skinny configs[2] (65536 x 256 x 1024, fp32 A and B in, the bench's public call)
under the current environment knobs: steady-state time (CUDA events over ~60 ms batches)
and the in-kernel clock.  Run once per knob setting (knobs are read once per process):
    EGEMM_AS_PREFETCH=4 python tools/skinny_pf.py
Tool code."""
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from paper_conf_ppopp_fengwcz0d21_b200 import egemm, inputs  # noqa: E402
from tune_sweep import timeit  # noqa: E402


def main():
    M, N, K = 65536, 256, 1024
    A = torch.from_numpy(inputs.uniform((M, K), 200)).cuda()
    B = torch.from_numpy(inputs.uniform((K, N), 201)).cuda()
    ws = torch.empty(egemm.gemm_workspace_size(M, N, K), dtype=torch.uint8, device="cuda")
    D = torch.empty((M, N), device="cuda")
    cfgs = [None] + [dict(cg=2, bn=256, sep=0, kc=kc, fused=1, stages=st)
                     for kc in (64, 256) for st in (2, 3)]
    for c in cfgs:
        if c:
            egemm.set_config_ex(**c)
        egemm.debug_clock_stats(reset=True)
        t = timeit(lambda: egemm.gemm(A, B, out=D, workspace=ws), reps=5)
        mhz, cyc, n = egemm.debug_clock_stats(reset=True)
        egemm.set_config_ex()
        print("%-8s cfg=%-60s %.4f ms %6.1f TF/s  %5.0f MHz  %7.0f cycles/launch" % (
            os.environ.get("EGEMM_AS_PREFETCH", "-"), c or egemm.query_config_ex("gemm_b32", M, N, K),
            t, 2.0 * M * N * K / t / 1e9, mhz, cyc), flush=True)


if __name__ == "__main__":
    main()
