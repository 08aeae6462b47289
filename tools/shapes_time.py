"""Steady-state time of the public egemm_gemm call (fp32 A and B, splits included) on the
square sweep and the tall-skinny shape -- the bench's square_sweep timing (CUDA-graph replay
below 0.2 ms).  A/B runs set environment knobs per process (e.g. EGEMM_NO_PDL=1).  Tool code.

usage: python tools/shapes_time.py [tag]
"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_fengwcz0d21_b200 import egemm, inputs  # noqa: E402
from tools.tune_sweep import timeit  # noqa: E402


def main():
    tag = sys.argv[1] if len(sys.argv) > 1 else ""
    shapes = [(1024, 1024, 1024), (2048, 2048, 2048), (4096, 4096, 4096), (65536, 256, 1024),
              (1024, 8192, 8192), (8192, 8192, 8192)]
    for M, N, K in shapes:
        A = torch.from_numpy(inputs.uniform((M, K), 1)).cuda()
        B = torch.from_numpy(inputs.uniform((K, N), 2)).cuda()
        D = torch.empty(M, N, device="cuda")
        ws = torch.empty(egemm.gemm_workspace_size(M, N, K), dtype=torch.uint8, device="cuda")
        f = lambda: egemm.gemm(A, B, out=D, workspace=ws)  # noqa: E731
        ms = timeit(f)
        print("%s %5d x %5d x %5d  %.4f ms  %.1f TF/s fp32-eq  cfg %s" %
              (tag, M, N, K, ms, 2.0 * M * N * K / ms / 1e9,
               egemm.query_config("gemm_b32", M, N, K, with_fused=True)), flush=True)
        del A, B, D, ws


if __name__ == "__main__":
    main()
