"""Tall-skinny configs[2] (65536 x 256 x 1024, the public call with fp32 A and B) at promotion
intervals Kc = 64 / 128 / 256 (fused A, 256 x 256 pair tiles), alternating rounds, with the
normwise error vs the fp64 oracle on a row sample.  Tool code."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_fengwcz0d21_b200 import egemm, inputs  # noqa: E402
from tools.tune_sweep import timeit  # noqa: E402


def main():
    import oracle
    M, N, K = 65536, 256, 1024
    An, Bn = inputs.uniform((M, K), 1), inputs.uniform((K, N), 2)
    A, B = torch.from_numpy(An).cuda(), torch.from_numpy(Bn).cuda()
    D = torch.empty(M, N, device="cuda")
    ws = torch.empty(egemm.gemm_workspace_size(M, N, K), dtype=torch.uint8, device="cuda")
    rows = np.arange(0, M, 97)
    C64 = oracle.gemm64(An[rows], Bn)
    e32 = oracle.normwise_error(oracle.gemm32_naive(An[rows], Bn), An[rows], Bn, C64)
    for rnd in range(3):
        for kc in (64, 128, 256):
            egemm.set_config_ex(cg=2, bn=256, sep=0, kc=kc, fused=1)
            ms = timeit(lambda: egemm.gemm(A, B, out=D, workspace=ws))
            e = oracle.normwise_error(D.cpu().numpy()[rows], An[rows], Bn, C64)
            print("round %d kc=%3d  %.4f ms  %.1f TF/s  err/naive %.3f" % (rnd, kc, ms, 2.0 * M * N * K / ms / 1e9, e / e32),
                  flush=True)
    egemm.set_config_ex()


if __name__ == "__main__":
    main()
