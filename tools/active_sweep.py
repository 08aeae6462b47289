"""Tensor throughput per SM vs the number of active CTA-pair clusters (max_clusters), on a
pre-split STORE GEMM with long K (M = 2 x 256 x clusters rows, N = 256, K = 8192, Kc = 256):
CTA 0's cycles per unit and the implied fp16 flops per SM-clock.  With the EGEMM_DIAG build
and EGEMM_DEBUG_NO_TMA=1 EGEMM_DEBUG_MODE=2 no operand is loaded (MMA issue rate alone).
Tool code."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_fengwcz0d21_b200 import egemm, inputs  # noqa: E402


def main():
    N, K = 256, int(os.environ.get("K", "8192"))
    upc = 2  # units per cluster
    for nc in (1, 2, 4, 8, 16, 32, 48, 64, 74):
        M = 256 * nc * upc
        A = torch.from_numpy(inputs.uniform((M, K), 1)).cuda()
        B = torch.from_numpy(inputs.uniform((K, N), 2)).cuda()
        a_s, b_s = egemm.split(A), egemm.split(B, transpose=True)
        D = torch.empty(M, N, device="cuda")
        egemm.set_config_ex(cg=2, bn=256, sep=0, kc=256, fused=0, max_clusters=nc)
        f = lambda: egemm.gemm(None, None, a_split=a_s, b_split=b_s, out=D)  # noqa: E731
        for _ in range(3):
            f()
        torch.cuda.synchronize()
        egemm.debug_clock_stats(reset=True)
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        for _ in range(20):
            f()
        e.record()
        e.synchronize()
        mhz, cyc, nl = egemm.debug_clock_stats(reset=True)
        ms = s.elapsed_time(e) / 20
        flops_sm = 2.0 * 128 * 256 * K * 3 * upc
        print("clusters %2d  %.4f ms  %4.0f MHz  %7.0f cyc/launch  %6.0f flops/clk/SM  %.1f TF/s/SM  chip-equiv %.0f TF/s"
              % (nc, ms, mhz, cyc, flops_sm / cyc, flops_sm / (ms * 1e-3) / 1e12 if False else flops_sm / cyc * mhz * 1e6 / 1e12,
                 2.0 * M * N * K * 3 / (ms * 1e-3) / 1e12), flush=True)
        egemm.set_config_ex()
        del A, B, a_s, b_s, D


if __name__ == "__main__":
    main()
