"""Tall-skinny (N=256, K=1024) cost per wave: the fused-A GEMM at M = w x 74 x 256 rows
(w whole waves of the 74 CTA-pair clusters) and at configs[2]'s M = 65536, with in-kernel
cycles per launch (CTA 0's clock64 span).  The slope over w is the steady-state cycles per
256 x 256 x 1024 unit; the intercept is the launch's fixed fill / drain.  Tool code.

usage: python tools/skinny_waves.py [kc ...]       (env knobs as usual, e.g. EGEMM_AS_PREFETCH)
"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_fengwcz0d21_b200 import egemm, inputs  # noqa: E402
from tools.tune_sweep import timeit  # noqa: E402


def main():
    N, K = 256, 1024
    kcs = [int(a) for a in sys.argv[1:]] or [64, 256]
    unit_cyc = 128 * 256 * 64 * 2 * 3 / 8192.0 * (K // 64)  # MMA-bound cycles per unit per SM
    print("MMA-bound cycles per 256x256x%d unit: %.0f" % (K, unit_cyc))
    Mmax = 8 * 74 * 256
    A = torch.from_numpy(inputs.uniform((Mmax, K), 200)).cuda()
    B = torch.from_numpy(inputs.uniform((K, N), 201)).cuda()
    b_s = egemm.split(B, transpose=True)
    D = torch.empty(Mmax, N, device="cuda")
    for kc in kcs:
        for stages in (0,):
            for M in (74 * 256, 2 * 74 * 256, 65536, 4 * 74 * 256, 8 * 74 * 256):
                fz = int(os.environ.get("FUSED", "1"))
                egemm.set_config_ex(cg=2, bn=256, sep=0, kc=kc, fused=fz, stages=stages)
                Am, Dm = A[:M], D[:M]
                ws = torch.empty(egemm.gemm_workspace_size(M, N, K, False, True), dtype=torch.uint8,
                                 device="cuda")
                a_s = egemm.split(Am) if fz == 0 else None
                f = (lambda: egemm.gemm(None, None, a_split=a_s, b_split=b_s, out=Dm, workspace=ws)) if fz == 0 \
                    else (lambda: egemm.gemm(Am, None, b_split=b_s, out=Dm, workspace=ws))  # noqa: E731
                egemm.debug_clock_stats(reset=True)
                ms = timeit(f)
                mhz, cyc, nl = egemm.debug_clock_stats(reset=True)
                waves = M / (74 * 256.0)
                print("kc=%3d stages=%d M=%6d waves=%.2f  %.4f ms  %4.0f MHz  %7.0f cyc/launch  "
                      "%6.0f cyc/wave  tensor-eff %.3f  TF/s(fp32eq) %.1f" %
                      (kc, stages, M, waves, ms, mhz, cyc, cyc / max(1, -(-M // (74 * 256))),
                       unit_cyc * M / (74 * 256.0) / cyc, 2.0 * M * N * K / ms / 1e9))
    egemm.set_config_ex()


if __name__ == "__main__":
    main()
