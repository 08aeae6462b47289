"""Tall-skinny configs[2] (M=65536, N=256, K=1024) diagnostics: the fused-A GEMM vs the
pre-split GEMM alone (split excluded), per config, with in-kernel cycle counts.  Tool code."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_fengwcz0d21_b200 import egemm, inputs  # noqa: E402


def timed(f, it=50):
    for _ in range(3):
        f()
    torch.cuda.synchronize()
    egemm.debug_clock_stats(reset=True)
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    for _ in range(it):
        f()
    e.record()
    e.synchronize()
    mhz, cyc, nl = egemm.debug_clock_stats(reset=True)
    return s.elapsed_time(e) / it, mhz, cyc


def main():
    M, N, K = 65536, 256, 1024
    A = torch.from_numpy(inputs.uniform((M, K), 200)).cuda()
    B = torch.from_numpy(inputs.uniform((K, N), 201)).cuda()
    a_s, b_s = egemm.split(A), egemm.split(B, transpose=True)
    D = torch.empty(M, N, device="cuda")
    need = 6.0 * M * N * K / (148 * 8192.0)
    ws = torch.empty(egemm.gemm_workspace_size(M, N, K, False, True), dtype=torch.uint8, device="cuda")
    print("tensor-bound cycles (all 148 SMs busy):", int(need))
    for cfg in ((2, 256, 0, 64), (2, 256, 0, 128), (2, 128, 1, 128), (2, 128, 0, 64), (2, 128, 0, 128), (1, 128, 0, 64)):
        egemm.set_config(*cfg)
        ms, mhz, cyc = timed(lambda: egemm.gemm(None, None, a_split=a_s, b_split=b_s, out=D))
        print("presplit GEMM", cfg, "%.4f ms  %.0f MHz  %.0f kcyc  eff %.3f" % (ms, mhz, cyc / 1e3, need / cyc))
        egemm.set_config_ex(cg=cfg[0], bn=cfg[1], sep=cfg[2], kc=cfg[3], fused=1)
        try:
            ms, mhz, cyc = timed(lambda: egemm.gemm(A, None, b_split=b_s, out=D, workspace=ws))
            print("fused-A GEMM ", cfg, "%.4f ms  %.0f MHz  %.0f kcyc  eff %.3f" % (ms, mhz, cyc / 1e3, need / cyc))
        except Exception as ex:  # unsupported combination
            print("fused-A GEMM ", cfg, "n/a", str(ex)[:80])
        egemm.set_config_ex()
    egemm.set_config(0, 0, 0, 0)
    ms, _, _ = timed(lambda: egemm.split(A, out=a_s))
    print("split A alone %.4f ms (%.0f GB/s)" % (ms, M * K * 8 / ms / 1e6))


if __name__ == "__main__":
    main()
