"""Promotion-interval A/B at 8192^3 (pre-split GEMM only), alternating the order, with the
in-kernel clock probe: mean SM clock and SM cycles per launch.  Tool code."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_fengwcz0d21_b200 import egemm  # noqa: E402


def main():
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
    kcs = [int(v) for v in (sys.argv[2:] or ["256", "128", "256", "128", "512", "256"])]
    A = torch.rand(n, n, device="cuda") * 2 - 1
    B = torch.rand(n, n, device="cuda") * 2 - 1
    a_s, b_s = egemm.split(A), egemm.split(B, transpose=True)
    D = torch.empty(n, n, device="cuda")
    need = 6.0 * n ** 3 / (148 * 8192.0)
    reps = max(10, int(2500 / (6.0 * n ** 3 / 1.3e12 * 1e3)))
    for kc in kcs:
        egemm.set_config(2, 256, 0, kc)
        f = lambda: egemm.gemm(None, None, a_split=a_s, b_split=b_s, out=D)
        for _ in range(3):
            f()
        torch.cuda.synchronize()
        egemm.debug_clock_stats(reset=True)
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        for _ in range(reps):
            f()
        e.record()
        e.synchronize()
        ms = s.elapsed_time(e) / reps
        mhz, cyc, _ = egemm.debug_clock_stats(reset=True)
        print("n=%d kc=%d  %.4f ms  %.0f TF-fp16  %.0f MHz  %.0f kcyc/launch  cycle-eff %.3f"
              % (n, kc, ms, 6.0 * n ** 3 / ms / 1e9, mhz, cyc / 1e3, need / cyc), flush=True)


if __name__ == "__main__":
    main()
