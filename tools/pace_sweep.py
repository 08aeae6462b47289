"""Sweep the k-pacing parameters (EGEMM_PACE_E k-blocks per epoch, EGEMM_PACE_S slack) on
square pre-split GEMMs: steady-state ms, mean SM clock and cycle efficiency.  Tool code."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_fengwcz0d21_b200 import egemm  # noqa: E402


def run(f, n, seconds=1.0):
    for _ in range(3):
        f()
    torch.cuda.synchronize()
    egemm.debug_clock_stats(reset=True)
    it = max(5, int(seconds * 1e3 / (6.0 * n ** 3 / 1.3e12 * 1e3)))
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    for _ in range(it):
        f()
    e.record()
    e.synchronize()
    ms = s.elapsed_time(e) / it
    mhz, cyc, _ = egemm.debug_clock_stats(reset=True)
    return ms, mhz, 6.0 * n ** 3 / (148 * 8192.0) / cyc


def main():
    sizes = [int(a) for a in sys.argv[1:]] or [8192, 16384]
    combos = [(None, None), (4, 2), (4, 3), (8, 2), (8, 3), (8, 4), (16, 2), (16, 3), (32, 2)]
    if os.environ.get("BANDS"):  # sweep the band height at the default pacing instead
        combos = [("band", int(b)) for b in os.environ["BANDS"].split(",")]
    for n in sizes:
        A = torch.rand(n, n, device="cuda") * 2 - 1
        B = torch.rand(n, n, device="cuda") * 2 - 1
        a_s, b_s = egemm.split(A), egemm.split(B, transpose=True)
        D = torch.empty(n, n, device="cuda")
        ws = torch.empty(egemm.gemm_workspace_size(n, n, n, True, True), dtype=torch.uint8, device="cuda")
        f = lambda: egemm.gemm(None, None, a_split=a_s, b_split=b_s, out=D, workspace=ws)  # noqa: E731
        for rep in range(2):
            for E, S in combos:
                for k in ("EGEMM_NO_PACE", "EGEMM_PACE_E", "EGEMM_PACE_S", "EGEMM_BAND"):
                    os.environ.pop(k, None)
                if E == "band":
                    os.environ["EGEMM_BAND"] = str(S)
                elif E is None:
                    os.environ["EGEMM_NO_PACE"] = "1"
                else:
                    os.environ["EGEMM_PACE_E"], os.environ["EGEMM_PACE_S"] = str(E), str(S)
                ms, mhz, ce = run(f, n)
                print("n=%d E=%s S=%s  %.3f ms  %.0f TF-fp16  %.0f MHz  cyc-eff %.3f"
                      % (n, E, S, ms, 6.0 * n ** 3 / ms / 1e9, mhz, ce), flush=True)
        del A, B, a_s, b_s, D
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
