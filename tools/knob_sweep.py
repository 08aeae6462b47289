"""The bench's 8192^3 step (table config: split(B^T) + fused-A GEMM) under the current
environment knobs (EGEMM_BAND, EGEMM_PACE_E, EGEMM_PACE_S, ...; read once per process):
a 20-step window (the driver's) and a ~1 s steady-state window, CUDA events.  Run once per
setting:  EGEMM_BAND=10 python tools/knob_sweep.py.  Tool code."""
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_ppopp_fengwcz0d21_b200 import egemm  # noqa: E402


def main():
    n = 8192
    g = torch.Generator(device="cuda").manual_seed(1)
    A = torch.rand(n, n, device="cuda", generator=g) * 2 - 1
    B = torch.rand(n, n, device="cuda", generator=g) * 2 - 1
    bs = (torch.empty((n, n), dtype=torch.int16, device="cuda"), torch.empty((n, n), dtype=torch.int16, device="cuda"))
    D = torch.empty(n, n, device="cuda")
    ws = torch.empty(egemm.gemm_workspace_size(n, n, n, False, True), dtype=torch.uint8, device="cuda")

    def step():
        egemm.split(B, transpose=True, out=bs)
        egemm.gemm(A, None, b_split=bs, out=D, workspace=ws)
    for _ in range(5):
        step()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    out = []
    for steps in (20, 400):
        torch.cuda.synchronize()
        egemm.debug_clock_stats(reset=True)
        s.record()
        for _ in range(steps):
            step()
        e.record()
        e.synchronize()
        ms = s.elapsed_time(e) / steps
        mhz, cyc, _ = egemm.debug_clock_stats(reset=True)
        out.append("%d steps: %.4f ms/step %.1f TF/s (%4.0f MHz, %.0f kcyc)" % (steps, ms, 2 * n ** 3 / ms / 1e9, mhz, cyc / 1e3))
    knobs = " ".join("%s=%s" % (k, v) for k, v in os.environ.items() if k.startswith("EGEMM_"))
    print("%-40s %s" % (knobs or "(defaults)", " | ".join(out)), flush=True)


if __name__ == "__main__":
    main()
