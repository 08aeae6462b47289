"""Step-level A/B at square sizes: {split A + split B^T + pre-split GEMM} vs {split B^T +
fused-A GEMM (TMA-staged converters)}, steady-state CUDA-event timing over many steps.
Tool code (decides whether the tuning table should pick the fused path for big squares)."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_fengwcz0d21_b200 import egemm  # noqa: E402


def steady(fn, reps):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    for _ in range(reps):
        fn()
    e.record()
    e.synchronize()
    return s.elapsed_time(e) / reps


def main():
    for n in [int(v) for v in (sys.argv[1:] or ["4096", "8192"])]:
        A = torch.rand(n, n, device="cuda") * 2 - 1
        B = torch.rand(n, n, device="cuda") * 2 - 1
        a_s, b_s = egemm.split(A), egemm.split(B, transpose=True)
        D = torch.empty(n, n, device="cuda")
        ws = torch.empty(egemm.gemm_workspace_size(n, n, n, False, True), dtype=torch.uint8,
                         device="cuda")
        reps = max(10, int(3000 / (6.0 * n ** 3 / 1.3e12 * 1e3)))
        for kc in (128, 256):
            egemm.set_config(2, 256, 0, kc)

            def pre():
                egemm.split(A, out=a_s)
                egemm.split(B, transpose=True, out=b_s)
                egemm.gemm(None, None, a_split=a_s, b_split=b_s, out=D)

            def fused():
                egemm.split(B, transpose=True, out=b_s)
                egemm.gemm(A, None, b_split=b_s, out=D, workspace=ws)

            t0 = steady(pre, reps)
            q = egemm.query_config_ex("gemm", n, n, n)
            egemm.set_config_ex(cg=q["cg"], bn=q["bn"], sep=q["sep"], kc=q["kc"], fused=1)
            t1 = steady(fused, reps)
            egemm.set_config_ex()
            f = 2.0 * n ** 3 / 1e9
            print("n=%d kc=%d  pre-split step %.4f ms (%.1f TF)  fused-A step %.4f ms (%.1f TF)"
                  % (n, kc, t0, f / t0, t1, f / t1), flush=True)
        egemm.set_config(0, 0, 0, 0)
        del A, B, a_s, b_s, D, ws
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
