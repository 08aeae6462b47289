"""Quick device-time sweep of the GEMM kernel configs at a square size (tool code)."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_fengwcz0d21_b200 import egemm  # noqa: E402


def timeit(fn, iters=10, warm=3):
    for _ in range(warm):
        fn()
    torch.cuda.synchronize()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ts = []
    for _ in range(iters):
        s.record()
        fn()
        e.record()
        e.synchronize()
        ts.append(s.elapsed_time(e))
    ts.sort()
    return ts[len(ts) // 2]


def main():
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
    cfgs = [tuple(int(v) for v in c.split(",")) for c in sys.argv[2:]] or \
        [(2, 256, 0, 64), (2, 256, 0, 128), (2, 256, 0, 256), (2, 128, 1, 256), (1, 128, 1, 256),
         (1, 128, 0, 256)]
    A = torch.rand(n, n, device="cuda") * 2 - 1
    B = torch.rand(n, n, device="cuda") * 2 - 1
    a_split = egemm.split(A)
    b_split = egemm.split(B, transpose=True)
    D = torch.empty(n, n, device="cuda")
    ws = torch.empty(egemm.gemm_workspace_size(n, n, n), dtype=torch.uint8, device="cuda")
    flop = 2.0 * n ** 3
    t = timeit(lambda: egemm.split(A, out=a_split))
    print("split %d^2: %.3f ms  %.0f GB/s" % (n, t, 8.0 * n * n / t / 1e6))
    t = timeit(lambda: egemm.split(B, transpose=True, out=b_split))
    print("split^T %d^2: %.3f ms  %.0f GB/s" % (n, t, 8.0 * n * n / t / 1e6))
    for cfg in cfgs:
        egemm.set_config(*cfg)
        t = timeit(lambda: egemm.gemm(None, None, a_split=a_split, b_split=b_split, out=D))
        t2 = timeit(lambda: egemm.gemm(A, B, out=D, workspace=ws))
        egemm.gemm(None, None, a_split=a_split, b_split=b_split, out=D)
        mhz = egemm.debug_last_clock()
        peak_at_clk = 148 * 8192 * mhz * 1e6 / 1e12
        print("cfg %-16s gemm(presplit) %.3f ms = %.1f TF (x3 = %.0f TF fp16, SM %.0f MHz -> "
              "%.0f%% of tensor peak at that clock)   full %.3f ms = %.1f TF"
              % (cfg, t, flop / t / 1e9, 3 * flop / t / 1e9, mhz,
                 100 * 3 * flop / t / 1e9 / peak_at_clk, t2, flop / t2 / 1e9), flush=True)
    egemm.set_config(0, 0, 0, 0)
    # cuBLAS context (library, not our path)
    t = timeit(lambda: torch.matmul(A, B))
    print("torch fp32 (tf32 off) matmul: %.3f ms = %.1f TF" % (t, flop / t / 1e9))
    Ah, Bh = A.half(), B.half()
    t = timeit(lambda: torch.matmul(Ah, Bh))
    print("torch fp16 matmul: %.3f ms = %.1f TF" % (t, flop / t / 1e9))


if __name__ == "__main__":
    main()
