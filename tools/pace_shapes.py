"""Paced vs unpaced (EGEMM_NO_PACE) steady-state time of the public GEMM call (fp32 in,
splits included, tuned config) over a set of shapes.  Tool code."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_fengwcz0d21_b200 import egemm  # noqa: E402

SHAPES = [(65536, 256, 1024), (4096, 4096, 1024), (8192, 8192, 1024), (8192, 8192, 2048),
          (8192, 8192, 4096), (4096, 4096, 8192), (16384, 1024, 8192), (2048, 2048, 2048),
          (65536, 1024, 4096), (32768, 8192, 8192)]


def steady(f, window_ms=300.0):
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    f()
    torch.cuda.synchronize()
    s.record()
    f()
    e.record()
    e.synchronize()
    n = max(3, int(window_ms / max(s.elapsed_time(e), 1e-3)))
    for _ in range(max(2, n // 3)):
        f()
    s.record()
    for _ in range(n):
        f()
    e.record()
    e.synchronize()
    return s.elapsed_time(e) / n


def main():
    for (M, N, K) in SHAPES:
        A = torch.rand(M, K, device="cuda") * 2 - 1
        B = torch.rand(K, N, device="cuda") * 2 - 1
        D = torch.empty(M, N, device="cuda")
        ws = torch.empty(egemm.gemm_workspace_size(M, N, K), dtype=torch.uint8, device="cuda")
        f = lambda: egemm.gemm(A, B, out=D, workspace=ws)  # noqa: E731
        res = []
        for rep in range(2):
            for pace in (1, 0):
                if pace:
                    os.environ.pop("EGEMM_NO_PACE", None)
                else:
                    os.environ["EGEMM_NO_PACE"] = "1"
                res.append((pace, steady(f)))
        os.environ.pop("EGEMM_NO_PACE", None)
        p = min(t for q, t in res if q)
        u = min(t for q, t in res if not q)
        print("(%d,%d,%d) cfg %s  paced %.4f ms  free %.4f ms  gain %.3f"
              % (M, N, K, egemm.query_config("gemm", M, N, K, with_fused=True), p, u, u / p), flush=True)
        del A, B, D, ws
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
