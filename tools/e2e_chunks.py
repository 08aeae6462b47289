"""egemm_gemm_host (pinned host buffers, copies inside the timed region) at 8192^3 for several
host chunk heights (EGEMM_HOST_CHUNK), plus the raw pinned H2D / D2H bandwidths.  Tool code."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_fengwcz0d21_b200 import egemm  # noqa: E402


def main():
    n = 8192
    A = (torch.rand(n, n) * 2 - 1).pin_memory()
    B = (torch.rand(n, n) * 2 - 1).pin_memory()
    D = torch.empty(n, n).pin_memory()
    dev = torch.empty(n, n, device="cuda")
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    for name, f in (("h2d", lambda: dev.copy_(A, non_blocking=True)),
                    ("d2h", lambda: D.copy_(dev, non_blocking=True))):
        f()
        torch.cuda.synchronize()
        s.record()
        for _ in range(5):
            f()
        e.record()
        e.synchronize()
        print("%s %.1f GB/s" % (name, 5 * n * n * 4 / (s.elapsed_time(e) * 1e-3) / 1e9), flush=True)
    # both directions at once (the e2e pipeline overlaps them)
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    dev2 = torch.empty(n, n, device="cuda")
    torch.cuda.synchronize()
    s.record()
    with torch.cuda.stream(s1):
        for _ in range(5):
            dev.copy_(A, non_blocking=True)
    with torch.cuda.stream(s2):
        for _ in range(5):
            D.copy_(dev2, non_blocking=True)
    torch.cuda.synchronize()
    e.record()
    e.synchronize()
    print("h2d+d2h concurrent: %.1f GB/s per direction"
          % (5 * n * n * 4 / (s.elapsed_time(e) * 1e-3) / 1e9), flush=True)
    del dev, dev2
    for chunk in (0, 512):
        if chunk:
            os.environ["EGEMM_HOST_CHUNK"] = str(chunk)
        else:
            os.environ.pop("EGEMM_HOST_CHUNK", None)
        ws = torch.empty(egemm.gemm_host_workspace_size(n, n, n), dtype=torch.uint8, device="cuda")
        egemm.gemm_host(A, B, out=D, workspace=ws)
        torch.cuda.synchronize()
        s.record()
        for _ in range(5):
            egemm.gemm_host(A, B, out=D, workspace=ws)
        e.record()
        e.synchronize()
        ms = s.elapsed_time(e) / 5
        print("chunk %s: %.3f ms  %.1f TF/s" % (chunk or "default", ms, 2.0 * n ** 3 / ms / 1e9), flush=True)
        del ws


if __name__ == "__main__":
    main()
