"""Per-rank shapes of the row-sharded bench (8192^3 over N = 1, 2, 4, 8 ranks: M = 8192 / N
rows of A and D per rank, all of B): steady-state time of the pre-split GEMM for a list of
tile configs, and of the whole per-rank step (split of A rows + split of B^T + GEMM) with
the tuning table's choice.  One GPU stands in for one rank.  Tool code.
usage: python tools/rank_shapes.py [cg,bn,sep,kc ...]"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from paper_conf_ppopp_fengwcz0d21_b200 import egemm  # noqa: E402
from tune_sweep import timeit  # noqa: E402


def main():
    cfgs = [tuple(int(v) for v in a.split(",")) for a in sys.argv[1:]] or \
        [(2, 256, 0, 256), (2, 224, 0, 256), (2, 224, 0, 128)]
    n = 8192
    B = torch.rand(n, n, device="cuda") * 2 - 1
    b_split = egemm.split(B, transpose=True)
    for world in (1, 2, 4, 8):
        m = n // world
        A = torch.rand(m, n, device="cuda") * 2 - 1
        a_split = egemm.split(A)
        D = torch.empty(m, n, device="cuda")
        ws = torch.empty(egemm.gemm_workspace_size(m, n, n, False, True), dtype=torch.uint8,
                         device="cuda")
        flop = 2.0 * m * n * n
        for cfg in cfgs:
            egemm.set_config(*cfg)
            t = timeit(lambda: egemm.gemm(None, None, a_split=a_split, b_split=b_split, out=D,
                                          workspace=ws))
            print("ranks=%d M=%5d cfg=%-18s gemm %.4f ms  %.1f TF fp32-eq" % (world, m, cfg, t, flop / t / 1e9),
                  flush=True)
        # B round-split inside the GEMM (fa bit 1): no separate B^T split pass per step
        for cfg in [(2, 256, 0, 256), (2, 224, 0, 256)]:
            egemm.set_config_ex(cg=cfg[0], bn=cfg[1], sep=cfg[2], kc=cfg[3], fused=2)
            t = timeit(lambda: egemm.gemm(None, B, a_split=a_split, out=D, workspace=ws))
            t2 = timeit(lambda: egemm.gemm(None, B, a_split=egemm.split(A), out=D,
                                           workspace=ws))
            egemm.set_config_ex()
            print("ranks=%d M=%5d cfg=%-18s fused-B gemm %.4f ms  %.1f TF;  step (A split + fused-B GEMM) "
                  "%.4f ms  %.1f TF per rank, x%d = %.1f" % (world, m, cfg, t, flop / t / 1e9, t2,
                                                             flop / t2 / 1e9, world, world * flop / t2 / 1e9),
                  flush=True)
        egemm.set_config(0, 0, 0, 0)
        choice = egemm.query_config("gemm", m, n, n, with_fused=True)

        def step():
            egemm.split(B, transpose=True, out=b_split)
            egemm.gemm(A, None, b_split=b_split, out=D, workspace=ws)
        t = timeit(step)
        print("ranks=%d M=%5d table=%s  step %.4f ms  %.1f TF fp32-eq per rank, x%d = %.1f" %
              (world, m, choice, t, flop / t / 1e9, world, world * flop / t / 1e9), flush=True)
        del A, a_split, D, ws
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
