"""Phase timeline of CTA 0 of one tensor-core launch (EGEMM_DIAG build, EGEMM_DEBUG_MODE
bit 2048): where a short launch's cycles go -- setup, first load, first MMA, MMA span, the
last chunk's drain and store, exit.  Tool code.

usage: EGEMM_LIB_PATH=.../libegemm_diag.so EGEMM_DEBUG_MODE=2048 python tools/timeline.py
"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_fengwcz0d21_b200 import egemm, inputs  # noqa: E402

NAMES = ["entry", "setup", "1st load", "1st MMA", "last commit", "last chunk rx", "last store",
         "exit bar", "1st conv", "unit2 MMA", "-", "last drained", "stores done", "pre-1st-TMA",
         "producer start"]


def run(M, N, K, fused, kc, cg=2, bn=256, reps=20):
    A = torch.from_numpy(inputs.uniform((M, K), 1)).cuda()
    B = torch.from_numpy(inputs.uniform((K, N), 2)).cuda()
    b_s = egemm.split(B, transpose=True)
    a_s = egemm.split(A)
    D = torch.empty(M, N, device="cuda")
    ws = torch.empty(egemm.gemm_workspace_size(M, N, K, False, True), dtype=torch.uint8, device="cuda")
    egemm.set_config_ex(cg=cg, bn=bn, sep=0, kc=kc, fused=fused)
    f = (lambda: egemm.gemm(A, None, b_split=b_s, out=D, workspace=ws)) if fused == 1 else \
        (lambda: egemm.gemm(None, None, a_split=a_s, b_split=b_s, out=D, workspace=ws))
    acc = None
    for i in range(reps + 3):
        egemm.debug_timeline(reset=True)
        f()
        torch.cuda.synchronize()
        t = egemm.debug_timeline(reset=True)
        if i < 3:
            continue
        d = [(x - t[0]) if x else -1 for x in t[:10]] + [t[11] - t[10]] + \
            [(x - t[0]) if x else -1 for x in t[12:16]]
        acc = d if acc is None else [a + b for a, b in zip(acc, d)]
    egemm.set_config_ex()
    mma = 128 * bn * K * 6 / 8192.0 * (2 if cg == 1 else 1) / (1 if cg == 2 else 2)
    print("M=%d N=%d K=%d fused=%d kc=%d cg=%d bn=%d  (MMA-bound cycles per unit %.0f)" %
          (M, N, K, fused, kc, cg, bn, mma))
    print("   " + "  ".join("%s=%.0f" % (n, a / reps) for n, a in zip(NAMES, acc) if n != "-") +
          "   entry->exit %.0f ns = %.0f MHz" % (acc[10] / reps, acc[7] / acc[10] * 1e3))


if __name__ == "__main__":
    for M, N, K, fz, kc in [(18944, 256, 1024, 0, 64), (18944, 256, 1024, 1, 128), (18944, 256, 1024, 1, 64),
                            (65536, 256, 1024, 1, 64), (2048, 2048, 2048, 1, 128), (256, 256, 4096, 0, 256)]:
        run(M, N, K, fz, kc)
    run(1024, 1024, 1024, 0, 64, 2, 128)
