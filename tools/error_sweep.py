"""Normwise error of egemm_gemm vs the fp64 oracle across tile / promotion configs and K
(evidence for the tuning table's acc_mode / Kc choice).  Tool code: calls oracle/."""
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
from paper_conf_ppopp_fengwcz0d21_b200 import egemm, inputs  # noqa: E402

CONFIGS = [(2, 256, 0, 64), (2, 256, 0, 128), (2, 256, 0, 256), (2, 128, 1, 256),
           (2, 128, 1, 1024), (1, 128, 1, 256), (1, 128, 1, 8192), (1, 128, 0, 64)]


def main():
    M = N = int(os.environ.get("SWEEP_MN", "256"))
    rows = []
    for K in (256, 1024, 4096, 8192):
        for dist in ("uniform", "in_zone"):
            gen = getattr(inputs, dist)
            A, B = gen((M, K), 7 + K), gen((K, N), 8 + K)
            C64 = oracle.gemm64(A, B)
            en = oracle.normwise_error(oracle.gemm32_naive(A, B), A, B, C64)
            e_emu = oracle.normwise_error(oracle.gemm_emu64(A, B, 3), A, B, C64)
            Ad, Bd = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
            for cfg in CONFIGS:
                egemm.set_config(*cfg)
                D = egemm.gemm(Ad, Bd).cpu().numpy()
                e = oracle.normwise_error(D, A, B, C64)
                rows.append(dict(K=K, dist=dist, cfg=cfg, e=e, e_naive=en, e_split=e_emu,
                                 ratio=e / en))
                print("K=%5d %-8s cfg=%-18s e=%.3e naive=%.3e split=%.3e ratio=%.2f" %
                      (K, dist, cfg, e, en, e_emu, e / en), flush=True)
            egemm.set_config(0, 0, 0, 0)
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    json.dump(rows, open(os.path.join(ROOT, "gpurun_out", "error_sweep.json"), "w"), indent=1)


if __name__ == "__main__":
    main()
