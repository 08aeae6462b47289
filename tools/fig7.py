"""Fig. 7 on B200 (NEXT-1): max error |V_p - V_single| (Eq. 10) of the emulated
GEMM vs N for the paper's three series -- EGEMM-TC (round-split), Markidis (truncate-split,
Fig. 4a) and tensor-core half -- plus the normwise error against fp64, on U[-1,1] N^3
problems.  V_single = the oracle's naive fp32 GEMM.  Writes
profiles/fig7_b200.json and prints the paper's T4 series beside ours.  Tool code.

usage: python tools/fig7.py [max_N]
"""
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
from paper_conf_ppopp_fengwcz0d21_b200 import egemm, inputs  # noqa: E402


def paper_series():
    rows = {}
    for line in open(os.path.join(ROOT, "tests", "golden", "fig7_max_error.txt")):
        if line.startswith("#") or not line.strip():
            continue
        n, e, m, h = line.split()
        rows[int(n)] = {"egemm_tc": float(e), "markidis": float(m), "tc_half": float(h)}
    return rows


def run(n_max=4096, sample_rows=256):
    paper = paper_series()
    out = []
    n = 128
    while n <= n_max:
        A, B = inputs.uniform((n, n), 700 + n.bit_length()), inputs.uniform((n, n), 800 + n.bit_length())
        rows = np.sort(inputs.rng(n).choice(n, size=min(n, sample_rows), replace=False))
        Ad, Bd = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
        V32 = oracle.gemm32_naive(A[rows], B)
        C64 = oracle.gemm64(A[rows], B)
        res = {"N": n}
        for name, mode, terms in (("egemm_tc", "round", 3), ("egemm_tc_4terms", "round", 4),
                                  ("markidis", "trunc", 4), ("markidis_3terms", "trunc", 3)):
            a_s = egemm.split(Ad, mode=mode)
            b_s = egemm.split(Bd, transpose=True, mode=mode)
            D = egemm.gemm(None, None, a_split=a_s, b_split=b_s, terms=terms).cpu().numpy()[rows]
            res[name] = {"eq10_max_err": oracle.eq10_max_error(D, V32),
                         "normwise_vs_fp64": oracle.normwise_error(D, A[rows], B, C64)}
        Dh = torch.matmul(Ad.half(), Bd.half()).float().cpu().numpy()[rows]  # cuBLAS-TC-Half
        res["tc_half"] = {"eq10_max_err": oracle.eq10_max_error(Dh, V32),
                          "normwise_vs_fp64": oracle.normwise_error(Dh, A[rows], B, C64)}
        res["paper_t4"] = paper.get(n)
        out.append(res)
        print("N=%5d  egemm %.2e (paper %.1e)  markidis %.2e (paper %.1e)  tc-half %.2e (paper %.1e)"
              % (n, res["egemm_tc"]["eq10_max_err"], paper[n]["egemm_tc"],
                 res["markidis"]["eq10_max_err"], paper[n]["markidis"],
                 res["tc_half"]["eq10_max_err"], paper[n]["tc_half"]), flush=True)
        n *= 2
    return out


if __name__ == "__main__":
    res = run(int(sys.argv[1]) if len(sys.argv) > 1 else 4096)
    os.makedirs(os.path.join(ROOT, "profiles"), exist_ok=True)
    json.dump({"what": "Fig. 7 (P:1768-1847) reproduced on B200: Eq. 10 max |V_p - V_single| "
                       "and normwise error vs fp64, U[-1,1], rows sampled",
               "series": res}, open(os.path.join(ROOT, "profiles", "fig7_b200.json"), "w"), indent=1)
