"""Launch a few pre-split EGEMM GEMMs (for ncu capture).  Tool code.
usage: python tools/prof_gemm.py N [cg bn sep kc] [reps]"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_fengwcz0d21_b200 import egemm  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
if len(sys.argv) > 5:
    cg, bn, sep, kc = [int(v) for v in sys.argv[2:6]]
    egemm.set_config_ex(cg=cg, bn=bn, sep=sep, kc=kc, fused=0)
reps = int(sys.argv[6]) if len(sys.argv) > 6 else 3
A = torch.rand(n, n, device="cuda") * 2 - 1
B = torch.rand(n, n, device="cuda") * 2 - 1
a_split = egemm.split(A)
b_split = egemm.split(B, transpose=True)
D = torch.empty(n, n, device="cuda")
for _ in range(reps):
    egemm.gemm(None, None, a_split=a_split, b_split=b_split, out=D)
torch.cuda.synchronize()
print("done")
