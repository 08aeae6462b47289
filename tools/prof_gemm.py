"""The bench's headline GEMM launch (bench.py gemm_call: the tuning table's choice of pre-split
operands, fused-A or fused-B at N^3), a few times, for ncu capture.  Tool code.
usage: python tools/prof_gemm.py N [reps]"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_fengwcz0d21_b200 import egemm, inputs  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 2
A = torch.from_numpy(inputs.uniform((n, n), 101)).cuda()
B = torch.from_numpy(inputs.uniform((n, n), 102)).cuda()
D = torch.empty(n, n, device="cuda")
fused_b = egemm.query_config("gemm_b32", n, n, n, with_fused=True)[4] == 2
fused_a = not fused_b and bool(egemm.query_config("gemm", n, n, n, with_fused=True)[4] & 1)
# the splits the bench's step runs outside the GEMM (the split ncu pass captures these)
a_split = None if fused_a else egemm.split(A)
b_split = None if fused_b else egemm.split(B, transpose=True)
for _ in range(reps):
    if fused_a:
        egemm.gemm(A, None, b_split=b_split, out=D)
    elif fused_b:
        egemm.gemm(None, B, a_split=a_split, out=D)
    else:
        egemm.gemm(None, None, a_split=a_split, b_split=b_split, out=D)
torch.cuda.synchronize()
print("done fused_a=%d fused_b=%d" % (fused_a, fused_b))
