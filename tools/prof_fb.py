"""One fused-B GEMM launch (the 8-GPU per-rank shape: 1024 x 8192 x 8192, pre-split A, fp32 B
split inside the kernel) for ncu.  Tool code."""
import os
import sys

import torch

sys.path.insert(0, os.getcwd())
from paper_conf_ppopp_fengwcz0d21_b200 import egemm, inputs  # noqa: E402

M, N, K = 1024, 8192, 8192
A = torch.from_numpy(inputs.uniform((M, K), 101)).cuda()
B = torch.from_numpy(inputs.uniform((K, N), 102)).cuda()
a_s = egemm.split(A)
D = torch.empty(M, N, device="cuda")
egemm.set_config_ex(cg=2, bn=256, sep=0, kc=256, fused=2)
for _ in range(2):
    egemm.gemm(None, B, a_split=a_s, out=D)
torch.cuda.synchronize()
print("ok")
