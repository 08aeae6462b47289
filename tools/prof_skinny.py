"""One tall-skinny configs[2] launch (65536 x 256 x 1024) through the bench's public call
(fp32 A and B in, the tuning table's choice, e.g. the fused-A split) for ncu.  Tool code."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_fengwcz0d21_b200 import egemm, inputs  # noqa: E402

M, N, K = 65536, 256, 1024
A = torch.from_numpy(inputs.uniform((M, K), 200)).cuda()
B = torch.from_numpy(inputs.uniform((K, N), 201)).cuda()
D = torch.empty(M, N, device="cuda")
ws = torch.empty(egemm.gemm_workspace_size(M, N, K), dtype=torch.uint8, device="cuda")
egemm.gemm(A, B, out=D, workspace=ws)
torch.cuda.synchronize()
print("ok", egemm.query_config_ex("gemm_b32", M, N, K))
