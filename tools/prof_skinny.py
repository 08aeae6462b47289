"""One pre-split (or fused-A with FA=1) tall-skinny GEMM launch for ncu.  Tool code."""
import os, sys, torch
sys.path.insert(0, os.getcwd())
from paper_conf_ppopp_fengwcz0d21_b200 import egemm, inputs
M, N, K = 65536, 256, 1024
A = torch.from_numpy(inputs.uniform((M, K), 200)).cuda()
B = torch.from_numpy(inputs.uniform((K, N), 201)).cuda()
a_s, b_s = egemm.split(A), egemm.split(B, transpose=True)
D = torch.empty(M, N, device="cuda")
egemm.set_config(2, 256, 0, 128)
if os.environ.get("FA") == "1":
    os.environ["EGEMM_FUSED_A"] = "1"
    egemm.gemm(A, None, b_split=b_s, out=D)
else:
    egemm.gemm(None, None, a_split=a_s, b_split=b_s, out=D)
torch.cuda.synchronize(); print("ok")
