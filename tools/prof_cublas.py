"""cuBLAS fp16 GEMM with the same MMA work as one 8192^3 EGEMM launch (n x n x 3n), for an
ncu side-by-side with egemm_tc_kernel.  Tool code (context, library kernel)."""
import sys
import torch
n = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
A = (torch.rand(n, 3 * n, device="cuda") * 2 - 1).half()
B = (torch.rand(3 * n, n, device="cuda") * 2 - 1).half()
for _ in range(2):
    torch.matmul(A, B)
torch.cuda.synchronize()
print("ok")
