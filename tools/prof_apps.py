import sys, os, torch
sys.path.insert(0, os.getcwd())
from paper_conf_ppopp_fengwcz0d21_b200 import egemm, inputs
which = sys.argv[1]
if which == "knn":
    nx, nq, d, k = 1 << 20, 1 << 14, 128, 16
    X = torch.from_numpy(inputs.uniform((nx, d), 300)).cuda()
    Q = torch.from_numpy(inputs.uniform((nq, d), 301)).cuda()
    xs = egemm.split(X)
    for _ in range(2): egemm.knn(X, Q, k, x_split=xs)
else:
    n, d, kc = 1 << 22, 64, 1024
    Xh, _, _ = inputs.mixture(n, d, kc, 400)
    X = torch.from_numpy(Xh).cuda(); C = torch.from_numpy(Xh[:kc].copy()).cuda()
    xs = egemm.split(X)
    for _ in range(2): egemm.kmeans_step(X, C, x_split=xs)
torch.cuda.synchronize(); print("ok")
