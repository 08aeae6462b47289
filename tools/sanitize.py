"""Small invocations of every tensor-core kernel variant and the CUDA-core kernels, for
compute-sanitizer (racecheck / synccheck / memcheck).  Tool code.

    compute-sanitizer --tool racecheck python tools/sanitize.py <variant>
"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_ppopp_fengwcz0d21_b200 import egemm, inputs  # noqa: E402

VARIANTS = {
    # name: (env, config (cg, bn, sep, kc), shape)
    "presplit_256": ({}, (2, 256, 0, 64), (300, 520, 200)),
    "presplit_224": ({}, (2, 224, 0, 128), (300, 460, 200)),
    "presplit_128": ({}, (2, 128, 0, 64), (300, 300, 200)),
    "presplit_128_sep": ({}, (2, 128, 1, 128), (300, 300, 200)),
    "cg1_128": ({}, (1, 128, 0, 64), (200, 200, 136)),
    "cg1_128_sep": ({}, (1, 128, 1, 64), (200, 200, 136)),
    "fused_a_staged": ({"fused": 1}, (2, 256, 0, 64), (300, 520, 256)),
    "fused_a_ldg": ({"fused": 1, "EGEMM_A_STAGED": "0"}, (2, 256, 0, 64), (300, 520, 200)),
    "fused_a_128_sep": ({"fused": 1}, (2, 128, 1, 64), (300, 300, 200)),
    "fused_b": ({"fused": 2}, (2, 256, 0, 64), (300, 520, 256)),
    "presplit_256_s2": ({"stages": 2}, (2, 256, 0, 64), (300, 520, 200)),
    "presplit_256_ksplit3": ({"ksplit": 3}, (2, 256, 0, 64), (300, 520, 700)),
    "cg1_128_ksplit2_sep": ({"ksplit": 2}, (1, 128, 1, 128), (200, 200, 600)),
    "fused_a_tail_peel": ({"fused": 1, "tail_peel": 1}, (2, 256, 0, 64), (94 * 256 + 37, 256, 256)),
    "bf16_parts": ({"operand_format": 1}, (2, 256, 0, 64), (300, 520, 200)),
    # 18 tiles on 8 clusters: the last 2 tiles as 4 k-parts each, last-arriver fix-up
    "tail_split": ({"tail_split": 1, "max_clusters": 8}, (2, 256, 0, 64), (5 * 256 + 37, 700, 1100)),
    "fused_a_tail_split": ({"fused": 1, "tail_split": 1, "max_clusters": 8}, (2, 256, 0, 64),
                           (5 * 256 + 37, 700, 1100)),
    "presplit_128_s3": ({"stages": 3}, (2, 128, 0, 64), (300, 300, 200)),
}


def run_gemm(opts, cfg, shape):
    os.environ.update({k: v for k, v in opts.items() if k.startswith("EGEMM_")})
    ex = {k: v for k, v in opts.items() if not k.startswith("EGEMM_")}
    egemm.set_config_ex(cg=cfg[0], bn=cfg[1], sep=cfg[2], kc=cfg[3], **ex)
    M, N, K = shape
    A = torch.from_numpy(inputs.uniform((M, K), 1)).cuda()
    B = torch.from_numpy(inputs.uniform((K, N), 2)).cuda()
    D = egemm.gemm(A, B)
    torch.cuda.synchronize()
    ref = A.double() @ B.double()
    err = (D.double() - ref).abs().max().item()
    print("gemm", cfg, shape, "max abs err %.3e" % err)


def main():
    v = sys.argv[1]
    torch.cuda.set_device(0)
    if v in VARIANTS:
        run_gemm(*VARIANTS[v])
    elif v == "split":
        x = torch.from_numpy(inputs.uniform((300, 333), 3)).cuda()
        flags = torch.zeros(1, dtype=torch.int32, device="cuda")
        egemm.split(x, range_flags=flags)
        egemm.split(x, transpose=True, range_flags=flags)
        egemm.split(x, mode="trunc")
        torch.cuda.synchronize()
        print("split ok")
    elif v in ("knn_ar", "knn_stream", "knn_k64", "knn_k32_stream", "knn_cg1"):
        d = 200 if "stream" in v else 128
        k = 64 if v == "knn_k64" else 32 if v == "knn_k32_stream" else 16
        if v == "knn_cg1":
            egemm.set_config_ex(cg=1, bn=128)
        X = torch.from_numpy(inputs.uniform((3000, d), 4)).cuda()
        Q = torch.from_numpy(inputs.uniform((300, d), 5)).cuda()
        idx, dist = egemm.knn(X, Q, k)
        torch.cuda.synchronize()
        print(v, "ok", idx[0, :4].tolist())
    elif v in ("kmeans", "kmeans_e8"):
        if v == "kmeans_e8":
            egemm.set_config_ex(epi_warps=8)
        X = torch.from_numpy(inputs.uniform((5000, 64), 6)).cuda()
        C = X[:300].clone()
        a, s, c, i = egemm.kmeans_step(X, C)
        egemm.kmeans_finalize(s, c, C)
        torch.cuda.synchronize()
        print("kmeans ok", int(c.sum().item()))
    elif v == "merge":
        keys = torch.sort(torch.rand(3, 100, 16, device="cuda"), dim=2).values
        ids = torch.arange(3 * 100 * 16, device="cuda", dtype=torch.int32).reshape(3, 100, 16)
        i, k = egemm.knn_merge(keys, ids, 20)
        torch.cuda.synchronize()
        print("merge ok", i[0, :3].tolist())
    else:
        raise SystemExit("unknown variant " + v)


if __name__ == "__main__":
    main()
