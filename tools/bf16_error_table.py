"""NEXT-3 error table: the fp16 round-split (the paper's) against its bf16 variant (bf16 hi / lo
parts: the fp32 exponent range, 8 + 8 significant bits), 3 and 4 terms, on input families
inside and outside fp16's range; cuBLAS's own fp32 emulation (BF16x9) as context.  Normwise
error vs the oracle's fp64 GEMM on 64 sampled rows, and the ratio to the oracle's naive fp32
GEMM (the north-star bar is <= 2x).  Writes gpurun_out/bf16_error_table.json.
Tool code (calls oracle/ for the reference)."""
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import bench  # noqa: E402  (cuBLAS BF16x9 helper; preloads the system cuBLAS before torch)

bench._preload_system_cublas()
import torch  # noqa: E402

import oracle  # noqa: E402
from paper_conf_ppopp_fengwcz0d21_b200 import egemm, inputs  # noqa: E402


def fam(name, shape, seed):
    g = inputs.rng(seed)
    u = g.uniform(-1, 1, shape)
    if name == "uniform":
        return inputs.uniform(shape, seed)
    if name == "in_zone":
        return inputs.in_zone(shape, seed)
    if name == "stress_fp16_range":
        return inputs.stress(shape, seed)
    if name == "wide_2^+-40":
        return (u * 2.0 ** g.integers(-40, 40, shape)).astype(np.float32)
    if name == "normal":
        return g.standard_normal(shape).astype(np.float32)
    raise ValueError(name)


def main():
    M, N, K = 512, 512, 1024
    rows = np.arange(0, M, M // 64)
    out = {"shape": [M, N, K], "rows_sampled": len(rows), "families": {}}
    for name in ("uniform", "normal", "in_zone", "stress_fp16_range", "wide_2^+-40"):
        A, B = fam(name, (M, K), 1), fam(name, (K, N), 2)
        Ad, Bd = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
        C64 = oracle.gemm64(A[rows], B)
        with np.errstate(all="ignore"):
            en = oracle.normwise_error(oracle.gemm32_naive(A[rows], B), A[rows], B, C64)
        res = {"naive_fp32": en}
        for fmt in (0, 1):
            for terms in (3, 4):
                egemm.set_config_ex(operand_format=fmt)
                try:
                    D = egemm.gemm(Ad, Bd, terms=terms).cpu().numpy()
                finally:
                    egemm.set_config_ex()
                with np.errstate(all="ignore"):
                    e = oracle.normwise_error(D[rows], A[rows], B, C64)
                res["%s_%dterms" % ("bf16" if fmt else "fp16", terms)] = e if np.isfinite(e) else "non-finite"
        try:
            D = torch.empty((M, N), device="cuda")
            bench._cublas_bf16x9_ms(Ad, Bd, D, reps=1)
            res["cublas_bf16x9"] = oracle.normwise_error(D.cpu().numpy()[rows], A[rows], B, C64)
        except Exception as ex:  # pragma: no cover
            res["cublas_bf16x9"] = "error: %s" % str(ex)[:80]
        out["families"][name] = res
        print(name, {k: (("%.2e" % v) if isinstance(v, float) else v) for k, v in res.items()}, flush=True)
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    json.dump(out, open(os.path.join(ROOT, "gpurun_out", "bf16_error_table.json"), "w"), indent=1)


if __name__ == "__main__":
    main()
