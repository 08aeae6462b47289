"""Single-wave GEMMs (public call, fp32 A and B, CUDA-graph replay): tail split on / off (with
a single partly filled wave every tile becomes k-parts), over tile configs.  Tool code."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_fengwcz0d21_b200 import egemm, inputs  # noqa: E402
from tools.tune_sweep import timeit  # noqa: E402


def main():
    cases = [((1024, 1024, 1024), [(2, 128, 0, 64, 0), (2, 128, 0, 128, 0), (2, 256, 0, 64, 0), (1, 128, 0, 64, 0)]),
             ((1024, 1024, 4096), [(2, 128, 0, 128, 0), (2, 256, 0, 128, 0)]),
             ((1024, 1024, 8192), [(2, 128, 0, 256, 0), (2, 256, 0, 256, 0)]),
             ((512, 2048, 2048), [(2, 128, 0, 128, 0), (2, 256, 0, 128, 0)]),
             ((256, 1024, 1024), [(2, 128, 0, 64, 0), (1, 128, 0, 64, 0)]),
             ((2048, 1024, 2048), [(2, 256, 0, 128, 0), (2, 128, 0, 128, 0)])]
    for (M, N, K), cfgs in cases:
        A = torch.from_numpy(inputs.uniform((M, K), 1)).cuda()
        B = torch.from_numpy(inputs.uniform((K, N), 2)).cuda()
        D = torch.empty(M, N, device="cuda")
        ws = torch.empty(egemm.gemm_workspace_size(M, N, K) + (64 << 20), dtype=torch.uint8, device="cuda")
        print("table pick", (M, N, K), egemm.query_config_ex("gemm_b32", M, N, K), flush=True)
        for cg, bn, sep, kc, fz in cfgs:
            for ts in (0, 1):
                egemm.set_config_ex(cg=cg, bn=bn, sep=sep, kc=kc, fused=fz, tail_split=ts)
                try:
                    ms = timeit(lambda: egemm.gemm(A, B, out=D, workspace=ws))
                except Exception as ex:
                    print((M, N, K), (cg, bn, sep, kc, fz), "ts", ts, "n/a", str(ex)[:80])
                    continue
                print("%s cfg %s ts=%d  %.4f ms  %.1f TF/s" % ((M, N, K), (cg, bn, sep, kc, fz), ts, ms,
                                                           2.0 * M * N * K / ms / 1e9), flush=True)
        egemm.set_config_ex()


if __name__ == "__main__":
    main()
