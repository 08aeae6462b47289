"""kMeans configs[4] (4M points, d=64, 1024 centroids, 20 Lloyd iterations as bench.py runs
them) with the point tile resident in smem (a_resident=1) vs streamed with every centroid
tile (0), alternating, plus the in-kernel clock; optionally with 8 / 16 epilogue warps.
    python tools/kmeans_ar_ab.py
Tool code."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_fengwcz0d21_b200 import distributed as edist  # noqa: E402
from paper_conf_ppopp_fengwcz0d21_b200 import egemm, inputs  # noqa: E402


def main():
    n, d, kc, iters = 1 << 22, 64, 1024, 20
    Xh, _, _ = inputs.mixture(n, d, kc, 400)
    X = torch.from_numpy(Xh).cuda()
    C0 = torch.from_numpy(Xh[:kc].copy()).cuda()
    del Xh
    x_split = egemm.split(X)
    ws = torch.empty(egemm.kmeans_workspace_size(n, d, kc, True), dtype=torch.uint8, device="cuda")
    bufs = (torch.empty(n, dtype=torch.int32, device="cuda"),
            torch.empty((kc, d), dtype=torch.float64, device="cuda"),
            torch.empty(kc, dtype=torch.int64, device="cuda"), None)
    C = C0.clone()
    res = {}
    for trial in range(6):
        for ar, epi in ([(0, 16), (1, 16), (1, 8)] if trial % 2 == 0 else [(1, 8), (1, 16), (0, 16)]):
            egemm.set_config_ex(a_resident=ar, epi_warps=epi)
            try:
                C.copy_(C0)
                edist.kmeans_fit(X, C, 2, x_split=x_split, workspace=ws, bufs=bufs, world=1)
                C.copy_(C0)
                egemm.debug_clock_stats(reset=True)
                s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                s.record()
                edist.kmeans_fit(X, C, iters, x_split=x_split, workspace=ws, bufs=bufs, world=1)
                e.record()
                e.synchronize()
                mhz, cyc, _ = egemm.debug_clock_stats(reset=True)
                res.setdefault("ar%d_e%d" % (ar, epi), []).append((s.elapsed_time(e) / iters, mhz, cyc))
            finally:
                egemm.set_config_ex()
    out = {}
    for k, v in res.items():
        v = sorted(v)
        out[k] = {"ms_per_iter_median": round(v[len(v) // 2][0], 4), "ms_min": round(v[0][0], 4),
                  "mhz_mean": round(sum(x[1] for x in v) / len(v), 0),
                  "gemm_cycles_min": round(min(x[2] for x in v), 0)}
    print(json.dumps(out, indent=1))
    with open(os.path.join("gpurun_out", "kmeans_ar_ab.json"), "w") as f:
        json.dump(out, f, indent=1)


if __name__ == "__main__":
    main()
