"""Tail split A/B: the public fp32-in GEMM call with the library's table configuration, tail
split off vs on (egemm_config_t.tail_split), steady-state time per call and the in-kernel
clock / CTA-0 cycles, on the shapes whose persistent grid ends in a partly filled wave
(configs[2] tall-skinny, the 2- / 4- / 8-rank row shards of configs[1], Fig. 9 shapes).
    python tools/tail_split_ab.py [--reps 5]
Tool code."""
import argparse
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from paper_conf_ppopp_fengwcz0d21_b200 import egemm, inputs  # noqa: E402
from tune_sweep import timeit  # noqa: E402

SHAPES = [(65536, 256, 1024), (2048, 8192, 8192), (4096, 4096, 8192), (4096, 4096, 4096),
          (16384, 4096, 4096), (8192, 2048, 2048), (16384, 16384, 16384), (1024, 8192, 8192)]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--out", default=None)
    ap.add_argument("--short", type=int, default=0,
                    help="also time windows of this many back-to-back calls (the bench's tall-skinny "
                         "window is 20), alternating off / on, 7 trials, median")
    args = ap.parse_args()
    rows = []
    for (M, N, K) in SHAPES:
        A = torch.from_numpy(inputs.uniform((M, K), 200)).cuda()
        B = torch.from_numpy(inputs.uniform((K, N), 201)).cuda()
        ws = torch.empty(egemm.gemm_workspace_size(M, N, K), dtype=torch.uint8, device="cuda")
        D = torch.empty((M, N), device="cuda")
        res = {}
        for rnd in range(2):
            for ts in ((0, 1) if rnd == 0 else (1, 0)):
                egemm.set_config_ex(tail_split=ts)
                try:
                    egemm.debug_clock_stats(reset=True)
                    t = timeit(lambda: egemm.gemm(A, B, out=D, workspace=ws), reps=args.reps)
                    mhz, cyc, n = egemm.debug_clock_stats(reset=True)
                    cfg = egemm.query_config_ex("gemm_b32", M, N, K)
                finally:
                    egemm.set_config_ex()
                res.setdefault(ts, []).append((t, mhz, cyc))
        r = {"shape": [M, N, K], "cfg": {k: cfg[k] for k in ("cg", "bn", "kc", "fused", "ksplit")}}
        for ts in (0, 1):
            t = min(x[0] for x in res[ts])
            r["ms_ts%d" % ts] = round(t, 5)
            r["tflops_ts%d" % ts] = round(2.0 * M * N * K / t / 1e9, 1)
            r["mhz_ts%d" % ts] = round(sum(x[1] for x in res[ts]) / len(res[ts]), 0)
            r["cycles_ts%d" % ts] = round(min(x[2] for x in res[ts]), 0)
        r["speedup"] = round(r["ms_ts0"] / r["ms_ts1"], 4)
        if args.short:
            sh = {0: [], 1: []}
            for trial in range(7):
                for ts in ((0, 1) if trial % 2 == 0 else (1, 0)):
                    egemm.set_config_ex(tail_split=ts)
                    try:
                        for _ in range(3):
                            egemm.gemm(A, B, out=D, workspace=ws)
                        s0, e0 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                        s0.record()
                        for _ in range(args.short):
                            egemm.gemm(A, B, out=D, workspace=ws)
                        e0.record()
                        e0.synchronize()
                        sh[ts].append(s0.elapsed_time(e0) / args.short)
                    finally:
                        egemm.set_config_ex()
            for ts in (0, 1):
                r["short_ms_ts%d" % ts] = round(sorted(sh[ts])[len(sh[ts]) // 2], 5)
            r["short_speedup"] = round(r["short_ms_ts0"] / r["short_ms_ts1"], 4)
        rows.append(r)
        print(json.dumps(r), flush=True)
        del A, B, ws, D
        torch.cuda.empty_cache()
    if args.out:
        with open(args.out, "w") as f:
            json.dump(rows, f, indent=1)


if __name__ == "__main__":
    main()
