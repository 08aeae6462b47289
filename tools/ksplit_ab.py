"""Split-K buckets of the tuning table: the table's pick (now with the in-kernel last-arriver
fix-up -- the experiment this tool was written for; the product keeps the reduce pass) vs the same tile without split-K, steady state
(CUDA-graph replay below 0.2 ms, tune_sweep.timeit), and vs the time the sweep recorded
with the reduce pass ("ms" in the table).  Also a few square / per-rank shapes with every
split-K count, to see whether the fix-up makes split-K win where the reduce pass did not.
    python tools/ksplit_ab.py [--out gpurun_out/ksplit_ab.json]
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


def run(M, N, K, b_f32, cfg):
    A = torch.from_numpy(inputs.uniform((M, K), 1)).cuda()
    B = torch.from_numpy(inputs.uniform((K, N), 2)).cuda()
    bs = None if b_f32 else egemm.split(B, transpose=True)
    D = torch.empty((M, N), device="cuda")
    egemm.set_config_ex(**cfg)
    try:
        ws = torch.empty(egemm.gemm_workspace_size(M, N, K, False, not b_f32), dtype=torch.uint8, device="cuda")
        if b_f32:
            t = timeit(lambda: egemm.gemm(A, B, out=D, workspace=ws), reps=3)
        else:
            t = timeit(lambda: egemm.gemm(A, None, b_split=bs, out=D, workspace=ws), reps=3)
    finally:
        egemm.set_config_ex()
    return t


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    tab = json.load(open(os.path.join(ROOT, "paper_conf_ppopp_fengwcz0d21_b200", "tune_table.json")))
    rows = []
    for e in tab["entries"]:
        if e.get("op") not in ("gemm", "gemm_b32") or e.get("ksplit", 0) <= 1:
            continue
        M, N, K = (min(e["m_max"], 65536), min(e["n_max"], 8192), min(e["k_max"], 8192))
        base = dict(cg=e["cg"], bn=e["bn"], sep=e["sep"], kc=e["kc"], fused=e["fa"], stages=e["stages"])
        b32 = e["op"] == "gemm_b32"
        t_k = run(M, N, K, b32, dict(base, ksplit=e["ksplit"]))
        t_1 = run(M, N, K, b32, dict(base, ksplit=1))
        r = {"op": e["op"], "shape": [M, N, K], "ksplit": e["ksplit"], "ms_table_reduce_pass": e["ms"],
             "ms_fixup": round(t_k, 5), "ms_no_split": round(t_1, 5)}
        rows.append(r)
        print(json.dumps(r), flush=True)
    for (M, N, K) in ((1024, 1024, 1024), (1024, 8192, 8192), (2048, 2048, 2048), (1024, 2048, 8192)):
        q = egemm.query_config_ex("gemm", M, N, K)
        base = dict(cg=q["cg"], bn=q["bn"], sep=q["sep"], kc=q["kc"], fused=q["fused"], stages=q["stages"])
        r = {"op": "gemm", "shape": [M, N, K], "table": [q["cg"], q["bn"], q["kc"], q["ksplit"]]}
        for ks in (1, 2, 3, 4, 6, 8):
            r["ms_ksplit%d" % ks] = round(run(M, N, K, False, dict(base, ksplit=ks)), 5)
        rows.append(r)
        print(json.dumps(r), flush=True)
    if args.out:
        json.dump(rows, open(args.out, "w"), indent=1)


if __name__ == "__main__":
    main()
