"""Tail split on single-wave buckets: for every finite tune-table bucket with K >= 4096 whose
pick fills at most half of the persistent clusters (tiles <= clusters / 2), time the pick
against the same tile config with tail_split = 1 (every tile of the partly filled single wave
becomes 2-4 k-parts with the in-kernel last-arriver fix-up; a split-K pick is compared with
its tile config unsplit + tail split), alternating rounds, and check the results against the
fp64 oracle on a row sample.  Writes a JSON list (argv[1]).  Tool code."""
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
from paper_conf_ppopp_fengwcz0d21_b200 import egemm, inputs  # noqa: E402
from tools.tune_sweep import timeit  # noqa: E402


def main(out):
    t = json.load(open(os.path.join(ROOT, "paper_conf_ppopp_fengwcz0d21_b200", "tune_table.json")))
    nsm = egemm.num_sms()
    res = []
    for e in t["entries"]:
        if e["op"] not in ("gemm", "gemm_b32") or max(e["m_max"], e["n_max"]) > 1 << 20:
            continue
        # (the open K bucket is represented by K = 8192, the sweep's grid point for it)
        M, N, K = e["m_max"], e["n_max"], min(e["k_max"], 8192)
        if K < 4096:
            continue
        ksp = e.get("ksplit", 0)
        cg, bn = e["cg"], e["bn"]
        tiles = -(-M // (128 * cg)) * -(-N // bn)
        if 2 * tiles > nsm // cg:
            continue
        A, B = inputs.uniform((M, K), 11 + M), inputs.uniform((K, N), 13 + N)
        Ad, Bd = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
        b32 = e["op"] == "gemm_b32"
        bs = None if b32 else egemm.split(Bd, transpose=True)
        D = torch.empty(M, N, device="cuda")
        ws = torch.empty(egemm.gemm_workspace_size(M, N, K, False, not b32) + (16 << 20), dtype=torch.uint8,
                         device="cuda")
        rs = np.arange(0, M, max(1, M // 32))
        C64 = oracle.gemm64(A[rs], B)
        en = oracle.normwise_error(oracle.gemm32_naive(A[rs], B), A[rs], B, C64)
        call = (lambda: egemm.gemm(Ad, Bd, out=D, workspace=ws)) if b32 else \
            (lambda: egemm.gemm(Ad, None, b_split=bs, out=D, workspace=ws))
        row = {"op": e["op"], "bucket": [e["m_max"], e["n_max"], e["k_max"]], "shape": [M, N, K], "cfg": [cg, bn, e["sep"], e["kc"], e.get("fa", 0)],
               "ksplit": ksp, "tiles": tiles}
        for rnd in range(3):
            for ts in (0, 1):
                kw = dict(cg=cg, bn=bn, sep=e["sep"], kc=e["kc"], fused=e.get("fa", 0), stages=e.get("stages", 0),
                          tail_split=ts)
                kw["ksplit"] = ksp if (ts == 0 and ksp > 1) else 1  # ts 0: the pick as it is
                egemm.set_config_ex(**kw)
                ms = timeit(call)
                call()
                torch.cuda.synchronize()
                err = oracle.normwise_error(D.cpu().numpy()[rs], A[rs], B, C64)
                row.setdefault("ms_ts%d" % ts, []).append(ms)
                row["err_ratio_ts%d" % ts] = err / en
        egemm.set_config_ex()
        row["speedup"] = float(np.median(row["ms_ts0"]) / np.median(row["ms_ts1"]))
        print(json.dumps(row), flush=True)
        res.append(row)
    json.dump(res, open(out, "w"), indent=1)


if __name__ == "__main__":
    main(sys.argv[1])
