"""(argv[2] = "gemm": the same for the pre-split rows, whose picks may be split-K already; plus
the pick's tile unsplit, ks1.)  Split-K (reduce pass) for the public fp32-B call: the gemm_b32 rows never had split-K
candidates (the sweep offered them only to the pre-split rows).  For every finite gemm_b32
bucket with K >= 1024 whose pick fills at most half of the clusters, time the table's pick
(tail split where the table sets it) against the pick's tile config with ksplit 2 and 4,
alternating rounds, with the oracle error on a row sample.  JSON list -> argv[1].  Tool code."""
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


def main(out, op="gemm_b32"):
    t = json.load(open(os.path.join(ROOT, "paper_conf_ppopp_fengwcz0d21_b200", "tune_table.json")))
    nsm = egemm.num_sms()
    res = []
    for e in t["entries"]:
        if e["op"] != op or max(e["m_max"], e["n_max"]) > 1 << 20 or e["k_max"] < 1024:
            continue
        M, N, K = e["m_max"], e["n_max"], min(e["k_max"], 8192)
        cg, bn = e["cg"], e["bn"]
        tiles = -(-M // (128 * cg)) * -(-N // bn)
        lo_t, hi_t = (int(v) for v in os.environ.get("TILES", "0,%d" % (nsm // cg // 2)).split(","))
        if not (lo_t < tiles <= hi_t) or e.get("fa", 0) == 2:
            continue
        if "MAXTILES" in os.environ and (tiles > int(os.environ["MAXTILES"]) or K < 2048):
            continue
        A, B = inputs.uniform((M, K), 11 + M), inputs.uniform((K, N), 13 + N)
        Ad, Bd = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
        bs = egemm.split(Bd, transpose=True) if op == "gemm" else None
        D = torch.empty(M, N, device="cuda")
        ws = torch.empty(egemm.gemm_workspace_size(M, N, K) + (64 << 20), dtype=torch.uint8, device="cuda")
        rs = np.arange(0, M, max(1, M // 32))
        C64 = oracle.gemm64(A[rs], B)
        en = oracle.normwise_error(oracle.gemm32_naive(A[rs], B), A[rs], B, C64)
        base = dict(cg=cg, bn=bn, sep=e["sep"], kc=e["kc"], fused=e.get("fa", 0), stages=e.get("stages", 0))
        kss = [int(v) for v in os.environ.get("KS", "2,4").split(",")]
        cands = {"pick": dict(base, tail_split=e.get("tsplit", 0), ksplit=max(1, e.get("ksplit", 0)))}
        if "KS" not in os.environ:
            cands["ks1"] = dict(base, fused=0, tail_split=0, ksplit=1)
        for v in kss:
            cands["ks%d" % v] = dict(base, fused=0, tail_split=0, ksplit=v)
        row = {"op": op, "bucket": [e["m_max"], e["n_max"], e["k_max"]], "shape": [M, N, K], "pick": base,
               "ksplit": e.get("ksplit", 0),
               "tsplit": e.get("tsplit", 0), "tiles": tiles}
        for rnd in range(3):
            for name, cfg in cands.items():
                egemm.set_config_ex(**cfg)
                call = (lambda: egemm.gemm(Ad, None, b_split=bs, out=D, workspace=ws)) if op == "gemm" else \
                    (lambda: egemm.gemm(Ad, Bd, out=D, workspace=ws))
                ms = timeit(call)
                call()
                torch.cuda.synchronize()
                err = oracle.normwise_error(D.cpu().numpy()[rs], A[rs], B, C64)
                row.setdefault("ms_" + name, []).append(ms)
                row["err_ratio_" + name] = err / en
        egemm.set_config_ex()
        print(json.dumps(row), flush=True)
        res.append(row)
    json.dump(res, open(out, "w"), indent=1)


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else "gemm_b32")
