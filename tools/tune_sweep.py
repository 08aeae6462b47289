"""Measured tile / promotion table -> paper_conf_ppopp_fengwcz0d21_b200/tune_table.json.

Replaces the paper's analytic model (Sec. 6, Eqs. 2-8) by measurement: for each
(op, shape bucket) every configuration the library implements is timed (CUDA events, median
of repeats, pre-split operands) and its normwise error vs the fp64 oracle is measured on a
row sample; the fastest configuration that meets the accuracy bar (<= 1e-6 and <= 2x the
naive-fp32 error, BJ north_star) is recorded.  Tool code (calls oracle/ for the error check).

usage: python tools/tune_sweep.py [--quick] [--prior T] [--out table.json]
       python tools/tune_sweep.py --from-log log.json [--keep old_table.json --margin 0.03]
                                  [--meta new_table.json]
"""
import json
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import oracle  # noqa: E402
from paper_conf_ppopp_fengwcz0d21_b200 import egemm, inputs  # noqa: E402

OUT = os.path.join(ROOT, "paper_conf_ppopp_fengwcz0d21_b200", "tune_table.json")
# (cg, bn, sep, kc, fa): fa = the fused in-kernel A split (converter warpgroup)
# Kc = 256 with one accumulator only passes the accuracy bar at large K (the per-chunk
# truncation error grows ~Kc / sqrt(K), tools/error_sweep.py): the bar decides per bucket.
CONFIGS = [(2, 256, 0, 64, 0), (2, 256, 0, 128, 0), (2, 256, 0, 256, 0), (2, 128, 1, 128, 0),
           (2, 128, 1, 256, 0), (1, 128, 1, 128, 0), (1, 128, 1, 256, 0), (1, 128, 0, 64, 0),
           (2, 256, 0, 64, 1), (2, 256, 0, 128, 1), (2, 256, 0, 256, 1), (2, 128, 1, 256, 1),
           (1, 128, 1, 256, 1), (2, 224, 0, 64, 0), (2, 224, 0, 128, 0), (2, 224, 0, 256, 0),
           (2, 128, 0, 64, 0), (2, 128, 0, 128, 0)]


def timeit(fn, reps=3, batch_ms=60.0):
    """Steady-state time per call: warm up ~batch_ms, then the median of `reps` batches of
    back-to-back calls, each ~batch_ms long (the power-capped clock settles within tens
    of ms; single short launches over-report the fast, cool-clock case)."""
    fn()
    torch.cuda.synchronize()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    fn()
    e.record()
    e.synchronize()
    n = max(1, int(batch_ms / max(s.elapsed_time(e), 1e-3)))
    for _ in range(n):
        fn()
    ts = []
    for _ in range(reps):
        s.record()
        for _ in range(n):
            fn()
        e.record()
        e.synchronize()
        ts.append(s.elapsed_time(e) / n)
    return float(np.median(ts))


def gemm_bucket(M, N, K, rows=64, configs=None):
    A, B = inputs.uniform((M, K), 11 + M), inputs.uniform((K, N), 13 + N)
    Ad, Bd = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
    b_split = egemm.split(Bd, transpose=True)
    D = torch.empty((M, N), device="cuda")
    rs = np.sort(inputs.rng(M + N + K).choice(M, size=min(rows, M), replace=False))
    C64 = oracle.gemm64(A[rs], B)
    en = oracle.normwise_error(oracle.gemm32_naive(A[rs], B), A[rs], B, C64)
    ws = torch.empty(egemm.gemm_workspace_size(M, N, K, False, True), dtype=torch.uint8, device="cuda")
    res = []
    for cfg in configs or CONFIGS:
        egemm.set_config(*cfg[:4])
        os.environ["EGEMM_FUSED_A"] = str(cfg[4])
        # the user call with an fp32 A (split separately, or fused into the GEMM) and a
        # pre-split B: the A split is part of every timed call
        t = timeit(lambda: egemm.gemm(Ad, None, b_split=b_split, out=D, workspace=ws))
        e = oracle.normwise_error(D.cpu().numpy()[rs], A[rs], B, C64)
        res.append({"cfg": cfg, "ms": t, "err": e, "err_naive": en,
                    "ok": bool(e <= 1e-6 and e <= 2 * en)})
    egemm.set_config(0, 0, 0, 0)
    os.environ.pop("EGEMM_FUSED_A", None)
    return res


RULE = ("fastest config whose normwise error, scaled to the bucket's smallest K, is <= 1e-6 "
        "and <= 1x the naive-fp32 error (extended precision: at least as accurate as SGEMM, "
        "P:63, Fig. 7) when any config reaches it, else the north-star bar (<= 2x naive); "
        "64 sampled rows, steady-state timing")


def select(res, k_scale=1.0):
    """The bucket's pick under RULE (None when nothing meets the north-star bar).  The
    bucket covers K in (K_prev, K]; the single-accumulator error ratio grows ~ Kc / sqrt(K)
    (tools/error_sweep.py), so the ratio measured at K is scaled by k_scale = sqrt(K / K_prev)
    to bound it over the whole bucket."""
    ok = [r for r in res if r["ok"] and r["err"] * k_scale <= 2 * r["err_naive"]]
    strict = [r for r in ok if r["err"] * k_scale <= r["err_naive"]]
    pool = strict or ok
    return min(pool, key=lambda r: r["ms"]) if pool else None


def k_scale(K, Ks):
    lower = max([k for k in Ks if k < K], default=None)
    return (K / lower) ** 0.5 if lower else 1.0


def build_table(log, Ms, Ns, Ks, extra=None, keep=None, margin=0.0):
    """keep: {(M, N, K): cfg} of a previous table -- its pick stays unless this sweep's best
    is more than `margin` faster than the previous pick re-measured in the same sweep (the
    power-capped clock drifts between consecutive configs by a few %: near-ties are noise)."""
    entries = []
    for b in log:
        M, N, K = b["M"], b["N"], b["K"]
        best = select(b["results"], k_scale(K, Ks))
        prev = (keep or {}).get((M, N, K))
        if best and prev and list(best["cfg"]) != list(prev):
            again = [r for r in b["results"] if list(r["cfg"]) == list(prev)]
            if again and again[0]["ok"] and again[0]["ms"] * (1.0 - margin) <= best["ms"]:
                best = again[0]
        if best:
            cg, bn, sep, kc, fa = best["cfg"]
            entries.append({"op": "gemm", "m_max": M, "n_max": N, "k_max": K, "cg": cg,
                            "bn": bn, "sep": sep, "kc": kc, "fa": fa,
                            "ms": round(best["ms"], 4),
                            "tflops_fp32eq": round(2.0 * M * N * K / best["ms"] / 1e9, 1),
                            "err_ratio": round(best["err"] / best["err_naive"], 3)})
    # the largest measured bucket in each dimension is open-ended, then bucket order:
    # smallest first so the library's first-match lookup picks the tightest bucket
    # M > 8192 is only swept for skinny N (<= 1024): the M = 8192 rows of wider N also
    # cover every larger M
    wide_top = max([M for M in Ms if M <= 8192], default=None)
    for e in entries:
        if e["m_max"] == wide_top and e["n_max"] > 1024:
            e["m_max"] = max(Ms)
        for key, top in (("m_max", max(Ms)), ("n_max", max(Ns)), ("k_max", max(Ks))):
            if e[key] == top:
                e[key] = 1 << 40
    entries.sort(key=lambda e: (e["m_max"], e["n_max"], e["k_max"]))
    doc = {"generated_by": "tools/tune_sweep.py", "rule": RULE, "entries": entries}
    doc.update(extra or {})
    return doc


B32_RULE = ("op gemm_b32 (B arrives as fp32: its round-split is part of the call): the fastest of "
            "the gemm row's pick (B split by egemm_split) and the fused-B kernels (2, 256, 0, Kc, "
            "fa=2) under the same accuracy rule")


def b32_sweep(Ms, Ns, Ks):
    """Buckets of the fp32-B user call gemm(A, B): the library's op-0 pick (separate B^T
    split inside the call) against the fused-B kernel at Kc 64 / 128 / 256."""
    log = []
    for M in Ms:
        for N in Ns:
            for K in Ks:
                if M > 8192 and N > 1024:
                    continue
                pick = list(egemm.query_config("gemm", M, N, K, with_fused=True))
                cfgs = [tuple(pick)] + [(2, 256, 0, kc, 2) for kc in (64, 128, 256)] + \
                    [(2, 224, 0, kc, 2) for kc in (128, 256)]
                A, B = inputs.uniform((M, K), 11 + M), inputs.uniform((K, N), 13 + N)
                Ad, Bd = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
                D = torch.empty((M, N), device="cuda")
                rs = np.sort(inputs.rng(M + N + K).choice(M, size=min(64, M), replace=False))
                C64 = oracle.gemm64(A[rs], B)
                en = oracle.normwise_error(oracle.gemm32_naive(A[rs], B), A[rs], B, C64)
                ws = torch.empty(egemm.gemm_workspace_size(M, N, K, False, False), dtype=torch.uint8,
                                 device="cuda")
                res = []
                for cfg in cfgs:
                    egemm.set_config(*cfg[:4])
                    os.environ["EGEMM_FUSED_A"] = str(cfg[4])
                    t = timeit(lambda: egemm.gemm(Ad, Bd, out=D, workspace=ws))
                    e = oracle.normwise_error(D.cpu().numpy()[rs], A[rs], B, C64)
                    res.append({"cfg": list(cfg), "ms": t, "err": e, "err_naive": en,
                                "ok": bool(e <= 1e-6 and e <= 2 * en)})
                egemm.set_config(0, 0, 0, 0)
                os.environ.pop("EGEMM_FUSED_A", None)
                best = select(res, k_scale(K, Ks))
                log.append({"M": M, "N": N, "K": K, "results": res})
                print("b32 M=%5d N=%5d K=%5d best=%s %s" % (M, N, K, best and best["cfg"],
                      " ".join("%s:%.3fms%s" % (r["cfg"], r["ms"], "" if r["ok"] else "x") for r in res)),
                      flush=True)
                del Ad, Bd, D, ws
    return log


def main():
    if "--b32" in sys.argv:  # add the fp32-B rows (op gemm_b32) to the current table
        Ms, Ns, Ks = [128, 256, 1024, 2048, 4096, 8192, 65536], [256, 1024, 8192], [256, 1024, 2048, 4096, 8192]
        if "--from-log" in sys.argv:
            log = json.load(open(sys.argv[sys.argv.index("--from-log") + 1]))
        else:
            log = b32_sweep(Ms, Ns, Ks)
            os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
            json.dump(log, open(os.path.join(ROOT, "gpurun_out", "tune_sweep_b32_log.json"), "w"), indent=1)
        doc = build_table(log, Ms, Ns, Ks)
        for e in doc["entries"]:
            e["op"] = "gemm_b32"
        table = json.load(open(OUT))
        table["entries"] = [e for e in table["entries"] if e["op"] != "gemm_b32"] + doc["entries"]
        table["rule_gemm_b32"] = B32_RULE
        out = sys.argv[sys.argv.index("--out") + 1] if "--out" in sys.argv else OUT
        json.dump(table, open(out, "w"), indent=1)
        print("wrote", out, len(doc["entries"]), "gemm_b32 entries")
        return
    if "--from-log" in sys.argv:  # re-derive the table from a committed sweep log
        log = json.load(open(sys.argv[sys.argv.index("--from-log") + 1]))
        Ms, Ns, Ks = (sorted({b[k] for b in log}) for k in ("M", "N", "K"))
        old = json.load(open(OUT))
        keep, margin = None, 0.0
        if "--keep" in sys.argv:  # hysteresis against a previous table (see build_table)
            prev = json.load(open(sys.argv[sys.argv.index("--keep") + 1]))
            margin = float(sys.argv[sys.argv.index("--margin") + 1]) if "--margin" in sys.argv else 0.03
            keep = {}
            for e in prev["entries"]:
                cfg = [e["cg"], e["bn"], e["sep"], e["kc"], e.get("fa", 0)]
                m = min([v for v in Ms if v >= e["m_max"]], default=max(Ms))
                n = min([v for v in Ns if v >= e["n_max"]], default=max(Ns))
                k = min([v for v in Ks if v >= e["k_max"]], default=max(Ks))
                if e["m_max"] > max(Ms) and n > 1024:  # wide N: the M = 8192 row covers larger M
                    m = max([v for v in Ms if v <= 8192])
                keep.setdefault((m, n, k), cfg)
        src = sys.argv[sys.argv.index("--meta") + 1] if "--meta" in sys.argv else OUT
        meta = json.load(open(src))
        doc = build_table(log, Ms, Ns, Ks, {k: meta[k] for k in ("device", "when", "sweep_seconds")
                                            if k in meta}, keep, margin)
        json.dump(doc, open(OUT, "w"), indent=1)
        print("rebuilt", OUT, len(doc["entries"]), "entries")
        return
    quick = "--quick" in sys.argv
    # 2048: the per-rank rows of the 4-GPU row-sharded 8192^3 bench (1024: 8 GPUs)
    Ms = [128, 256, 1024, 2048, 4096, 8192, 65536] if not quick else [128, 1024, 8192]
    Ns = [256, 1024, 8192] if not quick else [256, 8192]
    Ks = [256, 1024, 2048, 4096, 8192] if not quick else [1024, 8192]
    log = []
    t0 = time.time()
    # --prior T: measure every config only on the 8192^3 calibration bucket, then only the
    # analytic model's top T per bucket (NEXT-4; tools/analytic_model.py), widening to all
    # configs when none of those meets the accuracy bar
    prior = int(sys.argv[sys.argv.index("--prior") + 1]) if "--prior" in sys.argv else 0
    model = None
    if prior:
        import analytic_model as am
        cal = {"M": 8192, "N": 8192, "K": 8192, "results": gemm_bucket(8192, 8192, 8192)}
        model = am.calibrate([cal])
    for M in Ms:
        for N in Ns:
            for K in Ks:
                if M > 8192 and N > 1024:  # the tall bucket is for skinny N (configs[2])
                    continue
                if model and (M, N, K) == (8192, 8192, 8192):
                    res = cal["results"]
                elif model:
                    ranked = sorted(CONFIGS, key=lambda c: am.predict(c, M, N, K, *model))
                    res = gemm_bucket(M, N, K, configs=ranked[:prior])
                    if not any(r["ok"] for r in res):
                        res += gemm_bucket(M, N, K, configs=ranked[prior:])
                else:
                    res = gemm_bucket(M, N, K)
                best = select(res, k_scale(K, Ks))
                log.append({"M": M, "N": N, "K": K, "results": res})
                print("M=%5d N=%5d K=%5d best=%s %s" % (M, N, K, best and best["cfg"],
                      " ".join("%s:%.3fms%s" % (r["cfg"], r["ms"], "" if r["ok"] else "x") for r in res)),
                      flush=True)
    doc = build_table(log, Ms, Ns, Ks, {
        "device": torch.cuda.get_device_name(),
        "when": time.strftime("%Y-%m-%dT%H:%M:%SZ", time.gmtime()),
        "sweep_seconds": round(time.time() - t0, 1)})
    out = sys.argv[sys.argv.index("--out") + 1] if "--out" in sys.argv else OUT
    json.dump(doc, open(out, "w"), indent=1)
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    logname = "tune_sweep_prior%d_log.json" % prior if prior else "tune_sweep_log.json"
    json.dump(log, open(os.path.join(ROOT, "gpurun_out", logname), "w"), indent=1)
    print("wrote", out, len(doc["entries"]), "entries in %.1f s" % doc["sweep_seconds"])


if __name__ == "__main__":
    main()
