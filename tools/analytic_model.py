"""NEXT-4: the paper's analytic model (Sec. 6, Eqs. 2-8) re-derived for
tcgen05 on B200 and used as a PRIOR for the measured tuning sweep.

The paper sizes (bm, bn, bk) so that T_Comp >= T_Mem1 + T_Mem2 (Eqs. 5-8) under register and
shared-memory budgets (Table 3) and maximises the intensity 2 bm bn / (bm + bn) (Eq. 4).  On
B200 the register file no longer holds C (TMEM does), the smem->FRAG step (Eq. 7) is gone
(MMAs read shared memory directly) and the GEMM is power-capped, so the model becomes:

  resource constraints (Eq. 8 analogue, checked for every implemented config):
    smem:  STAGES * 4 (BM_cta + BN_cta) * BK  <= 227 KiB       (hi + lo, fp16: Eq. 2's 4 B)
    TMEM:  accumulators * BN                   <= 512 columns  (2 ping-pong, x2 for SEP)
  time for an (M, N, K) problem:
    T_mma  = ceil(tiles / slots) * terms * 128 * BN * Kp / (4096 MAC/clk * eta * f)   (Eq. 3, 5)
             + chunks per tile * switch cost                   (promotion, measured ~160 clk)
    T_l2   = tiles * 4 (BM + BN) Kp / BW_L2                   (Eq. 2, 6: operand traffic)
    T_hbm  = (4 (M + N) Kp + 4 M N) / BW_HBM                  (compulsory bytes)
    T      = max(T_mma, T_conv, T_l2, T_hbm) + T_switch + T_split(A) + T_fixed
  with eta (the MMA-issue efficiency of each kernel family) and the fused-split converter
  rate CALIBRATED on the single 8192^3 bucket of the committed sweep log; f is the
  power-capped clock (1.2 GHz); BW_L2 is an assumption (no L2 microbenchmark in this repo).

`evaluate(log)` reports, for every bucket of a sweep log, the model's pick vs the measured
best (top-1 / top-3 hit rate and the regret = measured time of the model's pick / best),
restricted to configs that pass the accuracy bar -- i.e. how well the model would prune the
sweep.  Tool code (no GPU needed).

usage: python tools/analytic_model.py [profiles/r01_tune_sweep_log.json]
"""
import json
import math
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

N_SM = 148
MAC_PER_CLK = 4096            # fp16 dense MACs / clk / SM (2.25 PF nominal / 148 / ~1.85 GHz)
F_CLK = 1.2e9                 # power-capped SM clock under sustained tensor load (measured)
BW_HBM = 6454e9               # MEASURED_PEAKS.json copy bandwidth
BW_L2 = 16e12                 # L2 -> SM operand bandwidth (assumption)
SPLIT_EFF = 0.75              # split kernel fraction of HBM bandwidth (measured 0.69-0.78)
T_FIXED = 8e-6                # GEMM launch + pipeline fill + last epilogue (s)
T_LAUNCH = 3e-6               # one more kernel launch (the separate A split)
SWITCH_CLK = 160              # accumulator switch per promotion chunk (tools/diag_gemm.py)
SMEM_BUDGET = 227 * 1024
TMEM_COLS = 512
BK = 64


def geometry(cfg):
    cg, bn, sep, kc, fa = cfg
    bm_cta, bn_cta = 128, bn // cg
    stages = 3
    return {"BM": 128 * cg, "BN": bn, "slots": N_SM // cg, "stages": stages,
            "smem": stages * 4 * (bm_cta + bn_cta) * BK,
            "tmem": (4 if sep else 2) * bn}


def intensity(bm, bn):
    """Eq. 4: flops per byte of split operands, 2 bm bn / (bm + bn)."""
    return 2.0 * bm * bn / (bm + bn)


def feasible(cfg):
    g = geometry(cfg)
    return g["smem"] <= SMEM_BUDGET and g["tmem"] <= TMEM_COLS


def family(cfg):
    return tuple(cfg[:3]) + (cfg[4],)


def predict(cfg, M, N, K, eta, conv, terms=3):
    """Predicted seconds of egemm_gemm(A fp32, B pre-split) -- the sweep's timed call."""
    cg, bn, sep, kc, fa = cfg
    g = geometry(cfg)
    kp = math.ceil(K / BK) * BK
    tiles = math.ceil(M / g["BM"]) * math.ceil(N / bn)
    per_slot = math.ceil(tiles / g["slots"])
    chunks = math.ceil(kp / kc)
    t_mma = per_slot * terms * 128 * bn * kp / MAC_PER_CLK / eta[family(cfg)] / F_CLK
    t_switch = per_slot * chunks * SWITCH_CLK / F_CLK
    # fused split: the converter warpgroup's cycles per (row, k) element of A
    t_conv = per_slot * 128 * kp * conv[family(cfg)] / F_CLK if fa else 0.0
    t_l2 = tiles * 4.0 * (g["BM"] + bn) * kp / BW_L2
    t_hbm = (4.0 * (M + N) * kp + 4.0 * M * N) / BW_HBM
    t_split = 0.0 if fa else 8.0 * M * K / (BW_HBM * SPLIT_EFF) + T_LAUNCH
    return max(t_mma, t_conv, t_l2, t_hbm) + t_switch + t_split + T_FIXED


def calibrate(log, at=(8192, 8192, 8192)):
    """eta per kernel family (pre-split) and the converter cycles per A element (fused
    families) from the one calibration bucket."""
    b = next(x for x in log if (x["M"], x["N"], x["K"]) == at)
    M, N, K = at
    eta, conv = {}, {}
    kp = math.ceil(K / BK) * BK
    for r in sorted(b["results"], key=lambda r: r["cfg"][4]):  # pre-split families first
        cfg = tuple(r["cfg"])
        fam = family(cfg)
        g = geometry(cfg)
        tiles = math.ceil(M / g["BM"]) * math.ceil(N / cfg[1])
        per_slot = math.ceil(tiles / g["slots"])
        chunks = math.ceil(kp / cfg[3])
        split = 0.0 if cfg[4] else 8.0 * M * K / (BW_HBM * SPLIT_EFF) + T_LAUNCH
        t = r["ms"] * 1e-3 - T_FIXED - split - per_slot * chunks * SWITCH_CLK / F_CLK
        mma_cyc = 3 * 128 * cfg[1] * kp / MAC_PER_CLK
        if not cfg[4]:
            eta[fam] = max(eta.get(fam, 0.0), per_slot * mma_cyc / (t * F_CLK))
        else:
            eta[fam] = eta.get(fam[:3] + (0,), 1.0)
            c = t * F_CLK / (per_slot * 128 * kp)
            conv[fam] = min(conv.get(fam, c), c)
    return eta, conv


def evaluate(log, eta=None, conv=None):
    if eta is None:
        eta, conv = calibrate(log)
    rows, hit1, hit3, regrets = [], 0, 0, []
    for b in log:
        M, N, K = b["M"], b["N"], b["K"]
        ok = [r for r in b["results"] if r["ok"]]
        if not ok:
            continue
        best = min(ok, key=lambda r: r["ms"])
        pred = sorted(ok, key=lambda r: predict(tuple(r["cfg"]), M, N, K, eta, conv))
        top3 = [tuple(r["cfg"]) for r in pred[:3]]
        h1 = tuple(pred[0]["cfg"]) == tuple(best["cfg"])
        h3 = tuple(best["cfg"]) in top3
        regret = pred[0]["ms"] / best["ms"]
        regret3 = min(r["ms"] for r in pred[:3]) / best["ms"]
        hit1 += h1
        hit3 += h3
        regrets.append((regret, regret3))
        rows.append({"M": M, "N": N, "K": K, "best": best["cfg"], "model": pred[0]["cfg"],
                     "model_top3": top3, "regret_top1": round(regret, 3),
                     "regret_top3": round(regret3, 3),
                     "pred_ms_best": round(predict(tuple(best["cfg"]), M, N, K, eta, conv) * 1e3, 4),
                     "meas_ms_best": round(best["ms"], 4)})
    n = len(rows)
    return {"buckets": n, "top1_hit": hit1 / n, "top3_hit": hit3 / n,
            "median_regret_top1": sorted(r[0] for r in regrets)[n // 2],
            "max_regret_top1": max(r[0] for r in regrets),
            "max_regret_top3": max(r[1] for r in regrets),
            "eta": {"%s" % (k,): round(v, 3) for k, v in eta.items()},
            "conv_clk_per_row_k": {"%s" % (k,): round(v, 4) for k, v in conv.items()},
            "rows": rows}


def main():
    path = sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "profiles",
                                                               "r01_tune_sweep_log.json")
    log = json.load(open(path))
    res = evaluate(log)
    out = os.path.join(ROOT, "profiles", "analytic_model_eval.json")
    json.dump(res, open(out, "w"), indent=1)
    print("buckets %d  top-1 hit %.2f  top-3 hit %.2f  median regret %.3f  max regret top-1 %.3f "
          "top-3 %.3f" % (res["buckets"], res["top1_hit"], res["top3_hit"],
                          res["median_regret_top1"], res["max_regret_top1"],
                          res["max_regret_top3"]))
    print("eta", res["eta"])
    print("wrote", out)


if __name__ == "__main__":
    main()
