"""NEXT-3: the paper's tensor-core precision profiling (Sec. 3.1) run on every
floating tcgen05 kind through egemm_tc_probe (kind::f16 with fp16 or bf16 operands,
kind::tf32), and the candidate accumulation models of oracle.tc_model fitted to the bits.

For each kind, designed input families go through ONE MMA chain on the GPU; every candidate
(exact-sum RN / RZ, and "align": terms truncated onto the grid 2^(E-23-x) below the largest
exponent estimate E, x = 0..4 extra bits, E from exponent fields or from values) is applied
MMA by MMA on the CPU and compared bitwise on a sample of outputs.  For tf32 the operand
conversion is probed too (fp32 inputs with non-zero low mantissa bits).  Writes
profiles/tc_profile_kinds.json.  Tool code (calls oracle/ for the models).

usage: python tools/probe_kinds.py [samples_per_family]
"""
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
from paper_conf_ppopp_fengwcz0d21_b200 import egemm  # noqa: E402

KSTEP = {"f16": 16, "bf16": 16, "tf32": 8}
TDT = {"f16": torch.float16, "bf16": torch.bfloat16, "tf32": torch.float32}
CANDIDATES = [("rn", 0, "fields"), ("rz", 0, "fields")] + \
    [("align", x, a) for a in ("fields", "value") for x in range(0, 5)]


def to_kind(x, kind, mode="rz"):
    """fp32/fp64 array -> values exactly representable in the kind's operand type."""
    t = torch.from_numpy(np.asarray(x, np.float32))
    if kind == "tf32":  # keep 10 mantissa bits: truncate (or round) the low 13 bits
        u = t.view(torch.int32)
        if mode == "rn":
            u = u + 0x0FFF + ((u >> 13) & 1)
        return (u & ~0x1FFF).view(torch.float32).numpy()
    return t.to(TDT[kind]).float().numpy()


def families(kind, g, N, K):
    ks = KSTEP[kind]
    tiny = {"f16": -24, "bf16": -133, "tf32": -126}[kind]
    fam = {}
    fam["one_mma_uniform"] = (g.uniform(-1, 1, (128, ks)), g.uniform(-1, 1, (N, ks)), None)
    A = np.zeros((128, ks))
    B = np.zeros((N, ks))
    A[:, 0] = g.uniform(1, 2, 128)
    A[:, 1] = g.uniform(1, 2, 128) * np.exp2(-g.integers(0, 40, 128)) * np.where(g.random(128) < .5, -1, 1)
    B[:, 0] = g.uniform(1, 2, N)
    B[:, 1] = g.uniform(1, 2, N)
    fam["two_products_ratio"] = (A, B, None)
    C = g.uniform(-4, 4, (128, N)).astype(np.float32)
    fam["c_plus_small"] = (g.uniform(-1, 1, (128, ks)) * np.exp2(-g.integers(0, 20, (128, 1))),
                           g.uniform(-1, 1, (N, ks)), C)
    fam["chain_K"] = (g.uniform(-1, 1, (128, K)), g.uniform(-1, 1, (N, K)), None)
    A = g.uniform(-1, 1, (128, ks))
    B = g.uniform(-1, 1, (N, ks))
    B[:, 1] = B[:, 0]
    A[:, 1] = -A[:, 0] * (1 + np.exp2(-g.integers(5, 12, (128,))))  # near-cancellation
    fam["cancellation"] = (A, B, None)
    fam["wide_exponents"] = (g.uniform(1, 2, (128, ks)) * np.exp2(g.integers(-12, 12, (128, ks))),
                             g.uniform(-2, 2, (N, ks)) * np.exp2(g.integers(-12, 12, (N, ks))), None)
    fam["tiny"] = (g.uniform(1, 2, (128, ks)) * np.exp2(g.integers(tiny // 2, tiny // 2 + 6, (128, ks))),
                   g.uniform(-2, 2, (N, ks)) * np.exp2(g.integers(tiny // 2, tiny // 2 + 6, (N, ks))),
                   None)
    return fam


def model_chain(a_row, b_row, c, ks, model, x, anchor):
    """The candidate applied MMA by MMA (each MMA consumes ks products + the accumulator)."""
    acc = 0.0 if c is None else float(c)
    for k0 in range(0, len(a_row), ks):
        acc = oracle.tc_model(a_row[k0:k0 + ks], b_row[k0:k0 + ks], acc, model, x, anchor)
    return acc


def run_kind(kind, g, N=64, samples=256):
    K = {"f16": 64, "bf16": 64, "tf32": 32}[kind]
    out = {}
    for name, (A, B, C) in families(kind, g, N, K).items():
        Aq, Bq = to_kind(A, kind), to_kind(B, kind)
        At = torch.from_numpy(Aq).cuda().to(TDT[kind])
        Bt = torch.from_numpy(Bq).cuda().to(TDT[kind])
        Ct = torch.from_numpy(C).cuda() if C is not None else None
        D = egemm.tc_probe(kind, At, Bt, Ct).cpu().numpy()
        idx = [(int(i), int(j)) for i, j in zip(g.integers(0, 128, samples), g.integers(0, N, samples))]
        res = {}
        for (model, x, anchor) in CANDIDATES:
            ok = 0
            for i, j in idx:
                m = model_chain(Aq[i].astype(np.float64), Bq[j].astype(np.float64),
                                None if C is None else C[i, j], KSTEP[kind], model, x, anchor)
                ok += (np.float32(m).view(np.uint32) == np.float32(D[i, j]).view(np.uint32))
            res["%s/%d/%s" % (model, x, anchor)] = ok / len(idx)
        out[name] = res
        print(kind, name, max(res.items(), key=lambda kv: kv[1]), flush=True)
    return out


def tf32_conversion(g, N=64):
    """fp32 operands with low mantissa bits: does kind::tf32 truncate or round them?"""
    A = g.uniform(-1, 1, (128, 8)).astype(np.float32)
    B = np.zeros((N, 8), np.float32)
    B[:, 0] = 1.0  # D[i, j] = A[i, 0] * 1 exactly -> reveals the converted A[i, 0]
    D = egemm.tc_probe("tf32", torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()).cpu().numpy()
    got = D[:, 0]
    rz, rn = to_kind(A[:, 0], "tf32", "rz"), to_kind(A[:, 0], "tf32", "rn")
    return {"matches_truncation": float(np.mean(got == rz)), "matches_rne": float(np.mean(got == rn)),
            "matches_fp32_unconverted": float(np.mean(got == A[:, 0]))}


def main():
    samples = int(sys.argv[1]) if len(sys.argv) > 1 else 256
    g = np.random.default_rng(2024)
    res = {"what": "tcgen05 precision profile per kind (Sec. 3.1 workflow): fraction of sampled "
                   "outputs bitwise equal to each candidate model, per input family",
           "candidates": ["%s/%d/%s" % c for c in CANDIDATES], "kinds": {}}
    for kind in ("f16", "bf16", "tf32"):
        fam = run_kind(kind, g, samples=samples)
        total = {c: float(np.mean([f[c] for f in fam.values()])) for c in res["candidates"]}
        best = max(total.items(), key=lambda kv: kv[1])
        res["kinds"][kind] = {"families": fam, "mean_over_families": total, "best": best}
        print("==", kind, "best", best, flush=True)
    res["tf32_operand_conversion"] = tf32_conversion(g)
    print("tf32 conversion", res["tf32_operand_conversion"])
    os.makedirs(os.path.join(ROOT, "profiles"), exist_ok=True)
    json.dump(res, open(os.path.join(ROOT, "profiles", "tc_profile_kinds.json"), "w"), indent=1)


if __name__ == "__main__":
    main()
