"""Collect tensor-core (tcgen05 kind::f16) accumulation data for the precision profiling of
Sec. 3.1: fp16-exact inputs through egemm_gemm (lo = 0, so every MMA's hh
accumulator sees plain fp16 products), D dumped to gpurun_out/probe.npz for offline model
fitting against oracle.tc_model.  Test/tool code."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_fengwcz0d21_b200 import egemm, inputs  # noqa: E402


def f16(x):
    return x.astype(np.float16).astype(np.float32)


def main(out="gpurun_out/probe.npz"):
    g = inputs.rng(1234)
    M = N = 128
    sets = {}
    # S1: one MMA, 16 random products, C = 0
    sets["s1"] = (f16(g.uniform(-1, 1, (M, 16))), f16(g.uniform(-1, 1, (16, N))))
    # S2: one MMA, two products with a magnitude ratio 2^-r, random signs
    A = np.zeros((M, 16), np.float32)
    B = np.zeros((16, N), np.float32)
    A[:, 0] = f16(g.uniform(1, 2, M))
    A[:, 1] = f16(g.uniform(1, 2, M) * np.exp2(-g.integers(0, 30, M)) * np.where(g.random(M) < .5, -1, 1))
    B[0, :] = f16(g.uniform(1, 2, N))
    B[1, :] = f16(g.uniform(1, 2, N))
    sets["s2"] = (A, B)
    # S3: two MMAs: C = one large product, then 16 random small products
    A = np.zeros((M, 32), np.float32)
    B = np.zeros((32, N), np.float32)
    A[:, 0] = f16(g.uniform(-2, 2, M))
    B[0, :] = f16(g.uniform(-2, 2, N))
    A[:, 16:] = f16(g.uniform(-1, 1, (M, 16)) * np.exp2(-g.integers(0, 14, (M, 1))))
    B[16:, :] = f16(g.uniform(-1, 1, (16, N)))
    sets["s3"] = (A, B)
    # S4: two MMAs, random, second half scaled 2^-6
    A = f16(g.uniform(-1, 1, (M, 32)))
    A[:, 16:] = f16(A[:, 16:] * 2.0 ** -6)
    sets["s4"] = (A, f16(g.uniform(-1, 1, (32, N))))
    # S5: one MMA, all-positive products
    sets["s5"] = (f16(g.uniform(0, 1, (M, 16))), f16(g.uniform(0, 1, (16, N))))
    # S6: 8 products only (k 0..7) vs 8 in k 8..15 of different scale
    A = f16(g.uniform(-1, 1, (M, 16)))
    A[:, 8:] = f16(A[:, 8:] * np.exp2(-g.integers(0, 12, (M, 1))))
    sets["s6"] = (A, f16(g.uniform(-1, 1, (16, N))))
    # S7: single product + C where the product sits far below C's ulp (K=32)
    A = np.zeros((M, 32), np.float32)
    B = np.zeros((32, N), np.float32)
    A[:, 0] = f16(g.uniform(1, 2, M))
    B[0, :] = 1.0
    A[:, 16] = f16(g.uniform(1, 2, M) * np.exp2(-g.integers(10, 30, M)) * np.where(g.random(M) < .5, -1, 1))
    B[16, :] = f16(g.uniform(1, 2, N))
    sets["s7"] = (A, B)
    # S8: subnormal fp16 operands (what the lo parts of |x| < 2^-3 become) mixed with normals
    sub = lambda shape: (g.integers(1, 1024, shape) * 2.0 ** -24 * np.where(g.random(shape) < .5, -1, 1))
    A = f16(g.uniform(-1, 1, (M, 32)))
    A[:, :8] = f16(sub((M, 8)))
    A[:, 16:28] = f16(sub((M, 12)))
    B = f16(g.uniform(-1, 1, (32, N)))
    B[4:12, :] = f16(sub((8, N)) * 2.0 ** 10)
    sets["s8"] = (A, B)
    # S9: all-subnormal A against normal B, with C from a first MMA of normals
    A = f16(sub((M, 32)))
    A[:, :16] = f16(g.uniform(-2.0 ** -10, 2.0 ** -10, (M, 16)))
    sets["s9"] = (A, f16(g.uniform(-1, 1, (32, N))))
    res = {}
    egemm.set_config(1, 128, 1, 1024)
    for name, (A, B) in sets.items():
        D = egemm.gemm(torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda())
        torch.cuda.synchronize()
        res[name + "_A"] = A
        res[name + "_B"] = B
        res[name + "_D"] = D.cpu().numpy()
    egemm.set_config(0, 0, 0, 0)
    os.makedirs(os.path.dirname(out), exist_ok=True)
    np.savez_compressed(out, **res)
    print("probe data ->", out)


if __name__ == "__main__":
    main(*sys.argv[1:])
