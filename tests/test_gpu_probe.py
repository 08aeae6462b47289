"""NEXT-3: egemm_tc_probe (one tcgen05.mma chain per kind) -- layout / descriptor correctness
on exactly representable problems for every kind, and the f16 kind against the profiled
accumulation model that the GEMM is bitwise-pinned to."""
import numpy as np
import pytest
import torch

import oracle
from paper_conf_ppopp_fengwcz0d21_b200 import inputs
from tests.gpu_util import require_gpu

pytestmark = pytest.mark.gpu

TDT = {"f16": torch.float16, "bf16": torch.bfloat16, "tf32": torch.float32}


@pytest.mark.parametrize("kind", ["f16", "bf16", "tf32"])
@pytest.mark.parametrize("N,K,with_c", [(16, 8, False), (64, 37, True), (256, 128, True)])
def test_probe_exact_integer_problems(kind, N, K, with_c):
    """Small integers: every partial sum is exact in fp32, so D = C + A B^T exactly under any
    accumulation model -- pins the probe's swizzled staging, descriptors, K tail and C load."""
    eg = require_gpu()
    g = inputs.rng(1000 + N + K)
    A = g.integers(-8, 9, (128, K)).astype(np.float32)
    B = g.integers(-8, 9, (N, K)).astype(np.float32)
    C = g.integers(-1000, 1000, (128, N)).astype(np.float32) if with_c else None
    D = eg.tc_probe(kind, torch.from_numpy(A).cuda().to(TDT[kind]),
                    torch.from_numpy(B).cuda().to(TDT[kind]),
                    None if C is None else torch.from_numpy(C).cuda()).cpu().numpy()
    ref = A.astype(np.float64) @ B.T.astype(np.float64) + (0 if C is None else C)
    assert np.array_equal(D.astype(np.float64), ref)


KSTEP = {"f16": 16, "bf16": 16, "tf32": 8}
NPDT = {"f16": np.float16, "bf16": None, "tf32": None}


def _quant(x, kind):
    t = torch.from_numpy(np.asarray(x, np.float32))
    if kind == "tf32":
        return (t.view(torch.int32) & ~0x1FFF).view(torch.float32).numpy()
    return t.to(TDT[kind]).float().numpy()


@pytest.mark.parametrize("kind", ["f16", "bf16", "tf32"])
def test_probe_matches_profiled_model(kind):
    """Every floating kind's MMA chain is bitwise oracle.tc_model('align', 2, 'fields') MMA by
    MMA (tools/probe_kinds.py measured 100 % over 7 input families per kind,
    profiles/tc_profile_kinds.json); for f16 this is the model DESIGN.md §6 found through the
    GEMM kernel, here seen through a different kernel."""
    eg = require_gpu()
    g = inputs.rng(77)
    ks = KSTEP[kind]
    K = 3 * ks
    A = _quant(g.uniform(-1, 1, (128, K)), kind)
    B = _quant(g.uniform(-1, 1, (64, K)) * np.exp2(g.integers(-8, 8, (64, K))), kind)
    C = g.uniform(-2, 2, (128, 64)).astype(np.float32)
    D = eg.tc_probe(kind, torch.from_numpy(A).cuda().to(TDT[kind]),
                    torch.from_numpy(B).cuda().to(TDT[kind]), torch.from_numpy(C).cuda()).cpu().numpy()
    for i, j in zip(g.integers(0, 128, 64), g.integers(0, 64, 64)):
        acc = float(C[i, j])
        for k0 in range(0, K, ks):
            acc = oracle.tc_model(A[i, k0:k0 + ks].astype(np.float64),
                                  B[j, k0:k0 + ks].astype(np.float64), acc, "align", 2, "fields")
        assert np.float32(acc).view(np.uint32) == D[i, j].view(np.uint32), (kind, i, j)


def test_probe_tf32_operands_are_truncated():
    """kind::tf32 reads an fp32 operand by dropping its 13 low mantissa bits (RZ), not RNE."""
    eg = require_gpu()
    g = inputs.rng(78)
    A = g.uniform(-1, 1, (128, 8)).astype(np.float32)
    B = np.zeros((16, 8), np.float32)
    B[:, 0] = 1.0
    D = eg.tc_probe("tf32", torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()).cpu().numpy()
    assert np.array_equal(D[:, 0], _quant(A[:, 0], "tf32"))
    assert not np.array_equal(D[:, 0], A[:, 0])
