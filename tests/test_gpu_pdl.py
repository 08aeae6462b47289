"""Stream-order safety of the programmatic dependent launches (split.cu PDL hooks, the
tensor-core kernel's griddepcontrol.wait): back-to-back calls on one stream with no host
synchronisation must give bitwise the results of the same calls separated by
synchronisations -- a GEMM reading the previous GEMM's D (read after write), a GEMM
overwriting the operand the previous one read (write after read), a GEMM after a torch
kernel, and the in-call chain split(A) -> split(B^T) (PDL follower) -> GEMM.  Any missing
wait shows up as stale or torn operands."""
import numpy as np
import pytest
import torch

from paper_conf_ppopp_fengwcz0d21_b200 import inputs
from tests.gpu_util import require_gpu, to_dev

pytestmark = pytest.mark.gpu


def _eq(a, b):
    a, b = a.cpu().numpy(), b.cpu().numpy()
    return np.array_equal(a.view(np.uint32), b.view(np.uint32)), int((a != b).sum())


@pytest.mark.parametrize("fused", [0, 1])
@pytest.mark.parametrize("shape", [(1024, 1024, 1024), (2048, 512, 512)])
def test_chain_read_after_write(fused, shape):
    """X_{i+1} = X_i @ B (B scaled to keep |X| bounded), 8 calls back to back vs synchronised."""
    eg = require_gpu()
    M, N, K = shape  # N == K: the chain multiplies by the same square B
    B = to_dev((inputs.uniform((K, N), 7) * np.float32(1.0 / np.sqrt(K))).astype(np.float32))
    X0 = to_dev(inputs.uniform((M, K), 8))
    eg.set_config_ex(fused=fused)
    try:
        xs = [X0]
        for _ in range(8):  # no host synchronisation inside the chain
            xs.append(eg.gemm(xs[-1], B))
        torch.cuda.synchronize()
        x = X0
        for i in range(8):
            torch.cuda.synchronize()
            y = eg.gemm(x, B)
            torch.cuda.synchronize()
            ok, bad = _eq(xs[i + 1], y)
            assert ok, "step %d: %d mismatches" % (i, bad)
            x = y
    finally:
        eg.set_config_ex()


def test_write_after_read_and_torch_predecessor():
    """D = A @ B, then A is overwritten by a torch kernel and used again; then the GEMM's
    output buffer is the next GEMM's input while a third GEMM overwrites the first's D."""
    eg = require_gpu()
    M, N, K = 2048, 1024, 1024
    A = to_dev(inputs.uniform((M, K), 11))
    A2 = to_dev(inputs.uniform((M, K), 12))
    B = to_dev(inputs.uniform((K, N), 13))
    ref1 = eg.gemm(A.clone(), B)
    ref2 = eg.gemm(A2.clone(), B)
    torch.cuda.synchronize()
    for _ in range(5):
        D1 = torch.empty(M, N, device="cuda")
        Ab = A.clone()
        eg.gemm(Ab, B, out=D1)   # reads Ab
        Ab.copy_(A2)             # torch kernel overwrites it (WAR against the GEMM above)
        D2 = eg.gemm(Ab, B)      # GEMM after a torch kernel (RAW)
        eg.gemm(Ab, B, out=D1)   # overwrites D1 right after ... (WAW)
        torch.cuda.synchronize()
        ok, bad = _eq(D2, ref2)
        assert ok, bad
        ok, bad = _eq(D1, ref2)
        assert ok, bad
    ok, bad = _eq(eg.gemm(A, B), ref1)
    assert ok, bad


@pytest.mark.parametrize("cfg", [(2, 128, 0, 64), (2, 256, 0, 128), (1, 128, 0, 64)])
def test_in_call_split_chain(cfg, oracle_lib):
    """fp32 A and B with pre-split operands forced: split(A), then split(B^T) as A's PDL
    follower, then the GEMM (waiting on both) -- equal to the Alg. 1 model bitwise, over
    back-to-back calls on fresh inputs."""
    eg = require_gpu()
    M, N, K = 1000, 700, 900
    outs, refs = [], []
    eg.set_config_ex(cg=cfg[0], bn=cfg[1], sep=cfg[2], kc=cfg[3], fused=0)
    try:
        for s in range(4):
            An, Bn = inputs.uniform((M, K), 40 + s), inputs.uniform((K, N), 50 + s)
            outs.append(eg.gemm(to_dev(An), to_dev(Bn)))
            refs.append((An, Bn))
        torch.cuda.synchronize()
    finally:
        eg.set_config_ex()
    for D, (An, Bn) in zip(outs, refs):
        ref = oracle_lib.gemm_alg1_tc(An, Bn, terms=3, sep=cfg[2], kc=cfg[3])
        d = D.cpu().numpy()
        assert np.array_equal(d.view(np.uint32), ref.view(np.uint32)), int((d != ref).sum())
