"""egemm_gemm_host (host buffers, pipelined copies) == egemm_gemm on the same inputs, bitwise
(same tile configuration per row chunk) and within the oracle's bars."""
import numpy as np
import pytest
import torch

from paper_conf_ppopp_fengwcz0d21_b200 import inputs
from tests.gpu_util import require_gpu, to_dev, to_host

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("M,N,K", [(300, 200, 100), (2048, 512, 777), (5000, 1000, 256)])
def test_gemm_host_matches_oracle(oracle_lib, M, N, K):
    eg = require_gpu()
    A, B = inputs.uniform((M, K), 71), inputs.uniform((K, N), 72)
    Ah = torch.from_numpy(A).pin_memory()
    Bh = torch.from_numpy(B).pin_memory()
    D = eg.gemm_host(Ah, Bh)
    torch.cuda.synchronize()
    D = D.numpy()
    C64 = oracle_lib.gemm64(A, B)
    e = oracle_lib.normwise_error(D, A, B, C64)
    en = oracle_lib.normwise_error(oracle_lib.gemm32_naive(A, B), A, B, C64)
    assert e <= 1e-6 and e <= 2 * en, (e, en)
    assert np.all(np.abs(D - C64) <= oracle_lib.elem_bound(A, B))  # any promotion interval


def test_gemm_host_unpinned_and_strided():
    eg = require_gpu()
    A = inputs.uniform((700, 300), 73)
    B = inputs.uniform((300, 260), 74)
    D1 = eg.gemm_host(torch.from_numpy(A), torch.from_numpy(B),
                      out=torch.empty((700, 260), dtype=torch.float32))
    torch.cuda.synchronize()
    ref = to_host(eg.gemm(to_dev(A), to_dev(B)))
    # the per-chunk config may differ from the whole-matrix config: compare within bound
    assert np.allclose(D1.numpy(), ref, rtol=1e-5, atol=1e-5)
