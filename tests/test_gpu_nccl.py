"""The NCCL / SymmetricMemory code paths of distributed.py on hardware, with the one GPU the
pool gives per box: a single torchrun rank with backend "nccl" (tests/nccl_worker.py).  The
collectives are identities on one rank, so the results must equal the collective-free
composition bitwise -- this checks the NCCL calls, dtypes and buffer handling, not the
multi-rank data plane (covered on CPU by the gloo tests, and with 2 ranks sharing a GPU over
gloo in test_gpu_distributed.py)."""
import os
import subprocess
import sys

import numpy as np
import pytest

from tests.gpu_util import require_gpu

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_single_rank_nccl_paths(tmp_path):
    require_gpu()
    out = str(tmp_path / "nccl.npz")
    env = dict(os.environ, MASTER_ADDR="127.0.0.1")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "1",
           "--master-addr", "127.0.0.1", "--master-port", "29671",
           os.path.join(ROOT, "tests", "nccl_worker.py"), out]
    r = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-3000:]
    d = dict(np.load(out))
    assert str(d["backend"][0]) == "nccl"
    assert bool(d["bcast_same"][0])
    assert np.array_equal(d["allreduce"], np.arange(10, dtype=np.float64))
    assert np.array_equal(d["km_assign1"], d["km_assign2"])
    assert np.array_equal(d["km_C1"].view(np.uint32), d["km_C2"].view(np.uint32))
    assert str(d["symm"][0]) == "ok", str(d["symm"][0])
    assert np.array_equal(d["km_assign1"], d["km_assign3"])
    assert np.array_equal(d["km_C1"].view(np.uint32), d["km_C3"].view(np.uint32))
