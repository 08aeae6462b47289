"""SURVEY §4 item 3 on one GPU: the sharded compositions of distributed.py (row-sharded GEMM,
query-sharded kNN, reference-sharded kNN with egemm_knn_merge, point-sharded kMeans with one
all_reduce per iteration) run by 2 ranks (torchrun, every rank on cuda:0, gloo collectives)
against the single-process library calls on the same seeded inputs.
  * GEMM with the tile / Kc / k-parts pinned: bitwise equal (the per-element k order does not
    depend on which rows a rank owns);
  * kNN (both shardings): bitwise equal indices and distances;
  * kMeans: the all_reduced sums are the per-rank sums added in another fp64 order, so the
    centroids agree to a few ulps and the assignments of this well-separated mixture agree."""
import os
import subprocess
import sys

import numpy as np
import pytest
import torch

from tests import dist_worker as W
from tests.gpu_util import require_gpu, to_dev, to_host

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def sharded(tmp_path_factory):
    require_gpu()
    out = str(tmp_path_factory.mktemp("dist") / "res.npz")
    env = dict(os.environ, MASTER_ADDR="127.0.0.1")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", "29655",
           os.path.join(ROOT, "tests", "dist_worker.py"), out]
    r = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stderr[-3000:]
    return dict(np.load(out))


def test_row_sharded_gemm_bitwise(sharded):
    eg = require_gpu()
    A, B = W.gemm_inputs()
    eg.set_config_ex(**W.CFG)
    try:
        D = to_host(eg.gemm(to_dev(A), to_dev(B)))
    finally:
        eg.set_config_ex()
    assert np.array_equal(sharded["gemm"].view(np.uint32), D.view(np.uint32))


def test_query_and_reference_sharded_knn_bitwise(sharded):
    eg = require_gpu()
    X, Q = W.knn_inputs()
    idx, dist = eg.knn(to_dev(X), to_dev(Q), W.KNN[3])
    idx, dist = to_host(idx).astype(np.int64), to_host(dist)
    for key in ("knn", "knn_ref"):
        assert np.array_equal(sharded[key + "_idx"].astype(np.int64), idx), key
        assert np.array_equal(sharded[key + "_dist"].view(np.uint32), dist.view(np.uint32)), key


def test_point_sharded_kmeans(sharded):
    require_gpu()
    from paper_conf_ppopp_fengwcz0d21_b200 import distributed as edist
    Xk, C0 = W.kmeans_inputs()
    C = torch.from_numpy(C0).cuda()
    a = to_host(edist.kmeans_fit(to_dev(Xk), C, W.KMEANS[3], world=1))
    Cs = sharded["kmeans_C"]
    assert np.mean(sharded["kmeans_assign"] == a) >= 0.999
    assert np.all(np.abs(Cs.astype(np.float64) - to_host(C)) <= 4 * np.spacing(np.abs(to_host(C))) + 1e-30)
