"""The multi-rank bench path (torchrun, row-sharded C, max-over-ranks timing, rank 0 prints
one JSON line) on a single GPU: EGEMM_BENCH_SHARE_GPU=1 puts every rank on cuda:0 and uses
gloo for the collectives (the real 2/4/8-GPU runs use NCCL, one GPU per rank)."""
import json
import os
import subprocess
import sys

import pytest

from tests.gpu_util import require_gpu

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.parametrize("world,n,apps", [(2, 2048, False), (4, 4096, False), (2, 4096, True)])
def test_bench_multirank_shared_gpu(world, n, apps):
    require_gpu()
    env = dict(os.environ, EGEMM_BENCH_SHARE_GPU="1", MASTER_ADDR="127.0.0.1")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", str(world),
           "--master-addr", "127.0.0.1", "--master-port", str(29611 + world + (7 if apps else 0)),
           os.path.join(ROOT, "bench.py"), "--gpus", str(world), "--steps", "3", "--warmup", "3",
           "--no-cpu", "--size", str(n)] + ([] if apps else ["--no-apps"])
    out = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=900)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = [ln for ln in out.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, out.stdout[-2000:]  # rank 0 alone prints
    d = json.loads(lines[0])
    assert d["n_gpus"] == world and d["value"] > 0 and d["scaling"] == "strong"
    assert d["config"]["rows_per_rank"] == n // world
    assert d["gpu_launches"] > 0
    if apps:
        assert d["knn"]["value"] > 0 and d["kmeans"]["value"] > 0
