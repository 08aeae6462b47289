"""The bench's reference arm (the CPU oracle timed on a bounded block of the workload) runs
on the host alone and prints one JSON line; its per-step budget shrinks with the step count,
so a driver run of any K stays within minutes."""
import json
import os
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_reference_arm_prints_one_bounded_line():
    t0 = time.time()
    # a short per-step budget keeps this CPU test to seconds; the driver's default run keeps
    # the whole --steps K --warmup W run within ~150 s of oracle work (bench.reference_arm)
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference",
                          "--steps", "12", "--warmup", "3", "--size", "2048", "--ref-step-s", "0.3"],
                         cwd=ROOT, capture_output=True, text=True, timeout=600)
    wall = time.time() - t0
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [ln for ln in out.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["impl"] == "reference" and d["value"] > 0 and d["steps"] == 12
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0
    assert wall < 120, wall  # ~5 s of oracle work, plus start-up and calibration
