"""Per-kernel device time of the kMeans (configs[4]) and kNN (configs[3]) steps, live (not
serialised like an ncu launch list): torch.profiler's CUDA activity records around a few
back-to-back steps.  Tool code (diagnostics)."""
import os
import sys
from collections import defaultdict

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_fengwcz0d21_b200 import egemm, inputs  # noqa: E402


def profile(f, reps, tag):
    for _ in range(3):
        f()
    torch.cuda.synchronize()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    for _ in range(reps):
        f()
    e.record()
    e.synchronize()
    wall = s.elapsed_time(e) / reps
    with torch.profiler.profile(activities=[torch.profiler.ProfilerActivity.CUDA]) as prof:
        for _ in range(reps):
            f()
        torch.cuda.synchronize()
    acc = defaultdict(float)
    for ev in prof.events():
        if ev.device_type == torch.autograd.DeviceType.CUDA:
            acc[ev.name[:90]] += ev.device_time / 1e3 / reps
    print("== %s: %.3f ms per step (events, unprofiled)" % (tag, wall))
    tot = 0.0
    for k, v in sorted(acc.items(), key=lambda x: -x[1]):
        print("  %8.4f ms  %s" % (v, k))
        tot += v
    print("  %8.4f ms  (sum)" % tot, flush=True)


def main():
    which = sys.argv[1] if len(sys.argv) > 1 else "both"
    if which in ("kmeans", "both"):
        n, d, kc = 1 << 22, 64, 1024
        Xh, _, _ = inputs.mixture(n, d, kc, 400)
        X = torch.from_numpy(Xh).cuda()
        C = torch.from_numpy(Xh[:kc].copy()).cuda()
        xs = egemm.split(X)
        ws = torch.empty(egemm.kmeans_workspace_size(n, d, kc, True), dtype=torch.uint8,
                         device="cuda")
        out = (torch.empty(n, dtype=torch.int32, device="cuda"),
               torch.empty((kc, d), dtype=torch.float64, device="cuda"),
               torch.empty(kc, dtype=torch.int64, device="cuda"), None)
        profile(lambda: egemm.kmeans_step(X, C, x_split=xs, want_inertia=False, workspace=ws,
                                          out=out), 20, "kmeans step 4M x 1024 x 64")
    if which in ("knn", "both"):
        nx, nq = 1 << 20, 1 << 16
        Xk = torch.from_numpy(inputs.uniform((nx, 128), 300)).cuda()
        Qk = torch.from_numpy(inputs.uniform((nq, 128), 301)).cuda()
        index = egemm.knn_index(Xk)
        profile(lambda: egemm.knn(None, Qk, 16, index=index), 3, "knn 1M x 64K d=128 k=16")


if __name__ == "__main__":
    main()
