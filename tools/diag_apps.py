"""kNN / kMeans tensor-core kernel diagnostics: cycles per launch and mean clock (in-kernel
probe) with and without the fused epilogue work (EGEMM_DEBUG_NO_EPI) and operand loads
(EGEMM_DEBUG_NO_TMA).  Tool code."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_fengwcz0d21_b200 import egemm, inputs  # noqa: E402


def measure(f, reps):
    for _ in range(2):
        f()
    torch.cuda.synchronize()
    egemm.debug_clock_stats(reset=True)
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    for _ in range(reps):
        f()
    e.record()
    e.synchronize()
    mhz, cyc, nl = egemm.debug_clock_stats(reset=True)
    return s.elapsed_time(e) / reps, mhz, cyc, nl / reps


def main():
    n, d, kc = 1 << 22, 64, 1024
    Xh, _, _ = inputs.mixture(n, d, kc, 400)
    X = torch.from_numpy(Xh).cuda()
    C = torch.from_numpy(Xh[:kc].copy()).cuda()
    xs = egemm.split(X)
    ws = torch.empty(egemm.kmeans_workspace_size(n, d, kc, True), dtype=torch.uint8, device="cuda")
    need_km = 6.0 * n * kc * d / (148 * 8192.0)
    nx, nq = 1 << 20, int(os.environ.get("DIAG_NQ", 1 << 14))
    only_knn = os.environ.get("DIAG_ONLY_KNN") == "1"
    Xk = torch.from_numpy(inputs.uniform((nx, 128), 300)).cuda()
    Qk = torch.from_numpy(inputs.uniform((nq, 128), 301)).cuda()
    index = egemm.knn_index(Xk)
    need_knn = 6.0 * nq * nx * 128 / (148 * 8192.0)
    for tag, env in (("full", {}), ("no_candidates", {"EGEMM_DEBUG_MODE": "128"}),
                     ("tmem_ld_only", {"EGEMM_DEBUG_MODE": "64"}),
                     ("no_epi", {"EGEMM_DEBUG_NO_EPI": "1"}),
                     ("no_tma+no_epi", {"EGEMM_DEBUG_NO_EPI": "1", "EGEMM_DEBUG_NO_TMA": "1"})):
        for k in ("EGEMM_DEBUG_NO_EPI", "EGEMM_DEBUG_NO_TMA", "EGEMM_DEBUG_MODE"):
            os.environ.pop(k, None)
        os.environ.update(env)
        if not only_knn:
            ms, mhz, cyc, lpc = measure(lambda: egemm.kmeans_step(X, C, x_split=xs, want_inertia=False,
                                                                  workspace=ws), 20)
            print("kmeans %-14s step %.3f ms  tc kernel %.0f kcyc (%.3f ms at %.0f MHz)  eff %.3f"
                  % (tag, ms, cyc / 1e3, cyc / mhz / 1e3, mhz, need_km / cyc), flush=True)
        ms, mhz, cyc, lpc = measure(lambda: egemm.knn(None, Qk, 16, index=index), 5)
        print("knn    %-14s call %.3f ms  tc kernel %.0f kcyc (%.3f ms at %.0f MHz)  eff %.3f  launches %.1f"
              % (tag, ms, cyc / 1e3, cyc / mhz / 1e3, mhz, need_knn / cyc, lpc), flush=True)


if __name__ == "__main__":
    main()
