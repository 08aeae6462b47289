import sys, os, time, torch
sys.path.insert(0, os.getcwd())
from paper_conf_ppopp_fengwcz0d21_b200 import egemm
for n in (8192, 16384, 12288):
    A = torch.rand(n, n, device="cuda") * 2 - 1
    B = torch.rand(n, n, device="cuda") * 2 - 1
    a_s, b_s = egemm.split(A), egemm.split(B, transpose=True)
    D = torch.empty(n, n, device="cuda")
    need = 6.0 * n ** 3 / (148 * 8192.0)
    ws = torch.empty(egemm.gemm_workspace_size(n, n, n, True, True), dtype=torch.uint8, device="cuda")
    for cfg, pace in (((2, 256, 0, 256), 1), ((2, 256, 0, 256), 0), ((2, 256, 0, 256), 1)):
        if pace:
            os.environ.pop("EGEMM_NO_PACE", None)
        else:
            os.environ["EGEMM_NO_PACE"] = "1"
        egemm.set_config(*cfg)
        f = lambda: egemm.gemm(None, None, a_split=a_s, b_split=b_s, out=D, workspace=ws)
        for _ in range(3): f()
        torch.cuda.synchronize()
        egemm.debug_clock_stats(reset=True)
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        it = max(5, int(1500 / (6.0 * n ** 3 / 1.3e12)))
        s.record()
        for _ in range(it): f()
        e.record(); e.synchronize()
        ms = s.elapsed_time(e) / it
        mhz, cyc, nl = egemm.debug_clock_stats(reset=True)
        print(n, cfg, "paced" if pace else "free ", "%.3f ms %.0f TF-fp16 %.0f MHz cycle-eff %.3f" % (ms, 6.0 * n ** 3 / ms / 1e9, mhz, need / cyc), flush=True)
    del A, B, a_s, b_s, D
    torch.cuda.empty_cache()
