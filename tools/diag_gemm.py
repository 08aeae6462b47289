"""Where does the GEMM kernel lose MMA-pipe time?  Runs the 8192^3 pre-split GEMM under
diagnostic switches (EGEMM_DEBUG_NO_TMA: no operand loads; EGEMM_DEBUG_NO_EPI: no promotion
TMEM reads) and chunk sizes, each with the in-kernel SM-clock probe, and cuBLAS fp16 at the
same size with nvidia-smi clocks sampled during a long loop.  Tool code (diagnostics only).

usage: python tools/diag_gemm.py [n]
"""
import os
import subprocess
import sys
import threading

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_fengwcz0d21_b200 import egemm  # noqa: E402


def timeit(fn, iters=20, warm=5):
    for _ in range(warm):
        fn()
    torch.cuda.synchronize()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    for _ in range(iters):
        fn()
    e.record()
    e.synchronize()
    return s.elapsed_time(e) / iters


def smi_clock_during(fn, seconds=2.0):
    samples, stop = [], threading.Event()

    def poll():
        while not stop.is_set():
            try:
                o = subprocess.run(["nvidia-smi", "--query-gpu=clocks.sm,power.draw",
                                    "--format=csv,noheader,nounits", "-i", "0"],
                                   capture_output=True, text=True, timeout=5).stdout
                a, b = o.strip().split(",")
                samples.append((float(a), float(b)))
            except Exception:
                pass
            stop.wait(0.05)

    t = threading.Thread(target=poll)
    t.start()
    import time
    t0 = time.time()
    n = 0
    while time.time() - t0 < seconds:
        fn()
        n += 1
        if n % 10 == 0:
            torch.cuda.synchronize()
    torch.cuda.synchronize()
    stop.set()
    t.join()
    samples = samples[len(samples) // 4:]
    if not samples:
        return None, None
    mh = sorted(s[0] for s in samples)[len(samples) // 2]
    pw = sorted(s[1] for s in samples)[len(samples) // 2]
    return mh, pw


_spin = None


def spin_mhz(fn, ms=1500.0):
    """SM clock (MHz) seen by a 1-warp spin kernel co-resident with fn() looping for ms."""
    global _spin
    import ctypes
    import time
    if _spin is None:
        so = os.path.join("gpurun_out", "clockspin.so")
        src = os.path.join(os.path.dirname(os.path.abspath(__file__)), "csrc", "clockspin.cu")
        subprocess.run(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O2", "-shared",
                        "-Xcompiler", "-fPIC", "-o", so, src], check=True)
        _spin = ctypes.CDLL(os.path.abspath(so))
        _spin.clockspin_launch.argtypes = [ctypes.c_double, ctypes.c_void_p]
        _spin.clockspin_read.argtypes = [ctypes.POINTER(ctypes.c_double)]
    # both on non-default streams: the legacy default stream would serialise them
    side, work = torch.cuda.Stream(), torch.cuda.Stream()
    with torch.cuda.stream(work):
        for _ in range(3):
            fn()
        torch.cuda.synchronize()
        _spin.clockspin_launch(ms, ctypes.c_void_p(side.cuda_stream))
        t0, it = time.time(), 0
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        while time.time() - t0 < ms / 1e3 - 0.2:
            for _ in range(5):
                fn()
            it += 5
            work.synchronize()
        e.record()
        e.synchronize()
    torch.cuda.synchronize()
    v = ctypes.c_double(0.0)
    _spin.clockspin_read(ctypes.byref(v))
    return v.value, s.elapsed_time(e) / it


def main():
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
    A = torch.rand(n, n, device="cuda") * 2 - 1
    B = torch.rand(n, n, device="cuda") * 2 - 1
    a_s, b_s = egemm.split(A), egemm.split(B, transpose=True)
    D = torch.empty(n, n, device="cuda")
    fl3 = 3 * 2.0 * n ** 3

    need = fl3 / (148 * 8192.0)  # SM cycles of pure MMA issue per launch at the dense peak

    def run(tag, cfg, env, seconds=1.5):
        for k in ("EGEMM_DEBUG_NO_TMA", "EGEMM_DEBUG_NO_EPI", "EGEMM_DEBUG_MODE"):
            os.environ.pop(k, None)
        os.environ.update(env)
        egemm.set_config(*cfg)
        f = lambda: egemm.gemm(None, None, a_split=a_s, b_split=b_s, out=D)  # noqa: E731
        timeit(f, 5, 5)
        egemm.debug_clock_stats(reset=True)
        import time
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        s.record()
        t0, it = time.time(), 0
        while time.time() - t0 < seconds:
            for _ in range(10):
                f()
            it += 10
            torch.cuda.synchronize()
        e.record()
        e.synchronize()
        ms = s.elapsed_time(e) / it
        mhz, cyc, nl = egemm.debug_clock_stats(reset=True)
        tf = fl3 / ms / 1e9
        print("%-22s cfg %-18s %.3f ms  %.0f TF(fp16)  mean %.0f MHz  %.0f kcyc/launch -> "
              "cycle efficiency %.3f" % (tag, cfg, ms, tf, mhz, cyc / 1e3, need / cyc), flush=True)

    which = os.environ.get("DIAG", "issue")
    if which == "power":  # operand-traffic power: NO_TMA on realistic (random) smem data
        for rep in range(2):
            run("normal kc=256", (2, 256, 0, 256), {})
            run("no_tma, random smem", (2, 256, 0, 256),
                {"EGEMM_DEBUG_NO_TMA": "1", "EGEMM_DEBUG_MODE": "32"})
            run("no_tma, stale smem", (2, 256, 0, 256), {"EGEMM_DEBUG_NO_TMA": "1"})
        return
    if which == "issue":  # MMA-issue mechanics: barrier handshakes and commits
        nt = {"EGEMM_DEBUG_NO_TMA": "1", "EGEMM_DEBUG_NO_EPI": "1"}
        kn = (2, 256, 0, n)
        tag = os.path.basename(egemm.LIB_PATH)
        for rep in range(2):
            for kc in (128, 256):
                run("%s kc=%d" % (tag, kc), (2, 256, 0, kc), {})
        run("%s mma-only kc=256" % tag, (2, 256, 0, 256), nt)
    else:
        # data-dependent MMA power: fp16-exact inputs (every lo = 0) vs U[-1,1] fp32 inputs
        a_full, b_full = a_s, b_s
        a_s = egemm.split(A.half().float())
        b_s = egemm.split(B.half().float(), transpose=True)
        run("lo=0 (fp16-exact in)", (2, 256, 0, 256), {})
        a_s, b_s = a_full, b_full
        run("normal", (2, 256, 0, 256), {})
        for rep in range(2):
            for cfg in ((2, 256, 0, 128), (2, 256, 0, 64), (2, 256, 0, 256), (2, 256, 0, n)):
                run("normal", cfg, {})
            cfg = (2, 256, 0, 128)
            run("no_tma", cfg, {"EGEMM_DEBUG_NO_TMA": "1"})
            run("no_epi", cfg, {"EGEMM_DEBUG_NO_EPI": "1"})
            run("no_tma+no_epi", cfg, {"EGEMM_DEBUG_NO_TMA": "1", "EGEMM_DEBUG_NO_EPI": "1"})
            run("no_tma+no_epi kc=n", (2, 256, 0, n), {"EGEMM_DEBUG_NO_TMA": "1",
                                                       "EGEMM_DEBUG_NO_EPI": "1"})
    for k in ("EGEMM_DEBUG_NO_TMA", "EGEMM_DEBUG_NO_EPI"):
        os.environ.pop(k, None)
    egemm.set_config(0, 0, 0, 0)
    if which == "issue":
        return
    Ah, Bh = A.half(), B.half()
    lo_a = (A - Ah.float()).half()
    lo_b = (B - Bh.float()).half()
    for tag, f in (("cublas fp16 hi*hi", lambda: torch.matmul(Ah, Bh)),
                   ("cublas fp16 lo*hi", lambda: torch.matmul(lo_a, Bh)),
                   ("cublas fp16 hi*hi", lambda: torch.matmul(Ah, Bh))):
        ms = timeit(f, 200, 50)
        print("%-24s %.3f ms (steady, 200 calls)" % (tag, ms), flush=True)
    Ahh = torch.cat([Ah, Ah, Ah], 1)  # K = 3n: the same MMA count as one EGEMM launch
    Bhh = torch.cat([Bh, Bh, Bh], 0)
    for tag, f, fl in (("cublas fp16 n^3", lambda: torch.matmul(Ah, Bh), 2.0 * n ** 3),
                       ("cublas fp16 n x n x 3n", lambda: torch.matmul(Ahh, Bhh), fl3),
                       ("egemm (2,256,0,128)", None, fl3)):
        if f is None:
            egemm.set_config(2, 256, 0, 128)
            f = lambda: egemm.gemm(None, None, a_split=a_s, b_split=b_s, out=D)  # noqa: E731
        mhz, ms = spin_mhz(f)
        tf = fl / ms / 1e9
        print("%-24s %.3f ms  %.0f TF | spin-probe SM clock %.0f MHz -> cycle efficiency %.3f"
              % (tag, ms, tf, mhz, tf / (148 * 8192 * mhz * 1e6 / 1e12)), flush=True)


if __name__ == "__main__":
    main()
