"""NEXT-2: Fig. 9's skewed shapes (M, N, K) = (N, N, 2N) and (4N, N, N)
 on B200, with the paper's vendor baselines (Table 5,
P:1663-1676) re-measured on the same GPU as CONTEXT (library code, not our path):

* cuBLAS-CUDA-FP32   cublasGemmEx fp32, CUBLAS_COMPUTE_32F (no TF32)
* cuBLAS-TC-Half     cublasGemmEx fp16 in, fp32 out
* cuBLAS-TC-Emulation Alg. 1 as 3 cublasGemmEx fp16 calls accumulating into one fp32 C
                     (beta = 1), on our split kernel's hi / lo
* cuBLAS-BF16x9      cublasGemmEx fp32 with CUBLAS_COMPUTE_32F_EMULATED_16BFX9 (cuBLAS 12.9's
                     own fp32 emulation on Blackwell tensor cores; no paper counterpart)

EGEMM is timed through the public call egemm.gemm(A, B) (fp32 in, split inside, tuned
config).  Every number includes the splits.  Precision: normwise error vs the oracle's fp64
GEMM on sampled rows.  Writes profiles/next2_skewed.json.  Tool code (imports oracle/ only
for the error reference).

usage: python tools/next2_skewed.py [N ...]      (default 1024 2048 4096 8192)
"""
import ctypes
import json
import os
import sys

# cuBLAS 12.9 (system) has the BF16x9 compute type; torch bundles 12.8.  Load the system
# libraries first (same sonames) so torch and this tool share one cuBLAS 12.9.
_CUDA_LIB = "/usr/local/cuda/lib64"
for _so in ("libcublasLt.so.12", "libcublas.so.12"):
    ctypes.CDLL(os.path.join(_CUDA_LIB, _so), mode=ctypes.RTLD_GLOBAL)

import numpy as np  # noqa: E402
import torch  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
from paper_conf_ppopp_fengwcz0d21_b200 import egemm, inputs  # noqa: E402

R_16F, R_32F = 2, 0
COMPUTE_32F, COMPUTE_32F_BF16X9 = 68, 78
OP_N = 0


class Cublas:
    """Minimal ctypes cublasGemmEx on row-major torch tensors (D = A @ B computed as the
    column-major D^T = B^T A^T)."""

    def __init__(self):
        self.L = ctypes.CDLL(os.path.join(_CUDA_LIB, "libcublas.so.12"))
        self.h = ctypes.c_void_p()
        assert self.L.cublasCreate_v2(ctypes.byref(self.h)) == 0
        self.L.cublasGemmEx.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_int,
                                        ctypes.c_int, ctypes.c_int, ctypes.c_int,
                                        ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int,
                                        ctypes.c_int, ctypes.c_void_p, ctypes.c_int,
                                        ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p,
                                        ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int]
        self.L.cublasSetStream_v2(self.h, ctypes.c_void_p(torch.cuda.current_stream().cuda_stream))
        v = ctypes.c_int()
        self.L.cublasGetVersion_v2(self.h, ctypes.byref(v))
        self.version = v.value

    def gemm(self, A, B, D, beta=0.0, compute=COMPUTE_32F):
        M, K = A.shape
        N = B.shape[1]
        t = {torch.float16: R_16F, torch.float32: R_32F}
        al, be = ctypes.c_float(1.0), ctypes.c_float(beta)
        st = self.L.cublasGemmEx(self.h, OP_N, OP_N, N, M, K, ctypes.byref(al),
                                 ctypes.c_void_p(B.data_ptr()), t[B.dtype], N,
                                 ctypes.c_void_p(A.data_ptr()), t[A.dtype], K, ctypes.byref(be),
                                 ctypes.c_void_p(D.data_ptr()), R_32F, N, compute, -1)
        if st != 0:
            raise RuntimeError("cublasGemmEx status %d" % st)


def _time(fn, reps=None, window_ms=400.0):
    """Steady-state ms per call: ~100 ms of warm-up calls, then one event-timed window of
    back-to-back calls lasting ~window_ms (the power-capped clock settles within tens of ms;
    short windows favour whichever kernel runs first on a cool GPU)."""
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    fn()
    torch.cuda.synchronize()
    s.record()
    fn()
    e.record()
    e.synchronize()
    one = max(s.elapsed_time(e), 1e-3)
    for _ in range(max(1, int(100.0 / one))):
        fn()
    n = max(3, int(window_ms / one))
    s.record()
    for _ in range(n):
        fn()
    e.record()
    e.synchronize()
    return s.elapsed_time(e) / n


def run_shape(cb, M, N, K, sample=64):
    A = torch.from_numpy(inputs.uniform((M, K), M ^ 31)).cuda()
    B = torch.from_numpy(inputs.uniform((K, N), N ^ 37 + K)).cuda()
    D = torch.empty(M, N, device="cuda")
    fl = 2.0 * M * N * K
    reps = None
    rows = np.sort(inputs.rng(M + N + K).choice(M, size=sample, replace=False))
    Ah, Bh = A.cpu().numpy()[rows], B.cpu().numpy()
    ref = oracle.gemm64(Ah, Bh)
    res = {"M": M, "N": N, "K": K}

    def record(name, fn):
        ms = _time(fn, reps)
        Dh = D.cpu().numpy()[rows] if name != "egemm" else None
        res[name] = {"ms": round(ms, 4), "tflops": round(fl / ms / 1e9, 1)}
        return Dh

    ws = torch.empty(egemm.gemm_workspace_size(M, N, K), dtype=torch.uint8, device="cuda")
    record("egemm", lambda: egemm.gemm(A, B, out=D, workspace=ws))
    res["egemm"]["normwise_vs_fp64"] = oracle.normwise_error(D.cpu().numpy()[rows], Ah, Bh, ref)
    cfg = egemm.query_config("gemm", M, N, K, with_fused=True)
    res["egemm"]["config"] = list(cfg)

    def tc_emulation():  # split A, split B (row-major hi/lo, fp16), 3 GemmEx into one fp32 C
        ah, al = egemm.split(A)
        bh, bl = egemm.split(B)
        cb.gemm(ah.view(torch.float16), bh.view(torch.float16), D, 0.0)
        cb.gemm(ah.view(torch.float16), bl.view(torch.float16), D, 1.0)
        cb.gemm(al.view(torch.float16), bh.view(torch.float16), D, 1.0)

    for name, fn in (("cublas_cuda_fp32", lambda: cb.gemm(A, B, D)),
                     ("cublas_tc_emulation_3x", tc_emulation),
                     ("cublas_bf16x9", lambda: cb.gemm(A, B, D, 0.0, COMPUTE_32F_BF16X9))):
        try:
            Dh = record(name, fn)
            res[name]["normwise_vs_fp64"] = oracle.normwise_error(Dh, Ah, Bh, ref)
        except Exception as ex:  # pragma: no cover
            res[name] = {"error": str(ex)[:160]}
    Ahf, Bhf = A.half(), B.half()
    try:
        Dh = record("cublas_tc_half", lambda: cb.gemm(Ahf, Bhf, D))
        res["cublas_tc_half"]["normwise_vs_fp64"] = oracle.normwise_error(Dh, Ah, Bh, ref)
    except Exception as ex:  # pragma: no cover
        res["cublas_tc_half"] = {"error": str(ex)[:160]}
    del A, B, D, ws
    torch.cuda.empty_cache()
    return res


def main():
    ns = [int(a) for a in sys.argv[1:]] or [1024, 2048, 4096, 8192]
    cb = Cublas()
    out = {"cublas_version": cb.version, "what": "Fig. 9 skewed shapes (P:2002-2081) + Table 5 vendor baselines on one B200; "
                   "TFLOP/s = 2MNK / time, splits included; normwise error vs fp64 on 64 rows",
           "shapes": []}
    for n in ns:
        for (M, N, K) in ((n, n, 2 * n), (4 * n, n, n)):
            r = run_shape(cb, M, N, K)
            out["shapes"].append(r)
            print(json.dumps(r), flush=True)
    os.makedirs(os.path.join(ROOT, "profiles"), exist_ok=True)
    json.dump(out, open(os.path.join(ROOT, "profiles", "next2_skewed.json"), "w"), indent=1)


if __name__ == "__main__":
    main()
