"""CPU checks of the C-ABI boundary: the library builds for sm_100a, loads without a GPU,
exports every symbol include/egemm.h declares, and validates arguments host-side."""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "egemm.h")


def _declared():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(egemm_[a-z_0-9]+)\s*\(", src)))


@pytest.fixture(scope="module")
def lib():
    from paper_conf_ppopp_fengwcz0d21_b200 import build, egemm
    build.build()
    return egemm.load()


def test_header_declares_the_boundary():
    names = _declared()
    for n in ("egemm_split", "egemm_gemm", "egemm_knn", "egemm_kmeans_step", "egemm_kmeans_finalize"):
        assert n in names


def test_library_exports_every_declared_symbol(lib):
    from paper_conf_ppopp_fengwcz0d21_b200 import egemm
    out = subprocess.check_output(["nm", "-D", "--defined-only", egemm.LIB_PATH]).decode()
    exported = set(line.split()[-1] for line in out.splitlines() if line.strip())
    missing = [n for n in _declared() if n not in exported]
    assert not missing, missing
    for n in _declared():
        getattr(lib, n)  # resolvable through ctypes


def test_library_is_sm100a_tcgen05(lib):
    """The cubin targets sm_100a and contains tcgen05 MMAs and TMA loads (SASS)."""
    from paper_conf_ppopp_fengwcz0d21_b200 import egemm
    sass = subprocess.check_output(["cuobjdump", "-sass", egemm.LIB_PATH]).decode()
    assert "sm_100a" in subprocess.check_output(["cuobjdump", "-lelf", egemm.LIB_PATH]).decode() or \
        "arch = sm_100a" in sass
    assert "UTCHMMA" in sass and "UTMALDG" in sass and "LDTM" in sass


def test_status_strings_and_host_validation(lib):
    from paper_conf_ppopp_fengwcz0d21_b200 import egemm
    assert lib.egemm_status_string(0) == b"EGEMM_OK"
    assert lib.egemm_status_string(4) == b"EGEMM_ERR_WORKSPACE"
    # negative sizes are rejected before any device work
    assert lib.egemm_split(None, -1, 4, 4, None, None, 4, 0, None, None) == egemm.ERR_INVALID_ARG
    op = egemm.Operand()
    assert lib.egemm_gemm(4, 4, 4, op, op, None, 0, None, 4, 7, None, 0, None) == egemm.ERR_INVALID_ARG
    # empty problems are a no-op
    assert lib.egemm_gemm(0, 4, 4, op, op, None, 0, None, 4, 0, None, 0, None) == egemm.OK
    assert lib.egemm_tc_probe(3, 64, 16, None, None, None, None, None) == egemm.ERR_INVALID_ARG
    assert lib.egemm_tc_probe(0, 17, 16, None, None, None, None, None) == egemm.ERR_INVALID_ARG
    assert lib.egemm_tc_probe(2, 64, 129, None, None, None, None, None) == egemm.ERR_INVALID_ARG
    assert lib.egemm_set_config(3, 256, 0, 0) == egemm.ERR_UNSUPPORTED
    assert lib.egemm_set_config(0, 0, 0, 0) == egemm.OK


def test_workspace_queries(lib):
    from paper_conf_ppopp_fengwcz0d21_b200 import egemm
    # hi + lo of A and B, plus 256 B of k-pacing counters (optional for egemm_gemm)
    assert egemm.gemm_workspace_size(256, 256, 256) == 4 * 256 * 256 * 2 + 256
    assert egemm.gemm_workspace_size(256, 256, 256, True, True) == 256
    assert egemm.gemm_workspace_size(0, 5, 5) == 0
    assert egemm.knn_workspace_size(1000, 10, 128, 16) > 0
    assert egemm.kmeans_workspace_size(1000, 64, 10) > 0


def test_tune_table_lookup(tmp_path):
    """The measured table (a-8) is parsed and consulted (first matching bucket wins);
    host-only, so it runs without a GPU (fresh process: the table is loaded once)."""
    import json
    import subprocess
    import sys
    t = {"entries": [
        {"op": "gemm", "m_max": 128, "n_max": 1 << 40, "k_max": 1 << 40, "cg": 1, "bn": 128,
         "sep": 1, "kc": 128, "note": {"nested": [1, 2]}},
        {"op": "gemm", "m_max": 1 << 40, "n_max": 1 << 40, "k_max": 1 << 40, "cg": 2, "bn": 256,
         "sep": 0, "kc": 128}]}
    p = tmp_path / "t.json"
    p.write_text(json.dumps(t))
    code = ("import sys; sys.path.insert(0, %r); from paper_conf_ppopp_fengwcz0d21_b200 import egemm;"
            "print(egemm.tune_table()[1], egemm.query_config('gemm', 100, 5000, 64),"
            " egemm.query_config('gemm', 9000, 9000, 9000), egemm.query_config('knn', 10, 10, 100))"
            % ROOT)
    out = subprocess.check_output([sys.executable, "-c", code],
                                  env=dict(os.environ, EGEMM_TUNE_TABLE=str(p))).decode().strip()
    assert out == "2 (1, 128, 1, 128) (2, 256, 0, 128) (2, 256, 0, 128)", out


def test_tune_table_gemm_b32_rows(tmp_path):
    """The fp32-B rows ("gemm_b32", the B split is part of the call) are consulted for that op
    only, fall back to the "gemm" rows where they have no bucket, and report the fused-B
    flag (2) for the fused-B kernel; the shipped table parses completely."""
    import json
    import subprocess
    import sys
    t = {"entries": [
        {"op": "gemm", "m_max": 1 << 40, "n_max": 1 << 40, "k_max": 1 << 40, "cg": 2, "bn": 224,
         "sep": 0, "kc": 256, "fa": 0},
        {"op": "gemm_b32", "m_max": 1024, "n_max": 1 << 40, "k_max": 1 << 40, "cg": 2, "bn": 256,
         "sep": 0, "kc": 256, "fa": 2}]}
    p = tmp_path / "t.json"
    p.write_text(json.dumps(t))
    code = ("import sys; sys.path.insert(0, %r); from paper_conf_ppopp_fengwcz0d21_b200 import egemm;"
            "print(egemm.query_config('gemm_b32', 1024, 8192, 8192, with_fused=True),"
            " egemm.query_config('gemm', 1024, 8192, 8192, with_fused=True),"
            " egemm.query_config('gemm_b32', 4096, 8192, 8192, with_fused=True))" % ROOT)
    out = subprocess.check_output([sys.executable, "-c", code],
                                  env=dict(os.environ, EGEMM_TUNE_TABLE=str(p))).decode().strip()
    assert out == "(2, 256, 0, 256, 2) (2, 224, 0, 256, 0) (2, 224, 0, 256, 0)", out
    shipped = json.load(open(os.path.join(ROOT, "paper_conf_ppopp_fengwcz0d21_b200", "tune_table.json")))
    code = ("import sys; sys.path.insert(0, %r); from paper_conf_ppopp_fengwcz0d21_b200 import egemm;"
            "print(egemm.tune_table()[1])" % ROOT)
    env = {k: v for k, v in os.environ.items() if k != "EGEMM_TUNE_TABLE"}
    n = int(subprocess.check_output([sys.executable, "-c", code], env=env).decode().strip())
    assert n == len(shipped["entries"])


def test_no_gpu_means_loud_failure(lib):
    """Without a device the compute entry points fail loudly (no CPU fallback)."""
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    from paper_conf_ppopp_fengwcz0d21_b200 import egemm
    buf = ctypes.create_string_buffer(64)
    r = lib.egemm_split(ctypes.cast(buf, ctypes.c_void_p), 2, 2, 2, ctypes.cast(buf, ctypes.c_void_p),
                        ctypes.cast(buf, ctypes.c_void_p), 2, 0, None, None)
    assert r == egemm.ERR_CUDA


def test_config_override_round_trip_and_validation(lib):
    """egemm_set_config_ex / egemm_query_config_ex (the tuning table's value type)
    work on the host: an override is visible in the query, invalid values are rejected, and
    NULL restores the table."""
    from paper_conf_ppopp_fengwcz0d21_b200 import egemm
    base = egemm.query_config_ex("gemm", 8192, 8192, 8192)
    egemm.set_config_ex(cg=2, bn=128, sep=1, kc=512, stages=4, fused=1, terms=4)
    try:
        q = egemm.query_config_ex("gemm", 8192, 8192, 8192)
        assert (q["cg"], q["bn"], q["sep"], q["kc"], q["stages"], q["fused"], q["terms"]) == \
            (2, 128, 1, 512, 4, 1, 4)
        k = egemm.query_config_ex("kmeans", 1 << 22, 1024, 64)
        assert k["sep"] == 0 and k["terms"] == 3  # the norm-MMA epilogues: one accumulator, 3 terms
    finally:
        egemm.set_config_ex()
    assert egemm.query_config_ex("gemm", 8192, 8192, 8192) == base
    for bad in (dict(cg=2, bn=200), dict(kc=100), dict(stages=7), dict(terms=5), dict(n_slices=17),
                dict(epi_warps=12), dict(fused=3), dict(tail_split=2), dict(ksplit=17)):
        with pytest.raises(egemm.EgemmError) as ei:
            egemm.set_config_ex(**bad)
        assert ei.value.status == egemm.ERR_UNSUPPORTED
    assert base["tail_split"] == 0  # the tail split is opt-in (profiles/r02_tail_split_ab.json)
    egemm.set_config_ex(epi_warps=8, n_slices=4, tail_split=1)
    try:
        assert egemm.query_config_ex("gemm", 65536, 256, 1024)["tail_split"] == 1
        assert egemm.query_config_ex("kmeans", 4096, 1024, 64)["epi_warps"] == 8
        assert egemm.query_config_ex("knn", 4096, 1 << 20, 128)["n_slices"] == 4
    finally:
        egemm.set_config_ex()


def test_knn_limits_and_merge_validation(lib):
    """k up to 64 is accepted by the kNN boundary; egemm_knn_merge validates its
    arguments host-side (no device work)."""
    from paper_conf_ppopp_fengwcz0d21_b200 import egemm
    op = egemm.Operand()
    assert lib.egemm_knn(op, None, 100, op, 10, 8, 65, None, None, None, 0, None) == egemm.ERR_INVALID_ARG
    assert lib.egemm_knn(op, None, 10, op, 10, 8, 11, None, None, None, 0, None) == egemm.ERR_INVALID_ARG
    assert lib.egemm_knn(op, None, 100, op, 0, 8, 64, None, None, None, 0, None) == egemm.OK  # nq = 0
    m = lib.egemm_knn_merge
    assert m(None, None, 2, 10, 16, 65, None, None, None, None) == egemm.ERR_INVALID_ARG
    assert m(None, None, 2, 10, 4, 9, None, None, None, None) == egemm.ERR_INVALID_ARG  # k > 2 * 4
    assert m(None, None, 0, 10, 4, 4, None, None, None, None) == egemm.ERR_INVALID_ARG
    assert m(None, None, 2, 0, 4, 4, None, None, None, None) == egemm.OK
    assert m(None, None, 2, 10, 4, 4, None, None, None, None) == egemm.ERR_INVALID_ARG  # NULL data


def test_peer_reduce_and_bf16_split_validation(lib):
    """egemm_kmeans_allreduce_finalize / egemm_split_bf16 validate host-side (no device work)."""
    import ctypes
    from paper_conf_ppopp_fengwcz0d21_b200 import egemm
    arr = (ctypes.c_void_p * 2)(None, None)
    f = lib.egemm_kmeans_allreduce_finalize
    assert f(arr, arr, 0, 4, 4, None, None, None, None) == egemm.ERR_INVALID_ARG   # no ranks
    assert f(arr, arr, 17, 4, 4, None, None, None, None) == egemm.ERR_INVALID_ARG  # > 16 peers
    assert f(arr, arr, 2, 4, 4, None, None, None, None) == egemm.ERR_INVALID_ARG   # NULL peers
    assert lib.egemm_split_bf16(None, -1, 4, 4, None, None, 4, 0, None) == egemm.ERR_INVALID_ARG
    assert lib.egemm_split_bf16(None, 0, 4, 4, None, None, 4, 0, None) == egemm.OK
    egemm.set_config_ex(operand_format=1)
    try:
        q = egemm.query_config_ex("gemm", 4096, 4096, 4096)
        assert q["operand_format"] == 1 and q["fused"] == 0  # the converters make fp16 parts only
        assert egemm.query_config_ex("knn", 4096, 4096, 128)["operand_format"] == 0
    finally:
        egemm.set_config_ex()


def test_split_k_workspace_size_grows(lib):
    """egemm_gemm_workspace_size includes the split-K parts buffer under a ksplit override."""
    from paper_conf_ppopp_fengwcz0d21_b200 import egemm
    base = egemm.gemm_workspace_size(1024, 1024, 1024)
    egemm.set_config_ex(cg=2, bn=256, sep=0, kc=64, ksplit=4)
    try:
        assert egemm.query_config_ex("gemm", 1024, 1024, 1024)["ksplit"] == 4
        grown = egemm.gemm_workspace_size(1024, 1024, 1024)
    finally:
        egemm.set_config_ex()
    assert grown >= base + 4 * 1024 * 1024 * 4
