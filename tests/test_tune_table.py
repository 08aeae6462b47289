"""The shipped measured table (tune_table.json) is well-formed: every entry names
a launch configuration the kernels implement, and the library parses all of them (no silent
fallback to the built-in defaults).  CPU-only (host code of the library)."""
import json
import os

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
TABLE = os.path.join(ROOT, "paper_conf_ppopp_fengwcz0d21_b200", "tune_table.json")

TILES = {(2, 256, 0), (2, 224, 0), (2, 128, 0), (2, 128, 1), (1, 128, 0), (1, 128, 1)}
FUSED_A = {(2, 256, 0), (2, 128, 0), (2, 128, 1), (1, 128, 0), (1, 128, 1)}
FUSED_B = {(2, 256, 0), (2, 224, 0)}


def _entries():
    return json.load(open(TABLE))["entries"]


def test_entries_are_implemented_configs():
    ops = {"gemm", "gemm_b32", "knn", "kmeans"}
    for e in _entries():
        assert e["op"] in ops, e
        tile = (e["cg"], e["bn"], e["sep"])
        assert tile in TILES, e
        assert e["m_max"] > 0 and e["n_max"] > 0 and e["k_max"] > 0
        if e["op"] in ("gemm", "gemm_b32"):
            assert e["kc"] % 64 == 0 and 64 <= e["kc"] <= 8192, e
            assert e.get("terms", 3) in (0, 3, 4), e
            assert 0 <= e.get("ksplit", 0) <= 16, e
            assert e.get("tsplit", 0) in (0, 1), e
            assert not (e.get("ksplit", 0) > 1 and e.get("tsplit", 0) == 1), e  # one k-split scheme
            fa = e.get("fa", 0)
            assert fa in (0, 1, 2), e
            if fa == 1:
                assert tile in FUSED_A, e
            if fa == 2:
                assert tile in FUSED_B and e["op"] == "gemm_b32", e
            assert e.get("stages", 0) in (0, 2, 3, 4), e
        else:
            assert tile in {(2, 256, 0), (1, 128, 0)}, e  # one accumulator (norm MMA)


def test_buckets_are_unique_and_cover_the_open_ends():
    seen = set()
    for e in _entries():
        key = (e["op"], e["m_max"], e["n_max"], e["k_max"])
        assert key not in seen, key
        seen.add(key)
    for op in ("gemm", "gemm_b32"):
        big = max(e["m_max"] for e in _entries())
        assert (op, big, big, big) in seen  # any shape has a row


def test_library_parses_every_entry():
    from paper_conf_ppopp_fengwcz0d21_b200 import egemm
    path, n = egemm.tune_table()
    assert os.path.samefile(path, TABLE)
    assert n == len(_entries())
    # a split-K row and a tail-split row come back through the query as written
    e = next(x for x in _entries() if x["op"] == "gemm_b32" and x.get("ksplit", 0) > 1)
    q = egemm.query_config_ex("gemm_b32", e["m_max"], e["n_max"], min(e["k_max"], 8192))
    assert q["ksplit"] == e["ksplit"] and q["tail_split"] == 0
    e = next(x for x in _entries() if x["op"] == "gemm_b32" and x.get("tsplit", 0) == 1)
    q = egemm.query_config_ex("gemm_b32", e["m_max"], e["n_max"], min(e["k_max"], 8192))
    assert q["tail_split"] == 1 and q["ksplit"] in (0, 1)
