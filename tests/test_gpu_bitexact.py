"""Bit-exact GEMM parity: the tcgen05 kernel == Alg. 1 executed on the profiled tensor-core
primitive in the paper's step order (oracle.gemm_alg1_tc, Alg. 1 P:749-755 with the
promotion reading R21) for every tile configuration / smem ring depth / promotion
interval / term count / accumulator mode, fused and pre-split A, ragged shapes and C.
The per-element arithmetic of the kernel does not depend on the tile shape, only on
(terms, sep, Kc), so every configuration must match the model bitwise."""
import numpy as np
import pytest

from paper_conf_ppopp_fengwcz0d21_b200 import inputs
from tests.gpu_util import require_gpu, to_dev, to_host

pytestmark = pytest.mark.gpu

CFGS = [(2, 256, 0, 64), (2, 256, 0, 128), (1, 128, 0, 64), (1, 128, 1, 128), (1, 128, 1, 256),
        (2, 128, 1, 256), (2, 224, 0, 128), (2, 224, 0, 256), (2, 128, 0, 64)]


def _gpu(eg, A, B, C, cfg, terms, fused, stages=0):
    """fused: 0 pre-split operands, 1 A split inside the GEMM, 2 B split inside the GEMM
    (the library falls back to pre-split where the tile config has no such variant)."""
    eg.set_config_ex(cg=cfg[0], bn=cfg[1], sep=cfg[2], kc=cfg[3], fused=int(fused), stages=stages)
    try:
        return to_host(eg.gemm(to_dev(A), to_dev(B), to_dev(C) if C is not None else None,
                               terms=terms))
    finally:
        eg.set_config_ex()


@pytest.mark.parametrize("cfg", CFGS)
@pytest.mark.parametrize("shape", [(256, 256, 256), (300, 200, 1000), (129, 257, 65)])
def test_bitexact_vs_alg1_model(oracle_lib, cfg, shape):
    eg = require_gpu()
    M, N, K = shape
    A, B = inputs.uniform((M, K), 20 + K), inputs.uniform((K, N), 21 + N)
    D = _gpu(eg, A, B, None, cfg, 3, False)
    ref = oracle_lib.gemm_alg1_tc(A, B, terms=3, sep=cfg[2], kc=cfg[3])
    assert np.array_equal(D.view(np.uint32), ref.view(np.uint32)), \
        "mismatches: %d" % int((D != ref).sum())


@pytest.mark.parametrize("cfg", [(2, 256, 0, 128), (1, 128, 1, 256), (2, 128, 0, 64)])
@pytest.mark.parametrize("gen", [inputs.stress, inputs.in_zone])
def test_bitexact_terms4_with_c_and_fused(oracle_lib, cfg, gen):
    eg = require_gpu()
    A, B, C = gen((200, 700), 30), gen((700, 300), 31), inputs.uniform((200, 300), 32)
    for terms in (3, 4):
        for fused in (0, 1, 2):
            D = _gpu(eg, A, B, C, cfg, terms, fused)
            ref = oracle_lib.gemm_alg1_tc(A, B, C, terms=terms, sep=cfg[2], kc=cfg[3])
            assert np.array_equal(D.view(np.uint32), ref.view(np.uint32)), (terms, fused)


@pytest.mark.parametrize("shape", [(256, 256, 256), (300, 300, 1000), (129, 260, 65), (512, 1024, 2048),
                                   (1000, 516, 4100)])
@pytest.mark.parametrize("kc,bn", [(64, 256), (256, 256), (128, 224)])
def test_bitexact_fused_b(oracle_lib, shape, kc, bn):
    """B round-split inside the GEMM (converter warpgroup transposing TMA-staged fp32 B
    tiles into the K-major stage) == the model bitwise, ragged N / K included."""
    eg = require_gpu()
    M, N, K = shape
    A, B = inputs.uniform((M, K), 40 + K), inputs.uniform((K, N), 41 + N)
    D = _gpu(eg, A, B, None, (2, bn, 0, kc), 3, 2)
    ref = oracle_lib.gemm_alg1_tc(A, B, terms=3, sep=0, kc=kc)
    assert np.array_equal(D.view(np.uint32), ref.view(np.uint32)), \
        "mismatches: %d" % int((D != ref).sum())


STAGE_CFGS = [((2, 256, 0, 128), 2), ((2, 224, 0, 128), 2), ((2, 128, 0, 64), 3), ((2, 128, 1, 256), 4),
              ((1, 128, 0, 64), 2), ((1, 128, 1, 128), 2)]


@pytest.mark.parametrize("cfg,stages", STAGE_CFGS)
def test_bitexact_stage_variants(oracle_lib, cfg, stages):
    """The non-default smem ring depths of the tuning table's stage axis: same bits."""
    eg = require_gpu()
    A, B = inputs.uniform((300, 1000), 50), inputs.uniform((1000, 260), 51)
    D = _gpu(eg, A, B, None, cfg, 3, 0, stages=stages)
    ref = oracle_lib.gemm_alg1_tc(A, B, terms=3, sep=cfg[2], kc=cfg[3])
    assert np.array_equal(D.view(np.uint32), ref.view(np.uint32))


def test_bitexact_order_worked_example():
    """The worked example of tests/test_oracle_alg1_tc.py on the GPU: a = b = 1.5 + 2^-22
    gives exactly 2.25 + 3 * 2^-22 only in Alg. 1's order (hi*hi first would give one ulp
    less), for every tile configuration."""
    eg = require_gpu()
    x = np.float32(1.5 + 2.0 ** -22)
    A = np.zeros((130, 70), np.float32)
    B = np.zeros((70, 140), np.float32)
    A[:, 37] = x
    B[37, :] = x
    want = np.float32(2.25 + 3 * 2.0 ** -22)
    for cfg in CFGS:
        for terms in (3, 4):
            D = _gpu(eg, A, B, None, cfg, terms, 0)
            assert np.all(D == want), (cfg, terms)


@pytest.mark.parametrize("cfg", [(2, 256, 0, 64), (2, 128, 1, 256), (1, 128, 0, 128)])
@pytest.mark.parametrize("terms", [3, 4])
def test_bitexact_bf16_variant(oracle_lib, cfg, terms):
    """NEXT-3: operand_format = 1 (bf16 hi / lo parts, egemm_split_bf16) == the oracle's Alg. 1
    on bf16 parts bitwise, with a wide exponent range (|x| ~ 2^U[-40, 40]) that fp16 parts
    could not represent."""
    eg = require_gpu()
    g = inputs.rng(60)
    A = (g.uniform(-1, 1, (200, 300)) * 2.0 ** g.integers(-40, 40, (200, 300))).astype(np.float32)
    B = (g.uniform(-1, 1, (300, 260)) * 2.0 ** g.integers(-40, 40, (300, 260))).astype(np.float32)
    eg.set_config_ex(cg=cfg[0], bn=cfg[1], sep=cfg[2], kc=cfg[3], operand_format=1)
    try:
        assert eg.query_config_ex("gemm", 200, 260, 300)["operand_format"] == 1
        D = to_host(eg.gemm(to_dev(A), to_dev(B), terms=terms))
    finally:
        eg.set_config_ex()
    ref = oracle_lib.gemm_alg1_tc(A, B, terms=terms, sep=cfg[2], kc=cfg[3], fmt="bf16")
    assert np.array_equal(D.view(np.uint32), ref.view(np.uint32))


@pytest.mark.parametrize("fused", [0, 1])
@pytest.mark.parametrize("M", [65536, 74 * 256 + 20 * 256 + 37])
def test_tail_peel_same_bits(oracle_lib, fused, M):
    """The peeled last wave (a programmatic dependent launch of 128 x 128 tiles) gives the
    same bits as one launch, and as the oracle's Alg. 1 on sampled rows of the tail."""
    import torch
    eg = require_gpu()
    N, K = 256, 1024
    A, B, C = inputs.uniform((M, K), 70), inputs.uniform((K, N), 71), inputs.uniform((M, N), 72)
    Ad, Bd, Cd = to_dev(A), to_dev(B), to_dev(C)
    out = {}
    for peel in (0, 1):
        eg.set_config_ex(cg=2, bn=256, sep=0, kc=128, fused=fused, tail_peel=peel, tail_split=0)
        try:
            out[peel] = to_host(eg.gemm(Ad, Bd, Cd))
        finally:
            eg.set_config_ex()
    assert np.array_equal(out[0].view(np.uint32), out[1].view(np.uint32))
    rows = np.array([0, M // 2, M - 300, M - 1])
    ref = oracle_lib.gemm_alg1_tc(A[rows], B, C[rows], terms=3, sep=0, kc=128)
    assert np.array_equal(out[1][rows].view(np.uint32), ref.view(np.uint32))


@pytest.mark.parametrize("cfg,fused", [((2, 256, 0, 128), 0), ((1, 128, 0, 64), 0), ((2, 128, 1, 128), 0),
                                       ((2, 256, 0, 64), 1), ((2, 224, 0, 128), 0)])
@pytest.mark.parametrize("ksplit", [2, 3, 4])
def test_bitexact_split_k(oracle_lib, cfg, fused, ksplit):
    """Split-K (R21's k-parts, the table's ksplit axis): each tile's k-parts run as separate
    units and a reduce pass adds their results in k order, then C -- bitwise the oracle's
    Alg. 1 with kpart = 64 * ceil(ceil(K / 64) / ksplit), on ragged shapes, with C."""
    eg = require_gpu()
    for (M, N, K) in ((300, 200, 1000), (129, 257, 4100)):
        A, B, C = inputs.uniform((M, K), 60 + K), inputs.uniform((K, N), 61 + N), inputs.uniform((M, N), 62)
        nkb = -(-K // 64)
        kpart = 64 * -(-nkb // ksplit)
        for terms in (3, 4):
            eg.set_config_ex(cg=cfg[0], bn=cfg[1], sep=cfg[2], kc=cfg[3], fused=fused, ksplit=ksplit)
            try:
                D = to_host(eg.gemm(to_dev(A), to_dev(B), to_dev(C), terms=terms))
            finally:
                eg.set_config_ex()
            ref = oracle_lib.gemm_alg1_tc(A, B, C, terms=terms, sep=cfg[2], kc=cfg[3], kpart=kpart)
            assert np.array_equal(D.view(np.uint32), ref.view(np.uint32)), (M, N, K, terms)


def test_split_k_workspace_too_small():
    """The split-K parts buffer lives in the caller's workspace: a workspace sized without it
    is rejected (EGEMM_ERR_WORKSPACE), never silently run with another arithmetic."""
    import torch
    eg = require_gpu()
    A, B = to_dev(inputs.uniform((256, 512), 1)), to_dev(inputs.uniform((512, 256), 2))
    eg.set_config_ex(cg=2, bn=256, sep=0, kc=64, fused=0)  # (an explicit tile: no split-K)
    small = torch.empty(eg.gemm_workspace_size(256, 256, 512), dtype=torch.uint8, device="cuda")
    D = torch.empty((256, 256), device="cuda")
    eg.set_config_ex(cg=2, bn=256, sep=0, kc=64, fused=0, ksplit=4)
    try:
        st = eg.load().egemm_gemm(256, 256, 512, eg.operand(A), eg.operand(B), None, 0, eg._ptr(D), 256,
                                  0, eg._ptr(small), small.numel(), eg._stream())
        assert st == eg.ERR_WORKSPACE
        D = eg.gemm(A, B)  # the wrapper sizes the workspace under the override
    finally:
        eg.set_config_ex()
    assert torch.isfinite(D).all()


@pytest.mark.parametrize("fused", [0, 1, 2])
@pytest.mark.parametrize("shape,clusters", [((51 * 256 + 37, 300, 1000), 16),  # 104 tiles: 8 split in 2
                                            ((5 * 256 + 37, 700, 4100), 8),     # 18 tiles: 2 split in 4
                                            ((65536, 256, 1024), 0)])          # configs[2]: 34 in 2
def test_tail_split_bitexact(oracle_lib, fused, shape, clusters):
    """Tail split: the tiles of the last, at most half-full wave run as 2..4 k-parts and the
    last part to finish adds them in k order (+ C) -- bitwise the oracle's Alg. 1 with kpart
    (R21) on those tiles and without on the others; the other tiles equal the unsplit launch."""
    import torch
    from tests.gpu_util import alg1_rows_with_tail, tail_split_tiles
    eg = require_gpu()
    M, N, K = shape
    A, B, C = inputs.uniform((M, K), 80 + K), inputs.uniform((K, N), 81), inputs.uniform((M, N), 82)
    Ad, Bd, Cd = to_dev(A), to_dev(B), to_dev(C)
    out = {}
    for ts in (0, 1):
        eg.set_config_ex(cg=2, bn=256, sep=0, kc=128, fused=fused, tail_split=ts, max_clusters=clusters)
        try:
            sched = tail_split_tiles(eg, "gemm_b32", M, N, K)
            out[ts] = to_host(eg.gemm(Ad, Bd, Cd))
        finally:
            eg.set_config_ex()
    tiles, kpart, th, bn = sched
    assert tiles and 2 * 64 <= kpart < K  # the shape exercises the split
    split_rows = sorted({m for m, _ in tiles})
    rows = np.unique(np.concatenate([np.arange(m * th, min(M, m * th + th), 37) for m in split_rows] +
                                    [np.array([m * th + th - 1 for m in split_rows if m * th + th - 1 < M]),
                                     np.array([0, M // 3, M - 1])]))
    ref = alg1_rows_with_tail(oracle_lib, A, B, rows, sched, C=C, kc=128)
    assert np.array_equal(out[1][rows].view(np.uint32), ref.view(np.uint32))
    # tiles outside the split: the unsplit launch's bits
    mask = np.ones((M, N), dtype=bool)
    for m, n in tiles:
        mask[m * th:(m + 1) * th, n * bn:(n + 1) * bn] = False
    assert np.array_equal(out[1][mask].view(np.uint32), out[0][mask].view(np.uint32))


@pytest.mark.parametrize("cfg", [(2, 128, 1, 256), (1, 128, 1, 128), (2, 224, 0, 128), (1, 128, 0, 64)])
def test_tail_split_other_tiles(oracle_lib, cfg):
    """The tail split's fix-up on the other tile shapes / accumulator modes (SEP: the parts
    carry hi*hi + cross totals; single-CTA tiles; 224-wide tiles), with C."""
    from tests.gpu_util import alg1_rows_with_tail, tail_split_tiles
    eg = require_gpu()
    M, N, K = 5 * 256 + 37, 650, 4100
    A, B, C = inputs.uniform((M, K), 83), inputs.uniform((K, N), 84), inputs.uniform((M, N), 85)
    eg.set_config_ex(cg=cfg[0], bn=cfg[1], sep=cfg[2], kc=cfg[3], fused=0, tail_split=1, max_clusters=8)
    try:
        sched = tail_split_tiles(eg, "gemm", M, N, K)
        D = to_host(eg.gemm(to_dev(A), to_dev(B), to_dev(C)))
    finally:
        eg.set_config_ex()
    tiles, kpart, th, bn = sched
    assert tiles and kpart < K
    rows = np.unique(np.concatenate([np.arange(m * th, min(M, m * th + th), 29) for m, _ in tiles] +
                                    [np.array([0, M - 1])]))
    ref = alg1_rows_with_tail(oracle_lib, A, B, rows, sched, C=C, sep=cfg[2], kc=cfg[3])
    assert np.array_equal(D[rows].view(np.uint32), ref.view(np.uint32))


@pytest.mark.parametrize("case", [((300, 700, 4100), (2, 128, 0, 128), 0),    # 2 x 6 tiles: 4 parts
                                  ((1000, 1000, 8192), (2, 128, 0, 128), 0),  # 4 x 8 tiles: 2 parts
                                  ((200, 300, 5000), (1, 128, 1, 128), 0),    # single CTAs, SEP
                                  ((8192, 256, 4096), (2, 256, 0, 128), 1)])  # fused A, 32 tiles
def test_tail_split_single_wave(oracle_lib, case):
    """A single, partly filled wave (tiles <= clusters / 2): every tile runs as k-parts with the
    in-kernel fix-up -- bitwise the oracle's Alg. 1 with kpart (R21), with C; the table turns
    this on for the single-wave K >= 4096 buckets (profiles/r02_tail_split_single_wave.json)."""
    from tests.gpu_util import alg1_rows_with_tail, tail_split_tiles
    eg = require_gpu()
    (M, N, K), cfg, fused = case
    A, B, C = inputs.uniform((M, K), 86), inputs.uniform((K, N), 87), inputs.uniform((M, N), 88)
    eg.set_config_ex(cg=cfg[0], bn=cfg[1], sep=cfg[2], kc=cfg[3], fused=fused, tail_split=1)
    try:
        sched = tail_split_tiles(eg, "gemm_b32", M, N, K)
        D = to_host(eg.gemm(to_dev(A), to_dev(B), to_dev(C)))
    finally:
        eg.set_config_ex()
    tiles, kpart, th, bn = sched
    assert len(tiles) == -(-M // th) * -(-N // bn) and kpart < K  # every tile is split
    rows = np.unique(np.concatenate([np.arange(0, M, 23), np.array([M - 1])]))
    ref = alg1_rows_with_tail(oracle_lib, A, B, rows, sched, C=C, sep=cfg[2], kc=cfg[3])
    assert np.array_equal(D[rows].view(np.uint32), ref.view(np.uint32))


@pytest.mark.parametrize("shape", [(128, 256, 4096), (200, 256, 8192), (256, 1000, 3000)])
def test_table_split_k_small_shapes(oracle_lib, shape):
    """The table's split-K picks for short-M/N, long-K calls (ksplit up to 16, post-sweep
    passes, profiles/r02_ksplit_8_16.json) through the public call with no override: bitwise
    the oracle's Alg. 1 with kpart = the part length the library reports (R21)."""
    eg = require_gpu()
    M, N, K = shape
    c = eg.query_config_ex("gemm_b32", M, N, K)
    assert c["ksplit"] > 1  # the shape exercises a table split-K row
    nkb = -(-K // 64)
    kpart = 64 * -(-nkb // c["ksplit"])
    A, B, C = inputs.uniform((M, K), 90), inputs.uniform((K, N), 91), inputs.uniform((M, N), 92)
    D = to_host(eg.gemm(to_dev(A), to_dev(B), to_dev(C)))
    ref = oracle_lib.gemm_alg1_tc(A, B, C, terms=3, sep=c["sep"], kc=c["kc"], kpart=kpart)
    assert np.array_equal(D.view(np.uint32), ref.view(np.uint32)), int((D != ref).sum())
