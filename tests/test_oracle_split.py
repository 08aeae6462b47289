"""Pins for the oracle's round-split (Alg. 1 l.2-3; Fig. 4b).

Every check compares the oracle with something other than itself: the host CPU's F16C
conversion instruction (exhaustive over all 2^32 fp32 patterns), numpy's binary16 cast,
exact float64 arithmetic, and the precision claims of Table 1.
"""
import os
import subprocess

import numpy as np
import pytest

from paper_conf_ppopp_fengwcz0d21_b200 import inputs

HERE = os.path.dirname(os.path.abspath(__file__))


def _has_f16c():
    try:
        return "f16c" in open("/proc/cpuinfo").read()
    except OSError:
        return False


@pytest.mark.skipif(not _has_f16c(), reason="host CPU has no F16C")
def test_f32_to_f16_exhaustive_vs_f16c(oracle_lib, tmp_path):
    """All 2^32 fp32 patterns: oracle bit-level RNE == vcvtps2ph; all 2^16 fp16 decodes
    == vcvtph2ps (NaN by class)."""
    exe = str(tmp_path / "f16c_exhaustive")
    libdir = os.path.dirname(oracle_lib.build())
    subprocess.check_call(["gcc", "-O2", "-mf16c", "-mavx2", "-fopenmp",
                           os.path.join(HERE, "pins", "f16c_exhaustive.c"), "-L" + libdir,
                           "-loracle", "-Wl,-rpath," + libdir, "-o", exe])
    out = subprocess.check_output([exe], timeout=600).decode().split()
    assert out == ["0", "0"], out


def test_split_hi_matches_numpy_cast(oracle_lib):
    """hi = numpy binary16 RNE cast; lo = binary16 cast of the fp32 residual."""
    x = np.concatenate([inputs.uniform(1 << 20, 1), inputs.stress(1 << 20, 2),
                        inputs.all_f32_patterns(0x33000000, 1 << 20)])
    hi, lo = oracle_lib.split(x)
    np_hi = x.astype(np.float16)
    assert np.array_equal(hi, np_hi.view(np.uint16))
    r = (x - np_hi.astype(np.float32)).astype(np.float32)
    assert np.array_equal(lo, r.astype(np.float16).view(np.uint16))


def test_split_exact_on_fp16_values(oracle_lib):
    """An fp16-representable x gives hi = x, lo = +0 (closed form)."""
    h = np.arange(0, 65536, dtype=np.uint32).astype(np.uint16)
    f = h.view(np.float16)
    ok = np.isfinite(f)
    x = f[ok].astype(np.float32)
    hi, lo = oracle_lib.split(x)
    assert np.array_equal(hi, h[ok])
    assert np.all(lo & 0x7FFF == 0)


def test_split_residual_exact_and_bounded(oracle_lib):
    """r = x - hi is exact in fp32 (checked in fp64 inside the oracle) and |lo| <= ulp(hi)/2."""
    x = np.concatenate([inputs.uniform(1 << 20, 3), inputs.in_zone(1 << 20, 4)])
    hi, lo = oracle_lib.split(x)  # raises if any residual was inexact
    fhi, flo = oracle_lib.h2f(hi), oracle_lib.h2f(lo)
    ulp_hi = np.exp2(np.floor(np.log2(np.abs(fhi))) - 10)
    ulp_hi = np.maximum(ulp_hi, 2.0 ** -24)
    assert np.all(np.abs(x.astype(np.float64) - fhi) <= ulp_hi / 2)
    assert np.all(np.abs(flo) <= ulp_hi / 2)


@pytest.mark.parametrize("e", list(range(-3, 16)))
def test_extended_precision_21_bits(oracle_lib, e):
    """Table 1 'Extended-Precision 1-5-21': in the 5-bit exponent range
    (here 2^-3 <= |x| < 65504) hi + lo carries >= 21 explicit mantissa bits, i.e.
    |x - hi - lo| <= 2^(e-22) for x in binade e."""
    g = inputs.rng(100 + e)
    man = g.integers(0, 1 << 23, size=1 << 16, dtype=np.uint32)
    sgn = (g.integers(0, 2, size=1 << 16, dtype=np.uint32) << 31)
    bits = sgn | (np.uint32(e + 127) << 23) | man
    x = bits.view(np.float32)
    x = x[np.abs(x) < 65504]
    hi, lo = oracle_lib.split(x)
    err = np.abs(x.astype(np.float64) - oracle_lib.h2f(hi) - oracle_lib.h2f(lo))
    assert err.max() <= 2.0 ** (e - 22)


def test_split_below_zone_absolute_bound(oracle_lib):
    """Below 2^-3 the lo part goes subnormal: |x - hi - lo| <= 2^-25 (reading R4)."""
    x = inputs.stress(1 << 20, 5)
    x = x[np.abs(x) < 2.0 ** -3]
    hi, lo = oracle_lib.split(x)
    err = np.abs(x.astype(np.float64) - oracle_lib.h2f(hi) - oracle_lib.h2f(lo))
    assert err.max() <= 2.0 ** -25


def test_split_ties_and_variants(oracle_lib):
    """Exact fp16 midpoints: RNE and the paper's literal round-half-away hi differ, but
    hi + lo reconstructs x exactly under both (R1).  Off ties they agree bitwise."""
    g = inputs.rng(6)
    h = g.integers(0x2000, 0x7800, size=4096).astype(np.uint16)  # normal fp16, not max
    f = h.view(np.float16).astype(np.float32)
    nxt = (h + 1).astype(np.uint16).view(np.float16).astype(np.float32)
    mid = ((f.astype(np.float64) + nxt) / 2).astype(np.float32)  # exact midpoint in fp32
    hi_n, lo_n = oracle_lib.split(mid, "rne")
    hi_a, lo_a = oracle_lib.split(mid, "rha")
    for hi, lo in ((hi_n, lo_n), (hi_a, lo_a)):
        assert np.array_equal(oracle_lib.h2f(hi) + oracle_lib.h2f(lo), mid.astype(np.float64))
    assert np.all(hi_n & 1 == 0)  # ties to even
    assert np.all(np.abs(oracle_lib.h2f(hi_a)) > np.abs(mid))  # half away from zero
    x = inputs.uniform(1 << 16, 7)
    tie = (x.view(np.uint32) & 0x1FFF) == 0x1000  # dropped 13 bits are exactly one half
    assert 0 < tie.sum() < 64
    a, b = oracle_lib.split(x, "rne")[0], oracle_lib.split(x, "rha")[0]
    assert np.array_equal(a[~tie], b[~tie])


def test_truncate_split_20_bits(oracle_lib):
    """Markidis truncate-split (Fig. 4a; Table 1 'Markidis 1-5-20'):
    hi = RZ, lo = RZ(x - hi): |x - hi - lo| < 2^(e-20), and hi never exceeds |x|."""
    for e in range(-2, 15):
        g = inputs.rng(200 + e)
        bits = (np.uint32(e + 127) << 23) | g.integers(0, 1 << 23, size=1 << 14, dtype=np.uint32)
        x = bits.view(np.float32)
        hi, lo = oracle_lib.split(x, "trunc")
        fh, fl = oracle_lib.h2f(hi), oracle_lib.h2f(lo)
        assert np.all(fh <= x) and np.all(fl >= 0)
        assert (np.abs(x.astype(np.float64) - fh - fl)).max() < 2.0 ** (e - 20)


def test_overflow_and_specials(oracle_lib):
    x = np.array([65504.0, 65519.99, 65520.0, 1e9, np.inf, -np.inf, np.nan, 0.0, -0.0,
                  2.0 ** -24, 2.0 ** -25, 3 * 2.0 ** -26, 2.0 ** -26], np.float32)
    hi, lo = oracle_lib.split(x)
    fh = oracle_lib.h2f(hi)
    assert fh[0] == 65504 and fh[1] == 65504
    assert np.isinf(fh[2]) and np.isinf(fh[3]) and np.isinf(fh[4]) and fh[5] == -np.inf
    assert np.isnan(fh[6])
    assert hi[7] == 0 and hi[8] == 0x8000
    assert fh[9] == 2.0 ** -24 and fh[10] == 0.0 and fh[11] == 2.0 ** -24 and fh[12] == 0.0


def test_bf16_split_vs_torch_cast_and_exactness(oracle_lib):
    """NEXT-3's bf16 round-split: hi = bf16_RNE(x) equals torch's float32 -> bfloat16 cast (a
    library RNE conversion) on sampled fp32 patterns incl. ties, specials and subnormals;
    x - hi is exact in fp32; |lo| <= half a bf16 ulp of hi; hi + lo keeps >= 16 bits."""
    import torch
    g = np.random.default_rng(123)
    bits = g.integers(0, 2 ** 32, 400000, dtype=np.uint64).astype(np.uint32)
    ties = (g.integers(0, 2 ** 16, 20000, dtype=np.uint32) << 16) | 0x8000  # exact ties
    specials = np.array([0, 0x80000000, 0x7F800000, 0xFF800000, 0x7FC00000, 0x00000001,
                         0x007FFFFF, 0x7F7FFFFF, 0x7F7F8000, 0x3F808000, 0x3F818000], np.uint32)
    x = np.concatenate([bits, ties, specials]).view(np.float32)
    hi, lo = oracle_lib.split(x, "bf16")
    ref = torch.from_numpy(x.copy()).to(torch.bfloat16).view(torch.int16).numpy().view(np.uint16)
    nan = np.isnan(x)
    assert np.array_equal(hi[~nan], ref[~nan])
    assert np.all(np.isnan(oracle_lib.bf16_bits_to_f64(hi[nan])))
    fin = np.isfinite(x) & np.isfinite(oracle_lib.bf16_bits_to_f64(hi))
    h = oracle_lib.bf16_bits_to_f64(hi[fin])
    l = oracle_lib.bf16_bits_to_f64(lo[fin])
    xf = x[fin].astype(np.float64)
    r = xf - h
    assert np.array_equal(r.astype(np.float32).astype(np.float64), r)  # exact in fp32
    ulp = np.where(h != 0, 2.0 ** (np.floor(np.log2(np.abs(np.where(h != 0, h, 1.0)))) - 7), 0)
    assert np.all(np.abs(l) <= ulp / 2 + 2.0 ** -149)
    big = np.abs(xf) > 2.0 ** -100  # away from fp32 subnormals
    assert np.all(np.abs(xf - h - l)[big] <= np.abs(xf[big]) * 2.0 ** -16)
