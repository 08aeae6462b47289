"""Seeded synthetic input generators shared by the tests, bench.py and the oracle legs.

This module holds NONE of the method's arithmetic (no split, no product, no distance):
only numpy PCG64 draws shaped like the paper's workloads.

* ``uniform``      U[-1, 1] fp32 -- the paper's distribution for Fig. 7.
* ``in_zone``      sign * 2^U[-3, 3): every element inside the 21-bit zone of the split.
* ``stress``       sign * 2^U[-14, 15): the whole normal fp16 exponent range.
* ``integers``     integers in [-lim, lim] (exact-GEMM pin).
* ``clustered``    kNN references / queries around 1024 centres, sigma 0.1.
* ``mixture``      kMeans points from a Gaussian mixture, sigma 0.2.
"""
from __future__ import annotations

import numpy as np


def rng(seed: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(int(seed)))


def uniform(shape, seed: int, lo: float = -1.0, hi: float = 1.0) -> np.ndarray:
    return rng(seed).uniform(lo, hi, size=shape).astype(np.float32)


def in_zone(shape, seed: int) -> np.ndarray:
    g = rng(seed)
    mag = np.exp2(g.uniform(-3.0, 3.0, size=shape))
    sgn = np.where(g.random(size=shape) < 0.5, -1.0, 1.0)
    return (sgn * mag).astype(np.float32)


def stress(shape, seed: int) -> np.ndarray:
    g = rng(seed)
    mag = np.exp2(g.uniform(-14.0, 15.0, size=shape))
    sgn = np.where(g.random(size=shape) < 0.5, -1.0, 1.0)
    return (sgn * mag).astype(np.float32)


def integers(shape, seed: int, lim: int = 32) -> np.ndarray:
    return rng(seed).integers(-lim, lim + 1, size=shape).astype(np.float32)


def clustered(n: int, d: int, seed: int, n_centres: int = 1024, sigma: float = 0.1,
              centres_seed: int | None = None):
    """Rows drawn around ``n_centres`` centres ~ U[-1,1]^d with N(0, sigma^2) noise.
    The centres come from ``centres_seed`` (default ``seed``) so that references and
    queries can share them."""
    cg = rng(seed if centres_seed is None else centres_seed)
    centres = cg.uniform(-1.0, 1.0, size=(n_centres, d))
    g = rng(seed + 7919)
    lab = g.integers(0, n_centres, size=n)
    x = centres[lab] + sigma * g.standard_normal(size=(n, d))
    return x.astype(np.float32)


def mixture(n: int, d: int, k: int, seed: int, sigma: float = 0.2):
    """kMeans workload (BJ configs[4]): n points from a k-centre Gaussian mixture with
    centres ~ U[-1,1]^d.  Returns (points fp32 [n, d], labels int32 [n], centres fp32)."""
    g = rng(seed)
    centres = g.uniform(-1.0, 1.0, size=(k, d))
    lab = g.integers(0, k, size=n)
    x = centres[lab] + sigma * g.standard_normal(size=(n, d))
    return x.astype(np.float32), lab.astype(np.int32), centres.astype(np.float32)


def all_f32_patterns(start: int, count: int) -> np.ndarray:
    """fp32 values whose bit patterns are start, start+1, ..., start+count-1."""
    return np.arange(start, start + count, dtype=np.uint64).astype(np.uint32).view(np.float32)
