"""Seeded synthetic inputs shared by the oracle tests and the CUDA path.

This module holds NO arithmetic of the method (no products, no sums, no
splitting): it only draws inputs, so both sides may import it (DESIGN.md
"Input recipe").  The paper states no value distribution for its DGEMM
workload (two 8192x8192 double matrices); the recipe
is SURVEY.md SS8(d):

* dense, row-major, contiguous;
* numpy ``Generator(PCG64(seed))``; float64 via ``.random()``, float32 via
  ``.random(dtype=float32)`` -> U[0, 1);
* seeds A = 1000*id + 1, B = 1000*id + 2 with config ids below;
* secondary distributions: signed U[-1, 1), integers in {-8..8}, and the
  structured identity / permutation / rank-1 families used by the pins.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np


@dataclass(frozen=True)
class Config:
    cid: int
    name: str
    M: int
    N: int
    K: int
    tile: int
    workers: tuple  # worker counts G this config is run with


# BASELINE.json "configs", in order, plus the paper's own shape C0
# (8192x8192 DGEMM on 1 and 2 GPU workers, L1428-1431).
CONFIGS = {
    "C1": Config(1, "64x64x64 matmul, 2x2 tile tasks, single-worker PDL", 64, 64, 64, 32, (1,)),
    "C2": Config(2, "1024^3 matmul, 128x128 tiles, 1 GPU worker", 1024, 1024, 1024, 128, (1,)),
    "C3": Config(3, "4096^3 matmul across 2 and 4 GPU workers", 4096, 4096, 4096, 256, (2, 4)),
    "C4": Config(4, "16384^3 matmul, strong scaling 1/2/4/8", 16384, 16384, 16384, 1024, (1, 2, 4, 8)),
    "C5": Config(5, "ragged 10000x7000x3000 across 8 GPUs", 10000, 7000, 3000, 128, (8,)),
    "C0": Config(8, "paper shape 8192^3 DGEMM", 8192, 8192, 8192, 512, (1, 2)),
}


def seeds(cid: int):
    return 1000 * cid + 1, 1000 * cid + 2


def uniform(shape, dtype, seed):
    """U[0,1) in the requested dtype (float64 or float32)."""
    g = np.random.Generator(np.random.PCG64(seed))
    if np.dtype(dtype) == np.float32:
        return g.random(shape, dtype=np.float32)
    return g.random(shape, dtype=np.float64)


def signed(shape, dtype, seed):
    """U[-1,1): 2*U[0,1) - 1 (exact in binary floating point)."""
    u = uniform(shape, dtype, seed)
    return (u + u - np.asarray(1, dtype=u.dtype)).astype(dtype, copy=False)


def integers(shape, dtype, seed, lo=-8, hi=8):
    g = np.random.Generator(np.random.PCG64(seed))
    return g.integers(lo, hi + 1, size=shape).astype(dtype)


def dyadic(shape, dtype, seed, bits=8):
    """Values k / 2**bits with k uniform in [-2**bits, 2**bits]: exact in fp32/64."""
    g = np.random.Generator(np.random.PCG64(seed))
    k = g.integers(-(1 << bits), (1 << bits) + 1, size=shape)
    return (k.astype(np.float64) / float(1 << bits)).astype(dtype)


def identity(n, m, dtype):
    return np.eye(n, m, dtype=dtype)


def permutation(n, dtype, seed):
    g = np.random.Generator(np.random.PCG64(seed))
    p = g.permutation(n)
    P = np.zeros((n, n), dtype=dtype)
    P[np.arange(n), p] = 1
    return P, p


def rank1_factors(m, n, seed, lo=-4, hi=4):
    """Integer vectors u (m,), v (n,) with entries in [lo, hi] (int64)."""
    g = np.random.Generator(np.random.PCG64(seed))
    return (g.integers(lo, hi + 1, size=m).astype(np.int64),
            g.integers(lo, hi + 1, size=n).astype(np.int64))


def config_inputs(name: str, dtype=np.float64, dist: str = "uniform"):
    """(A, B) for a named config with the SS8(d) seeds."""
    c = CONFIGS[name]
    sa, sb = seeds(c.cid)
    gen = {"uniform": uniform, "signed": signed, "integers": integers}[dist]
    return gen((c.M, c.K), dtype, sa), gen((c.K, c.N), dtype, sb)


def sampled_rows(M: int, boundaries=(), tile: int = 0, n_random: int = 128,
                 seed: int = 7):
    """SURVEY.md SS8(d) sampled-rows rule: {0,1,M-2,M-1}, every worker-boundary
    row +-1, first/last row of the last (partial) task row, plus n_random
    seeded rows.  Returns a sorted int64 array of unique valid row indices."""
    s = {0, 1, M - 2, M - 1}
    for b in boundaries:
        s.update((b - 1, b, b + 1))
    if tile > 0 and M % tile:
        last = (M // tile) * tile
        s.update((last, M - 1))
    g = np.random.Generator(np.random.PCG64(seed))
    s.update(int(x) for x in g.integers(0, M, size=n_random))
    return np.array(sorted(r for r in s if 0 <= r < M), dtype=np.int64)
