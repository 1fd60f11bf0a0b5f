"""Seeded synthetic inputs shared by the oracle tests, the GPU parity tests and bench.py.

This module holds NONE of the method's arithmetic (no packing, no deltas, no RLE):
it only draws columns with the shapes and value distributions of the paper's
workloads.  Every generator takes an explicit seed.

Recipes (BASELINE.json configs):
  C1  uniform(b):      rng(1000+b).integers(0, 2**b, n)            P:1419-1423 [R21]
  C2  sweep(b):        b=0 zeros; 1..31 integers(0, 2**b); 32 full-range uint32 as int32
  C3  sorted keys:     D1 floor(i * U / n), sorted uniform sample,
                       near-sorted (1% positions jittered), consecutive 0..n-1
  C4  runs(L):         lengths integers(1, 2L) (mean L), values integers(0, 2**16), repeated
"""
from __future__ import annotations

import numpy as np


def uniform_bits(b: int, n: int, seed: int | None = None) -> np.ndarray:
    """Values uniform in [0, 2^b) -- 'exactly b effective bits'.
    b = 0 gives zeros; b = 32 gives full-range uint32 bit-cast to int32 [R21]."""
    if seed is None:
        seed = 2000 + b
    rng = np.random.default_rng(seed)
    if b == 0:
        return np.zeros(n, np.int32)
    if b == 32:
        return rng.integers(0, 2**32, n, dtype=np.uint32).view(np.int32)
    return rng.integers(0, 2**b, n, dtype=np.int32)


def c1_column(b: int, n: int = 1_000_000) -> np.ndarray:
    """BASELINE config 1: 1M uniform int32 at bitwidth b (seed 1000+b)."""
    return np.random.default_rng(1000 + b).integers(0, 2**b, n, dtype=np.int32)


def d1_sorted(n: int, ndv: int) -> np.ndarray:
    """D1: sorted array with `ndv` unique values spread evenly:
    x_i = floor(i * ndv / n)."""
    i = np.arange(n, dtype=np.int64)
    return ((i * ndv) // n).astype(np.int32)


def d1_prefix(n: int, ndv: int, total: int) -> np.ndarray:
    """The first n entries of the `total`-long D1 column (cheap slices of huge columns)."""
    i = np.arange(n, dtype=np.int64)
    return ((i * ndv) // total).astype(np.int32)


def sorted_uniform(n: int, seed: int = 3000, density: float = 1.074) -> np.ndarray:
    rng = np.random.default_rng(seed)
    x = rng.integers(0, int(density * n) + 1, n, dtype=np.int64)
    x.sort()
    return x.astype(np.int32)


def near_sorted(n: int, seed: int = 3001, frac: float = 0.01, jitter: int = 64) -> np.ndarray:
    x = sorted_uniform(n, seed).astype(np.int64)
    rng = np.random.default_rng(seed + 1)
    k = max(1, int(frac * n)) if n else 0
    if k:
        pos = rng.integers(0, n, k)
        sign = rng.integers(0, 2, k) * 2 - 1
        x[pos] += sign * rng.integers(1, jitter + 1, k)
    return x.astype(np.int32)


def consecutive(n: int, start: int = 0) -> np.ndarray:
    return np.arange(start, start + n, dtype=np.int64).astype(np.int32)


def runs(n: int, mean_len: int, seed: int | None = None, value_bits: int = 16) -> np.ndarray:
    """Run-heavy column: run lengths uniform in [1, 2L) (mean ~L), run values
    uniform in [0, 2^value_bits), repeated and truncated to n (BASELINE config 4)."""
    if seed is None:
        seed = 4000 + mean_len
    rng = np.random.default_rng(seed)
    nruns = n // max(1, mean_len) + 16
    out = np.empty(0, np.int32)
    chunks = []
    total = 0
    while total < n:
        lens = rng.integers(1, 2 * mean_len, nruns)
        vals = rng.integers(0, 2**value_bits, nruns, dtype=np.int32)
        c = np.repeat(vals, lens)
        chunks.append(c)
        total += len(c)
    out = np.concatenate(chunks)[:n] if chunks else out
    return np.ascontiguousarray(out, dtype=np.int32)


def small_alphabet_columns(max_len: int = 4):
    """Every column of length 0..max_len over {INT32_MIN, -1, 0, 1, 2, 3, INT32_MAX}
    (brute force; 2,801 columns for max_len = 4)."""
    import itertools
    alpha = [-(2**31), -1, 0, 1, 2, 3, 2**31 - 1]
    for L in range(max_len + 1):
        for t in itertools.product(alpha, repeat=L):
            yield np.array(t, dtype=np.int32)


RAGGED_LENGTHS = (0, 1, 31, 32, 33, 127, 128, 129, 511, 512, 513, 1023, 1025, 4097, 5000)


def mixed_columns(seed: int = 77):
    """A spread of value distributions at ragged lengths (edge-case parity)."""
    rng = np.random.default_rng(seed)
    for n in RAGGED_LENGTHS:
        yield f"b0_n{n}", np.zeros(n, np.int32)
        for b in (1, 5, 16, 31):
            yield f"b{b}_n{n}", rng.integers(0, 2**b, n, dtype=np.int32)
        yield f"b32_n{n}", rng.integers(0, 2**32, n, dtype=np.uint32).view(np.int32)
        yield f"neg_n{n}", rng.integers(-(2**31), 2**31, n, dtype=np.int64).astype(np.int32)
        yield f"runs_n{n}", runs(n, 6, seed=int(rng.integers(1 << 30)))
        yield f"sorted_n{n}", np.sort(rng.integers(0, 1 << 20, n)).astype(np.int32)


def bernoulli_bitmap(n: int, sigma: float, seed: int = 6000) -> np.ndarray:
    """Predicate bitvector of the random-access experiment: each of the n rows
    selected independently with probability sigma.  Returned as little-endian u32 words,
    bit i of word k = row 32 k + i (include/tilepack.h tp_bitmap_sum), ceil(n/32) words."""
    rng = np.random.default_rng(seed)
    words = (n + 31) // 32
    bits = np.zeros(words * 32, np.uint8)
    if sigma >= 1.0:
        bits[:n] = 1
    elif sigma > 0.0:
        k = rng.binomial(n, sigma)
        bits[rng.choice(n, size=k, replace=False) if k < n // 4 else np.flatnonzero(rng.random(n) < sigma)] = 1
    return np.packbits(bits, bitorder="little").view(np.uint32).copy()
