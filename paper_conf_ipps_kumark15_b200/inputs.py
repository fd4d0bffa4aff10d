"""Seeded synthetic input generators (shared by tests, bench and smoke).

This module holds NO arithmetic of the method: it only draws the inputs the paper's workloads
are shaped like.  The paper names no datasets; the recipes below are the
DESIGN.md §4 input recipe.  numpy ``default_rng(seed)`` (PCG64); arrays are drawn in the order
listed from one generator.

Workload shapes (BASELINE.json configs):
  C1 LCS 1024 x 1024 ACGT            C2 DTW 16384 x 16384 fp32 random walks
  C3 FS 8192 x 8192 uint8 image      C4 min-path 32768 x 32768 int32 costs in [0, 1024)
  C5 LCS 100000 x 100000 ACGT
"""
from __future__ import annotations

import numpy as np

ACGT = np.frombuffer(b"ACGT", dtype=np.uint8)


def gen_strings(seed: int, m: int, n: int, alphabet: bytes = b"ACGT"):
    """Two i.i.d. uniform strings over ``alphabet`` (ASCII bytes), lengths m and n.

    DNA-like 4-letter alphabet: the paper's LDDP examples are bioinformatics [L26]."""
    rng = np.random.default_rng(seed)
    alpha = np.frombuffer(alphabet, dtype=np.uint8)
    a = alpha[rng.integers(0, len(alpha), m)]
    b = alpha[rng.integers(0, len(alpha), n)]
    return np.ascontiguousarray(a), np.ascontiguousarray(b)


def gen_walks(seed: int, m: int, n: int):
    """Two Gaussian random walks (fp32 cumulative sums of std-normal fp32 steps)."""
    rng = np.random.default_rng(seed)
    x = np.cumsum(rng.standard_normal(m, dtype=np.float32), dtype=np.float32)
    y = np.cumsum(rng.standard_normal(n, dtype=np.float32), dtype=np.float32)
    return np.ascontiguousarray(x), np.ascontiguousarray(y)


def gen_int_walks(seed: int, m: int, n: int, lo: int = -5, hi: int = 5):
    """Integer-valued fp32 series (every DTW sum is exact in fp32: brute-force pins)."""
    rng = np.random.default_rng(seed)
    x = rng.integers(lo, hi + 1, m).astype(np.float32)
    y = rng.integers(lo, hi + 1, n).astype(np.float32)
    return x, y


def gen_image(seed: int, H: int, W: int, kind: str = "ramp"):
    """Synthetic grayscale image (uint8).

    ``ramp``: horizontal ramp 0..255 plus N(0, 16) noise, clipped (C3 primary);
    ``uniform``: i.i.d. uniform bytes (C3 secondary)."""
    rng = np.random.default_rng(seed)
    if kind == "uniform":
        return rng.integers(0, 256, (H, W), dtype=np.uint8)
    if kind == "ramp":
        j = np.arange(W, dtype=np.float64)
        base = 255.0 * j / max(W - 1, 1)
        noise = rng.normal(0.0, 16.0, (H, W))
        return np.clip(np.round(base[None, :] + noise), 0, 255).astype(np.uint8)
    raise ValueError(kind)


def gen_costs(seed: int, H: int, W: int, hi: int = 1024):
    """i.i.d. uniform int32 cell costs in [0, hi) (checkerboard grid, C4)."""
    rng = np.random.default_rng(seed)
    return rng.integers(0, hi, (H, W), dtype=np.int32)


def gen_init(seed: int, H: int, W: int, hi: int = 1 << 20):
    """i.i.d. uniform int32 initial table values in [0, hi) (synthetic f's of [L298])."""
    rng = np.random.default_rng(seed)
    return rng.integers(0, hi, (H, W), dtype=np.int32)
