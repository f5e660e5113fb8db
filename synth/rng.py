"""Counter-based random numbers shared by the numpy and C++ input generators.

Seeded-input infrastructure only: nothing in this package computes any part of
the PCGCN method (no normalisation, no aggregation, no partitioning).  Both the
oracle side (tests) and the CUDA side (bench / tests) consume what it produces.

The generator is splitmix64 (Steele, Lea, Flood 2014): the i-th draw of stream
``key`` is ``mix64(key + (i + 1) * GOLDEN)``.  A pure function of (key, i), so
the C++ generator in ``csrc/synth_gen.cpp`` produces bit-identical streams with
any number of threads.
"""
from __future__ import annotations

import numpy as np

GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_C1 = np.uint64(0xBF58476D1CE4E5B9)
_C2 = np.uint64(0x94D049BB133111EB)
_S30 = np.uint64(30)
_S27 = np.uint64(27)
_S31 = np.uint64(31)
_S11 = np.uint64(11)


def mix64(x: np.ndarray) -> np.ndarray:
    """splitmix64 finaliser on a uint64 array (wrapping arithmetic)."""
    x = np.asarray(x, dtype=np.uint64)
    with np.errstate(over="ignore"):
        x = x ^ (x >> _S30)
        x = x * _C1
        x = x ^ (x >> _S27)
        x = x * _C2
        x = x ^ (x >> _S31)
    return x


def stream_key(seed: int, stream: int) -> np.uint64:
    """Key of an independent stream derived from (seed, stream)."""
    a = np.array([seed & 0xFFFFFFFFFFFFFFFF], dtype=np.uint64)
    b = np.array([stream & 0xFFFFFFFFFFFFFFFF], dtype=np.uint64)
    with np.errstate(over="ignore"):
        k = mix64(a * GOLDEN) ^ mix64(b + GOLDEN)
    return np.uint64(mix64(k)[0])


def draws(key: np.uint64, ctr: np.ndarray) -> np.ndarray:
    """uint64 draws number ``ctr`` of stream ``key``."""
    ctr = np.asarray(ctr, dtype=np.uint64)
    with np.errstate(over="ignore"):
        return mix64(np.uint64(key) + (ctr + np.uint64(1)) * GOLDEN)


def to_unit(u: np.ndarray) -> np.ndarray:
    """uint64 -> float64 uniform in [0, 1) using the top 53 bits (exact)."""
    return (np.asarray(u, dtype=np.uint64) >> _S11).astype(np.float64) * (1.0 / 9007199254740992.0)
