"""Counter-based random numbers (SplitMix64 finaliser), shared by the oracle tests
and the GPU path's harness as the ONLY common input source.

Every draw is a pure function of ``(seed, stream, counter)``, so a tensor's
values do not depend on thread count, chunking or call order.  This module
holds no SNICIT arithmetic.
"""
from __future__ import annotations

import numpy as np

_GOLD = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)

# named streams (any distinct 64-bit constants)
STREAMS = {
    "template": 1,
    "class": 2,
    "shift": 3,
    "dropout": 4,
    "perm": 5,
    "random_idx": 6,
    "random_val": 7,
    "bias": 8,
    "dense_in": 9,
    "misc": 10,
}


def _mix(z: np.ndarray) -> np.ndarray:
    z = np.asarray(z, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
    return z ^ (z >> np.uint64(31))


def _key(seed: int, stream: int, sub: int = 0) -> np.uint64:
    with np.errstate(over="ignore"):
        k = _mix(np.array([np.uint64(seed & 0xFFFFFFFFFFFFFFFF)], dtype=np.uint64) * _GOLD
                 + np.uint64(stream) * _M1 + np.uint64(sub & 0xFFFFFFFFFFFFFFFF) * _M2)
    return k[0]


def u64(seed: int, stream: str, counters: np.ndarray, sub: int = 0) -> np.ndarray:
    """64-bit random words for the given integer counters."""
    k = _key(seed, STREAMS[stream], sub)
    c = np.asarray(counters, dtype=np.uint64)
    with np.errstate(over="ignore"):
        return _mix(k + c * _GOLD)


def uniform(seed: int, stream: str, counters: np.ndarray, sub: int = 0) -> np.ndarray:
    """Uniform doubles in [0, 1) with 53 random bits."""
    w = u64(seed, stream, counters, sub)
    return (w >> np.uint64(11)).astype(np.float64) * (1.0 / 9007199254740992.0)


def randint(seed: int, stream: str, counters: np.ndarray, high: int, sub: int = 0) -> np.ndarray:
    """Integers in [0, high) (multiply-shift on 53-bit uniforms; bias < 2^-40 for high < 2^13)."""
    return np.minimum((uniform(seed, stream, counters, sub) * high).astype(np.int64), high - 1)


def permutation(seed: int, stream: str, n: int, sub: int = 0) -> np.ndarray:
    """A seeded permutation of range(n): argsort of n random keys (ties broken by index)."""
    keys = u64(seed, stream, np.arange(n, dtype=np.uint64), sub)
    return np.argsort(keys, kind="stable").astype(np.int64)
