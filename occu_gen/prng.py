"""Counter-based PRNG shared (by specification, not by code) between the input
generators and the C library's ``occu_init_weights``.

splitmix64 (Steele, Lea & Flood 2014): state += 0x9E3779B97F4A7C15, then the
output mix.  Both the Python generator (here) and ``csrc/weights.cpp`` implement
this same sequence independently.  This module holds none of
the method's arithmetic.
"""
from __future__ import annotations

import numpy as np

_GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)


def splitmix64_stream(seed: int, count: int, offset: int = 0) -> np.ndarray:
    """Return outputs ``offset .. offset+count-1`` of the splitmix64 stream.

    Output j (0-based) is mix(seed + (j+1)*golden), so the stream is
    counter-based and any element can be produced independently.
    """
    with np.errstate(over="ignore"):
        j = np.arange(offset + 1, offset + count + 1, dtype=np.uint64)
        z = np.uint64(seed) + j * _GOLDEN
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        z = z ^ (z >> np.uint64(31))
    return z


def uniform01(seed: int, count: int, offset: int = 0) -> np.ndarray:
    """Doubles in [0, 1): top 53 bits of each splitmix64 output times 2^-53."""
    z = splitmix64_stream(seed, count, offset)
    return (z >> np.uint64(11)).astype(np.float64) * (1.0 / 9007199254740992.0)


class Rng:
    """Small sequential wrapper used by the graph/feature generators."""

    def __init__(self, seed: int):
        self.seed = int(seed) & 0xFFFFFFFFFFFFFFFF
        self.pos = 0

    def uniform(self, n: int = 1) -> np.ndarray:
        u = uniform01(self.seed, n, self.pos)
        self.pos += n
        return u

    def randint(self, lo: int, hi: int, n: int = 1) -> np.ndarray:
        """Integers in [lo, hi] inclusive."""
        u = self.uniform(n)
        return (lo + np.floor(u * (hi - lo + 1))).astype(np.int64)

    def choice(self, seq):
        i = int(self.randint(0, len(seq) - 1, 1)[0])
        return seq[i]

    def permutation(self, n: int) -> np.ndarray:
        """Fisher-Yates driven by the stream (deterministic across platforms)."""
        p = np.arange(n, dtype=np.int64)
        if n <= 1:
            return p
        u = self.uniform(n - 1)
        for i in range(n - 1, 0, -1):
            j = int(u[n - 1 - i] * (i + 1))
            p[i], p[j] = p[j], p[i]
        return p
