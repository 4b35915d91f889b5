"""Counter-free SplitMix64 stream used by every synthetic-input generator.

This module holds no arithmetic of the method (no makespan, no move decoding):
it only produces seeded pseudo-random numbers for building inputs, so both the
oracle-side tests and the CUDA-side tests can draw identical graphs, orders and
placements from the same seed (SURVEY.md §8(d) "Generators are deterministic
given a seed (SplitMix64)").
"""

from __future__ import annotations

import math

MASK64 = (1 << 64) - 1


def mix64(z: int) -> int:
    """SplitMix64 finaliser (Steele, Lea, Flood 2014), uint64 wrap-around."""
    z &= MASK64
    z ^= z >> 30
    z = (z * 0xBF58476D1CE4E5B9) & MASK64
    z ^= z >> 27
    z = (z * 0x94D049BB133111EB) & MASK64
    z ^= z >> 31
    return z


class SplitMix64:
    """Sequential SplitMix64 generator: state += golden gamma, output = mix64(state)."""

    GAMMA = 0x9E3779B97F4A7C15

    def __init__(self, seed: int):
        self.state = seed & MASK64

    def next_u64(self) -> int:
        self.state = (self.state + self.GAMMA) & MASK64
        return mix64(self.state)

    def below(self, bound: int) -> int:
        """Integer in [0, bound) (modulo reduction; bias is irrelevant for inputs)."""
        if bound <= 0:
            raise ValueError("bound must be positive")
        return self.next_u64() % bound

    def uniform(self) -> float:
        """Float in [0, 1) with 53 random bits."""
        return (self.next_u64() >> 11) * (1.0 / (1 << 53))

    def chance(self, prob: float) -> bool:
        return self.uniform() < prob

    def log_uniform_int(self, lo: int, hi: int) -> int:
        """Integer in [lo, hi) drawn log-uniformly (lo >= 1)."""
        v = math.exp(math.log(lo) + self.uniform() * (math.log(hi) - math.log(lo)))
        return max(lo, min(hi - 1, int(v)))

    def choice(self, seq):
        return seq[self.below(len(seq))]

    def shuffle(self, lst: list) -> None:
        for i in range(len(lst) - 1, 0, -1):
            j = self.below(i + 1)
            lst[i], lst[j] = lst[j], lst[i]
