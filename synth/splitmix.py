"""SplitMix64 (Steele, Lea, Flood 2014; Vigna's public-domain splitmix64.c).

Counter-based: output for counter value ``s`` is ``mix(s)`` where the state
sequence is ``seed + k * GOLDEN``.  Vectorised with numpy uint64 (wrapping).
The CUDA side (paper_conf_ipps_boyermk13_b200/csrc/synth.cu) implements the
same function independently; tests compare the two.
"""
import numpy as np

GOLDEN = 0x9E3779B97F4A7C15
M1 = 0xBF58476D1CE4E5B9
M2 = 0x94D049BB133111EB
MASK64 = (1 << 64) - 1


def mix64(z):
    """SplitMix64 finaliser on a numpy uint64 array (or python int)."""
    if isinstance(z, int):
        z &= MASK64
        z ^= z >> 30
        z = (z * M1) & MASK64
        z ^= z >> 27
        z = (z * M2) & MASK64
        z ^= z >> 31
        return z
    z = np.asarray(z, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = z ^ (z >> np.uint64(30))
        z = z * np.uint64(M1)
        z = z ^ (z >> np.uint64(27))
        z = z * np.uint64(M2)
        z = z ^ (z >> np.uint64(31))
    return z


def counter(seed, k):
    """Output number k (k >= 0) of the stream seeded with ``seed``:
    mix(seed + (k + 1) * GOLDEN)."""
    if isinstance(k, int):
        return mix64((seed + (k + 1) * GOLDEN) & MASK64)
    k = np.asarray(k, dtype=np.uint64)
    with np.errstate(over="ignore"):
        s = np.uint64(seed & MASK64) + (k + np.uint64(1)) * np.uint64(GOLDEN)
    return mix64(s)


class Stream:
    """Sequential SplitMix64 stream (used to build random skeletons)."""

    def __init__(self, seed):
        self.state = seed & MASK64

    def next(self):
        self.state = (self.state + GOLDEN) & MASK64
        return mix64(self.state)

    def randint(self, lo, hi):
        """Uniform-ish integer in [lo, hi] (modulo reduction)."""
        return lo + self.next() % (hi - lo + 1)

    def uniform(self):
        return (self.next() >> 11) * (1.0 / (1 << 53))

    def bernoulli(self, p):
        return self.uniform() < p

    def choice(self, seq):
        return seq[self.randint(0, len(seq) - 1)]

    def sample(self, n, k):
        """k distinct values of range(n) (partial Fisher-Yates)."""
        pool = list(range(n))
        for i in range(k):
            j = self.randint(i, n - 1)
            pool[i], pool[j] = pool[j], pool[i]
        return pool[:k]
