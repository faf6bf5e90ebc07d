"""Seed nodes and per-batch RNG seeds (fixture).

* seed nodes of global batch b: Generator(PCG64(base + b)).choice(n, S, replace=False)
  (unique, as Append Unique assumes unique targets);
* rng_seed_b = splitmix64(base_seed ^ b);
* rank r runs the global batches b = r (mod W).
"""

import numpy as np

from .hashing import splitmix64_int


def seed_nodes(n: int, count: int, base: int, batch: int) -> np.ndarray:
    g = np.random.Generator(np.random.PCG64(base + batch))
    return g.choice(n, size=min(count, n), replace=False).astype(np.int64)


def rng_seed(base_seed: int, batch: int) -> int:
    return splitmix64_int((base_seed ^ batch) & ((1 << 64) - 1))


def rank_batches(num_batches: int, rank: int, world: int):
    return [b for b in range(num_batches) if b % world == rank]


def gather_ids(n: int, count: int, base: int, rank: int) -> np.ndarray:
    """Config 4: ids uniform over [0, n) with replacement, PCG64(base + rank)."""
    g = np.random.Generator(np.random.PCG64(base + rank))
    return g.integers(0, n, size=count, dtype=np.int64)
