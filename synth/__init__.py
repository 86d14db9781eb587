"""Seeded synthetic inputs shared by the oracle tests and the GPU tests/bench.

This module holds NO arithmetic of the method (no SpMV, dot, update or CG
step); it only draws numbers.  Both sides receive the same arrays from here.

Generator: splitmix64 (Steele, Lea & Flood 2014) on a counter, top 53 bits
-> U[0,1).  Recipes:

* ``jacc_vector(n, seed)``: the paper's BLAS-1 input ``round.(rand(SIZE)*100)``
  (Fig. 2): rint(100*U) -> integers 0..100 (ties to even, as
  Julia's ``round``), seeds 42 / 43 for x / y.
* ``uniform(n, seed, lo, hi)``: real-valued test vectors.
* ``integers(n, seed, lo, hi)``: integer-valued fp64 vectors (exact arithmetic
  pins).
"""
from __future__ import annotations

import numpy as np

_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)


def splitmix64(n: int, seed: int) -> np.ndarray:
    """n outputs of splitmix64 started at state `seed` (counter form)."""
    with np.errstate(over="ignore"):
        z = (np.uint64(seed) + np.arange(1, n + 1, dtype=np.uint64)
             * np.uint64(0x9E3779B97F4A7C15))
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        z = z ^ (z >> np.uint64(31))
    return z


def unit(n: int, seed: int) -> np.ndarray:
    """U[0,1) doubles from the top 53 bits."""
    return (splitmix64(n, seed) >> np.uint64(11)).astype(np.float64) * (2.0 ** -53)


def jacc_vector(n: int, seed: int) -> np.ndarray:
    """round(rand*100): integer values 0..100."""
    return np.rint(unit(n, seed) * 100.0)


def uniform(n: int, seed: int, lo: float = -1.0, hi: float = 1.0) -> np.ndarray:
    return lo + (hi - lo) * unit(n, seed)


def integers(n: int, seed: int, lo: int = -1000, hi: int = 1000) -> np.ndarray:
    """Integer-valued fp64 in [lo, hi]."""
    u = unit(n, seed)
    return np.floor(lo + (hi - lo + 1) * u).clip(lo, hi)


def sample_rows(n: int, k: int, seed: int) -> np.ndarray:
    """k distinct sorted row ids in [0, n) plus the first/last rows."""
    k = min(k, n)
    idx = (splitmix64(k, seed) % np.uint64(max(n, 1))).astype(np.int64)
    return np.unique(np.concatenate([idx, [0, n - 1]]).astype(np.int64))


def lbm_state(S: int, seed: int, amp: float = 0.05) -> np.ndarray:
    """A positive D2Q9 state (9 S^2 doubles, distribution k at k S^2 + x S + y):
    1/9 (1 + amp U[-1,1)) everywhere -- density ~1, small random velocities.
    (Input shaping only: no lattice constant of the method is used here.)"""
    return (1.0 / 9.0) * (1.0 + amp * uniform(9 * S * S, seed))
