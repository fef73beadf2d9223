"""Seeded synthetic input generators shared by tests, bench and smoke.

Holds none of the method's arithmetic: random linked lists (the workload of
PAPER.md:20 §V-A, "We use random lists ... pre-compute the predecessor and
successor array") and Monte Carlo layer presets.  Random numbers here come
from numpy's PCG64, not from the generator under test.
"""
from __future__ import annotations

import numpy as np


def random_list(n: int, seed: int = 0x5EED0003):
    """A random linked list over nodes 0..n-1 stored in arrays (§V-A).

    Returns (succ, pred, head): succ[v] = next node or -1 at the tail,
    pred[v] = previous node or -1 at the head.
    """
    perm = np.random.default_rng(seed).permutation(n).astype(np.int32)
    succ = np.full(n, -1, dtype=np.int32)
    pred = np.full(n, -1, dtype=np.int32)
    if n > 1:
        succ[perm[:-1]] = perm[1:]
        pred[perm[1:]] = perm[:-1]
    return succ, pred, int(perm[0])


def ordered_list(n: int):
    """The identity list 0 -> 1 -> ... -> n-1 (best case for memory access)."""
    succ = np.arange(1, n + 1, dtype=np.int32)
    succ[-1] = -1
    pred = np.arange(-1, n - 1, dtype=np.int32)
    return succ, pred, 0
