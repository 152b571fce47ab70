"""Definitional oracle for tiny cases -- TEST INFRASTRUCTURE ONLY.

The mapper's result written out as the paper states it (SS V.A: the
mapping "that minimizes the concurrent execution time"; L2106-2118: cost = data transfer
+ kernel execution cost), with the search order and the tie rule fixed by library
semantics rather than by hand-written loops:

* ``itertools.product(range(D), repeat=Q)`` yields device tuples in lexicographic order,
  i.e. increasing mapping index with queue 0 the most significant base-D digit (the same
  as ``numpy.unravel_index(m, (D,)*Q)`` in C order);
* ``min(..., key=score)`` returns the FIRST minimal element in iteration order, which is
  the lowest-index tie rule of BASELINE.json's north_star.

Pure Python, exponential: use only for D**Q up to ~1e5.
"""
from __future__ import annotations

import itertools

import numpy as np


def score(C, mapping) -> int:
    """Concurrent execution time of one mapping: max over devices of the summed cost of
    the queues placed on that device (an idle device contributes 0)."""
    D = len(C[0])
    load = [0] * D
    for q, d in enumerate(mapping):
        load[d] += int(C[q][d])
    return max(load)


def tiny_map(K, X):
    """Return (index, makespan, mapping tuple) for one epoch's [Q][D] tables."""
    K = np.asarray(K, dtype=np.uint64)
    X = np.asarray(X, dtype=np.uint64)
    Q, D = K.shape
    C = [[int(K[q, d]) + int(X[q, d]) for d in range(D)] for q in range(Q)]
    best = min(itertools.product(range(D), repeat=Q), key=lambda t: score(C, t))
    index = int(np.ravel_multi_index(best, (D,) * Q)) if Q > 0 else 0
    return index, score(C, best), tuple(best)


def tiny_map_constrained(K, X, base=None, elig=None):
    """Constrained definition: devices start at ``base`` loads; queue q may only use the
    devices in its mask ``elig[q]`` (0 = any). Enumeration is over the eligible tuples in
    lexicographic order (``itertools.product`` of the per-queue device lists), so ``min``'s
    first-minimum rule is again the lowest full index."""
    K = np.asarray(K, dtype=np.uint64)
    X = np.asarray(X, dtype=np.uint64)
    Q, D = K.shape
    C = [[int(K[q, d]) + int(X[q, d]) for d in range(D)] for q in range(Q)]
    b = [0] * D if base is None else [int(v) for v in base]
    choices = []
    for q in range(Q):
        mask = 0 if elig is None else int(elig[q])
        choices.append([d for d in range(D) if mask == 0 or (mask >> d) & 1])

    def score_b(t):
        load = list(b)
        for q, d in enumerate(t):
            load[d] += C[q][d]
        return max(load)

    best = min(itertools.product(*choices), key=score_b)
    index = int(np.ravel_multi_index(best, (D,) * Q)) if Q > 0 else 0
    return index, score_b(best), tuple(best)
