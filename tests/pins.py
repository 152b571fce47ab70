"""Independent exact methods used to PIN the oracle (not to test the CUDA path directly).

Each function reaches the optimal makespan by a different algorithm than brute-force
enumeration, so a plausible mistake in the oracle (dropped transfer term, transposed
table, wrong digit order, wrong tie rule, sum/max swapped) disagrees with at least one.
"""
from __future__ import annotations

import math

import numpy as np


def subset_sum_two_identical(w) -> int:
    """Optimal makespan for D = 2 IDENTICAL devices (C[q][0] == C[q][1] == w_q).

    Textbook two-way partition: makespan* = S - (largest subset sum <= floor(S/2)),
    by a subset-sum reachability DP (bitset over sums).
    """
    w = [int(v) for v in w]
    S = sum(w)
    reach = 1  # bit s set <=> some subset sums to s
    for v in w:
        reach |= reach << v
    half = S // 2
    best = max(s for s in range(half + 1) if (reach >> s) & 1)
    return S - best


def load_vector_dp(C, base=None, elig=None) -> int:
    """Optimal makespan for unrelated devices by a DP over queues whose state is the set of
    reachable device-load vectors (the pseudo-polynomial 'dynamic programming' reading of
    PAPER.md L1048-1052, reading R1). Only for small integer costs. Optional
    ``base`` (initial device loads) and ``elig`` (per-queue device masks, 0 = any) give the
    constrained variant: the DP simply starts from ``base`` and only takes eligible moves."""
    C = [[int(v) for v in row] for row in C]
    D = len(C[0])
    states = {tuple([0] * D) if base is None else tuple(int(v) for v in base)}
    for q, row in enumerate(C):
        mask = 0 if elig is None else int(elig[q])
        nxt = set()
        for s in states:
            for d in range(D):
                if mask and not (mask >> d) & 1:
                    continue
                t = list(s)
                t[d] += row[d]
                nxt.add(tuple(t))
        states = nxt
    return min(max(s) for s in states)


def lower_bounds(C) -> tuple[int, int]:
    """Two valid lower bounds on the optimal makespan for unrelated devices:
    ceil(sum_q min_d C[q][d] / D)   (total work spread perfectly), and
    max_q min_d C[q][d]             (every queue must run somewhere)."""
    C = np.asarray(C, dtype=object)
    Q, D = C.shape
    mins = [min(int(v) for v in C[q]) for q in range(Q)]
    return math.ceil(sum(mins) / D), max(mins)


def all_equal_closed_form(Q: int, D: int, c: int) -> tuple[int, int, tuple]:
    """All costs equal c: makespan* = c * ceil(Q / D); the lexicographically first tuple
    with no device used more than ceil(Q/D) times is (0,..,0,1,..,1,..) with each device
    repeated ceil(Q/D) times in order. Returns (index, makespan, tuple)."""
    cap = -(-Q // D)
    tup = tuple(t // cap for t in range(Q))
    idx = 0
    for d in tup:
        idx = idx * D + d
    return idx, c * cap, tup
