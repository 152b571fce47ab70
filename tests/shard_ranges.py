"""Test-side shard layout of masked (mixed-radix) calls, shared by the GPU parity tests and
the gloo protocol test (no method arithmetic: only which full-index range each shard covers).
"""
from __future__ import annotations

import numpy as np


def mixed_shard_ranges(elig_row, Q, D, G, wide=False):
    """Full-index ranges [lo, hi) of the G shards of a masked single-epoch call
    (include/mcl.h: the feasible enumeration cut into contiguous pieces). The mixed-radix
    kernel's reduced space: pinned queues (one eligible device) leave it; the other queues
    keep their order; blocks are the digits of all but the last three of them, each over
    its eligible devices (for u32 with D <= 5 the last of those over all D devices); shard r
    takes blocks [nb r / G, nb (r + 1) / G). A block's first leaf (inner digits 0) bounds
    its full indices from below, so every feasible mapping of shard r lies in
    [first(block lo), first(block hi))."""
    full = (1 << D) - 1
    masks = [(int(m) & full) if int(m) else full for m in elig_row]
    devs = [[d for d in range(D) if (m >> d) & 1] for m in masks]
    w = [D ** (Q - 1 - q) for q in range(Q)]
    pinned = [q for q in range(Q) if len(devs[q]) == 1]
    free = [q for q in range(Q) if len(devs[q]) != 1]
    O = max(0, len(free) - 3)
    outer = free[:O]
    lists = [devs[q] for q in outer]
    if not wide and D <= 5 and O >= 1:
        lists[-1] = list(range(D))
    nb = int(np.prod([len(x) for x in lists])) if lists else 1
    pin_idx = sum(devs[q][0] * w[q] for q in pinned)

    def first(b):
        if b >= nb:
            return D**Q
        f = pin_idx
        for p in range(O - 1, -1, -1):
            r = len(lists[p])
            f += lists[p][b % r] * w[outer[p]]
            b //= r
        return f

    return [(first(nb * r // G), first(nb * (r + 1) // G)) for r in range(G)]
