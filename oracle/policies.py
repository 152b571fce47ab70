"""Policy baselines of MultiCL's scheduler -- TEST INFRASTRUCTURE ONLY (same rules as
``oracle/__init__.py``: only tests/, smoke() and bench.py's CPU legs may use it; it imports
nothing from the product).

``static_mapping`` is the SCHED_AUTO_STATIC policy written out as the paper states it
(SS V.B "Static Command Queue Scheduling"): "we statically decide the
command queue schedules based only on the device profiles ... The MultiCL runtime uses the
command queue properties (compute intensive, memory intensive, or I/O intensive) as the
selection criterion and chooses the best available device for the given command queue."
Reading R18: every queue independently takes, among its eligible ("available")
devices, the device whose device-profile cost for the queue's class is lowest; equal costs
go to the lowest device id.

``round_robin_mapping`` is ROUND_ROBIN ("schedules the command queue to
the next available device"): queue q of an epoch on device q mod D (reading R14).

Parity status: pinned (tests/test_oracle_policies.py: hand-worked cases, numpy.argmin on a
masked score table, invariants).
"""
from __future__ import annotations

import numpy as np


def static_mapping(hints, device_score, eligible=None):
    """hints [E, Q] class ids; device_score [C, D] (lower is better); eligible [E, Q] bit
    masks (0 = any device) or None. Returns mappings [E, Q] uint8. Raises ValueError for a
    hint >= C or a queue without an eligible device below D."""
    hints = np.asarray(hints)
    score = np.asarray(device_score)
    E, Q = hints.shape
    C, D = score.shape
    out = np.zeros((E, Q), np.uint8)
    for e in range(E):
        for q in range(Q):
            c = int(hints[e, q])
            if c >= C:
                raise ValueError("hint names a class >= C")
            mask = 0 if eligible is None else int(eligible[e, q])
            best_d = None
            for d in range(D):  # ascending device ids: a strict < keeps the lowest on ties
                if mask != 0 and not (mask >> d) & 1:
                    continue
                if best_d is None or int(score[c, d]) < int(score[c, best_d]):
                    best_d = d
            if best_d is None:
                raise ValueError("queue with no eligible device")
            out[e, q] = best_d
    return out


def round_robin_mapping(E: int, Q: int, D: int):
    """ROUND_ROBIN: queue q on device q mod D in every epoch."""
    return np.tile((np.arange(Q) % D).astype(np.uint8), (E, 1))
