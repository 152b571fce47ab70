"""Pins of the policy baselines' oracle (oracle/policies.py), CPU only."""
from __future__ import annotations

import numpy as np

from oracle import policies

# Device profiles of a CPU + 2 GPU node (device 0 = CPU), lower is
# better: compute-bound kernels run faster on the GPUs, memory-bound ones on the CPU (the
# SNU-NPB pattern of Fig. 3), I/O-bound queues stay on the host-resident CPU.
SCORES = np.array([[4, 1, 1],   # class 0: compute-bound
                   [1, 2, 2],   # class 1: memory-bound
                   [0, 1, 1]],  # class 2: I/O-bound
                  np.uint64)


def test_hand_worked_static_policy():
    hints = np.array([[0, 1, 2, 0]], np.uint8)
    # compute -> the first best GPU (1; GPU 1 ties at 1 and loses to the lower id), memory and
    # I/O -> the CPU
    assert policies.static_mapping(hints, SCORES).tolist() == [[1, 0, 0, 1]]
    # "best available device": queue 0 may only use GPU 1, queue 1 only the GPUs
    elig = np.array([[0b100, 0b110, 0, 0]], np.uint16)
    assert policies.static_mapping(hints, SCORES, elig).tolist() == [[2, 1, 0, 1]]


def test_static_policy_matches_masked_argmin():
    """numpy.argmin (first occurrence) over the score row with ineligible devices at +inf."""
    rng = np.random.default_rng(5)
    for _ in range(200):
        E, Q, D, C = (int(rng.integers(1, 5)), int(rng.integers(1, 7)), int(rng.integers(1, 9)),
                      int(rng.integers(1, 5)))
        score = rng.integers(0, 4, size=(C, D)).astype(np.uint64)  # many equal scores
        hints = rng.integers(0, C, size=(E, Q)).astype(np.uint8)
        elig = rng.integers(0, 1 << D, size=(E, Q)).astype(np.uint16)
        elig[elig == 0] = 0  # 0 = any device
        got = policies.static_mapping(hints, score, elig)
        for e in range(E):
            for q in range(Q):
                row = score[hints[e, q]].astype(np.float64)
                m = int(elig[e, q])
                if m:
                    row = np.where([(m >> d) & 1 for d in range(D)], row, np.inf)
                assert got[e, q] == int(np.argmin(row))


def test_round_robin():
    assert policies.round_robin_mapping(2, 5, 3).tolist() == [[0, 1, 2, 0, 1]] * 2
