"""Pins for the constrained oracle (R11): per-device base loads
(queues outside the pool, SCHED_OFF: "statically mapped to the chosen device", PAPER.md
L838-845, L654-672) and per-queue eligible-device sets. CPU only."""
from __future__ import annotations

import numpy as np
import pytest

import oracle
from oracle.tiny import tiny_map_constrained
from paper_conf_cluster_ajipbf15_b200 import workloads
from pins import load_vector_dp


def _instance(seed, Q, D, hi=1 << 12, base_hi=1 << 12):
    rng = np.random.default_rng(seed)
    K, X = workloads.random_tables(seed, 1, Q, D, hi=hi)
    base = rng.integers(0, base_hi, size=(1, D), dtype=np.uint64)
    elig = rng.integers(0, 1 << D, size=(1, Q), dtype=np.uint16)
    return K, X, base, elig


def test_unconstrained_is_special_case():
    K, X = workloads.random_tables(1, 20, 5, 3, hi=64)
    a = oracle.oracle_map(K, X)
    b = oracle.oracle_map_constrained(K, X, np.zeros((20, 3), np.uint64), np.zeros((20, 5), np.uint16))
    full = np.full((20, 5), 0b111, np.uint16)
    c = oracle.oracle_map_constrained(K, X, None, full)
    for r in (b, c):
        assert all((x == y).all() for x, y in zip(a, r))


@pytest.mark.parametrize("seed", range(12))
def test_constant_base_shifts_makespan(seed):
    """Adding the same load c to every device adds c to every makespan: same index."""
    K, X, _, elig = _instance(100 + seed, 5, 3)
    i0, m0, _ = oracle.oracle_map_constrained(K, X, None, elig)
    c = 12345
    i1, m1, _ = oracle.oracle_map_constrained(K, X, np.full((1, 3), c, np.uint64), elig)
    assert i1[0] == i0[0] and int(m1[0]) == int(m0[0]) + c


@pytest.mark.parametrize("seed", range(12))
def test_pinned_queue_equals_reduced_problem(seed):
    """Pinning queue q to device d == removing q and adding C[q][d] to d's base load; the
    index is the reduced problem's tuple with digit d re-inserted at position q."""
    rng = np.random.default_rng(200 + seed)
    Q, D = 6, 3
    K, X, base, _ = _instance(200 + seed, Q, D)
    q, d = int(rng.integers(0, Q)), int(rng.integers(0, D))
    elig = np.zeros((1, Q), np.uint16)
    elig[0, q] = 1 << d
    i_pin, m_pin, mp_pin = oracle.oracle_map_constrained(K, X, base, elig)
    keep = [t for t in range(Q) if t != q]
    b2 = base.copy()
    b2[0, d] += K[0, q, d] + X[0, q, d]
    i_red, m_red, mp_red = oracle.oracle_map_constrained(K[:, keep], X[:, keep], b2, None)
    assert int(m_pin[0]) == int(m_red[0])
    tup = list(mp_red[0])
    tup.insert(q, d)
    assert list(mp_pin[0]) == tup
    assert int(i_pin[0]) == int(np.ravel_multi_index(tuple(tup), (D,) * Q))


@pytest.mark.parametrize("seed", range(40))
def test_constrained_vs_load_vector_dp(seed):
    rng = np.random.default_rng(300 + seed)
    Q, D = int(rng.integers(1, 8)), int(rng.integers(1, 4))
    K, X, base, elig = _instance(300 + seed, Q, D, hi=16, base_hi=16)
    _, ms, mp = oracle.oracle_map_constrained(K, X, base, elig)
    assert int(ms[0]) == load_vector_dp((K[0] + X[0]).tolist(), base[0], elig[0])
    for qq in range(Q):  # the returned mapping respects the masks
        assert elig[0, qq] == 0 or (int(elig[0, qq]) >> int(mp[0, qq])) & 1
    assert oracle.oracle_score_base(K[0], X[0], base[0], mp[0]) == int(ms[0])


def test_c_constrained_matches_definition():
    rng = np.random.default_rng(7)
    n = 0
    for Q in range(1, 6):
        for D in range(1, 5):
            E = 30
            K = rng.integers(0, 6, size=(E, Q, D), dtype=np.uint64)
            X = rng.integers(0, 6, size=(E, Q, D), dtype=np.uint64)
            base = rng.integers(0, 8, size=(E, D), dtype=np.uint64)
            elig = rng.integers(0, 1 << D, size=(E, Q), dtype=np.uint16)
            ci, cm, cp = oracle.oracle_map_constrained(K, X, base, elig, threads=3)
            for e in range(E):
                ti, tm, tp = tiny_map_constrained(K[e], X[e], base[e], elig[e])
                assert (int(ci[e]), int(cm[e]), tuple(cp[e])) == (ti, tm, tp)
                n += 1
    assert n == 600


def test_infeasible_and_range():
    K = np.zeros((1, 3, 2), np.uint64)
    with pytest.raises(oracle.OracleError) as e:
        oracle.oracle_map_constrained(K, K, None, np.array([[0, 0b100, 0]], np.uint16))
    assert e.value.code == -1  # queue 1 may only use device 2, which does not exist
    with pytest.raises(oracle.OracleError) as e:
        oracle.oracle_map_constrained(K, K, np.array([[0, 1 << 48]], np.uint64), None)
    assert e.value.code == -2
