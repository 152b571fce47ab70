"""Pins for the CPU oracle (oracle/): it is checked against things other than itself.

Runs on CPU only (-m "not gpu"). See DESIGN.md "Pins" for which plausible oracle mistake
each test is there to catch.
"""
from __future__ import annotations

import itertools
import json
import os

import numpy as np
import pytest

import oracle
from oracle.tiny import tiny_map
from paper_conf_cluster_ajipbf15_b200 import workloads
from pins import all_equal_closed_form, load_vector_dp, lower_bounds, subset_sum_two_identical

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _hand_cases():
    with open(os.path.join(GOLDEN, "hand_cases.json")) as f:
        return json.load(f)["cases"]


@pytest.mark.parametrize("case", _hand_cases(), ids=lambda c: c["name"])
def test_hand_cases(case):
    """SURVEY.md Appendix A, re-derived by hand (DESIGN.md Pins P1)."""
    K = np.array(case["K"], dtype=np.uint64)
    X = np.array(case["X"], dtype=np.uint64)
    idx, ms, mp = oracle.oracle_map(K, X, threads=2)
    assert int(idx[0]) == case["index"]
    assert int(ms[0]) == case["makespan"]
    assert list(mp[0]) == case["mapping"]
    Q, D = K.shape
    if "all_scores" in case:
        for m, want in enumerate(case["all_scores"]):
            tup = np.unravel_index(m, (D,) * Q)
            assert oracle.oracle_score(K, X, tup) == want
    for s in case.get("schedules", []):
        assert int(np.ravel_multi_index(s["mapping"], (D,) * Q)) == s["index"]
        assert oracle.oracle_score(K, X, s["mapping"]) == s["makespan"]
        assert int(ms[0]) <= s["makespan"]  # the optimum bounds every manual schedule
    # the definitional oracle agrees too
    t_idx, t_ms, t_map = tiny_map(K, X)
    assert (t_idx, t_ms, list(t_map)) == (case["index"], case["makespan"], case["mapping"])


def test_fig9_ratios():
    """column-major worst/best = 2.7x, row-major (C,C)/best = 2.3x."""
    cases = {c["name"]: c for c in _hand_cases()}
    col, row = cases["D-col"], cases["D-row"]
    assert max(col["all_scores"]) * 10 == 27 * col["makespan"]
    assert row["all_scores"][0] * 10 == 23 * row["makespan"]
    # Fig. 9 enumerates exactly 3^2 = 9 mappings (L2181, L2229-2233)
    assert len(col["all_scores"]) == 9 == len(list(itertools.product(range(3), repeat=2)))


def test_index_convention_is_c_order():
    """Queue 0 is the most significant base-D digit (numpy C order); a reversed digit order
    gives index 2 instead of 1 on case A."""
    K = np.array([[3, 5], [4, 2]], dtype=np.uint64)
    idx, _, mp = oracle.oracle_map(K, np.zeros_like(K))
    assert int(idx[0]) == int(np.ravel_multi_index(tuple(mp[0]), (2, 2))) == 1
    # asymmetric 3 queues x 2 devices where only mapping (1,0,0) is optimal
    K = np.array([[50, 1], [1, 50], [1, 50]], dtype=np.uint64)
    idx, ms, mp = oracle.oracle_map(K, np.zeros_like(K))
    assert list(mp[0]) == [1, 0, 0] and int(idx[0]) == 4 and int(ms[0]) == 2


@pytest.mark.parametrize("Q,D", [(1, 1), (5, 1), (1, 5), (1, 16), (7, 1)])
def test_closed_forms_d1_q1(Q, D):
    K, X = workloads.random_tables(11 + Q * 17 + D, 1, Q, D, hi=1 << 30, x_cpu_zero=False)
    idx, ms, mp = oracle.oracle_map(K, X)
    C = K[0].astype(object) + X[0].astype(object)
    if D == 1:
        assert int(idx[0]) == 0 and int(ms[0]) == sum(int(v) for v in C[:, 0])
    if Q == 1:
        assert int(idx[0]) == int(np.argmin(C[0].astype(np.int64))) and int(ms[0]) == min(C[0])


@pytest.mark.parametrize("Q,D,c", [(4, 3, 7), (8, 4, 5), (5, 3, 1), (6, 4, 9), (3, 5, 2), (9, 2, 3)])
def test_all_equal_closed_form(Q, D, c):
    K = np.full((Q, D), c, dtype=np.uint64)
    X = np.zeros_like(K)
    idx, ms, mp = oracle.oracle_map(K, X)
    want_idx, want_ms, want_tup = all_equal_closed_form(Q, D, c)
    assert (int(idx[0]), int(ms[0]), tuple(mp[0])) == (want_idx, want_ms, want_tup)


@pytest.mark.parametrize("seed", range(40))
def test_two_identical_devices_subset_sum(seed):
    rng = np.random.default_rng(1000 + seed)
    Q = int(rng.integers(1, 13))
    w = rng.integers(0, 200, size=Q, dtype=np.uint64)
    # split each w_q as K + X arbitrarily so the transfer term must be included
    k = (w * rng.integers(0, 3, size=Q, dtype=np.uint64)) // 2
    K = np.stack([k, k], axis=1)
    X = np.stack([w - k, w - k], axis=1)
    _, ms, _ = oracle.oracle_map(K, X)
    assert int(ms[0]) == subset_sum_two_identical(w)


@pytest.mark.parametrize("seed", range(60))
def test_load_vector_dp(seed):
    rng = np.random.default_rng(2000 + seed)
    Q = int(rng.integers(1, 9))
    D = int(rng.integers(1, 4))
    K = rng.integers(0, 20, size=(Q, D), dtype=np.uint64)
    X = rng.integers(0, 20, size=(Q, D), dtype=np.uint64)
    _, ms, _ = oracle.oracle_map(K, X)
    assert int(ms[0]) == load_vector_dp((K + X).tolist())


def test_transfer_term_matters():
    """X alone decides: with K = 0 the result equals the K-only run on X (and vice versa);
    swapping K and X gives the same result (the aggregate is a sum)."""
    K, X = workloads.random_tables(5, 4, 6, 3)
    a = oracle.oracle_map(K, X)
    b = oracle.oracle_map(X, K)
    c = oracle.oracle_map(K + X, np.zeros_like(K))
    d = oracle.oracle_map(np.zeros_like(K), K + X)
    for r in (b, c, d):
        assert (a[0] == r[0]).all() and (a[1] == r[1]).all()
    only_x = oracle.oracle_map(np.zeros_like(K), X)
    only_k = oracle.oracle_map(K, np.zeros_like(X))
    assert not ((only_x[1] == a[1]).all() and (only_k[1] == a[1]).all())


@pytest.mark.parametrize("seed", range(20))
def test_bounds(seed):
    """lower: ceil(sum min / D), max min; upper: every single-device mapping, the
    round-robin mapping and sum_q min_d C."""
    K, X = workloads.random_tables(3000 + seed, 1, 7, 3, hi=1 << 16)
    idx, ms, mp = oracle.oracle_map(K, X)
    C = (K[0] + X[0]).astype(np.int64)
    Q, D = C.shape
    lb1, lb2 = lower_bounds(C)
    m = int(ms[0])
    assert m >= lb1 and m >= lb2
    for d in range(D):
        assert m <= int(C[:, d].sum())
    assert m <= int(C.min(axis=1).sum())
    rr = [q % D for q in range(Q)]
    assert m <= oracle.oracle_score(K[0], X[0], rr)
    assert oracle.oracle_score(K[0], X[0], mp[0]) == m


@pytest.mark.parametrize("seed", range(10))
def test_metamorphic(seed):
    rng = np.random.default_rng(4000 + seed)
    Q, D = int(rng.integers(2, 7)), int(rng.integers(2, 5))
    K, X = workloads.random_tables(4100 + seed, 1, Q, D, hi=1 << 12)
    idx, ms, mp = oracle.oracle_map(K, X)
    # scale by k: same index, makespan * k
    k = int(rng.integers(2, 9))
    i2, m2, _ = oracle.oracle_map(K * np.uint64(k), X * np.uint64(k))
    assert int(i2[0]) == int(idx[0]) and int(m2[0]) == k * int(ms[0])
    # permute devices: same optimal makespan
    perm = rng.permutation(D)
    _, m3, _ = oracle.oracle_map(K[:, :, perm], X[:, :, perm])
    assert int(m3[0]) == int(ms[0])
    # permute queues: same optimal makespan
    qp = rng.permutation(Q)
    _, m4, _ = oracle.oracle_map(K[:, qp, :], X[:, qp, :])
    assert int(m4[0]) == int(ms[0])
    # append an all-zero queue last: index * D, same makespan
    Kz = np.concatenate([K, np.zeros((1, 1, D), np.uint64)], axis=1)
    Xz = np.concatenate([X, np.zeros((1, 1, D), np.uint64)], axis=1)
    i5, m5, _ = oracle.oracle_map(Kz, Xz)
    assert int(i5[0]) == int(idx[0]) * D and int(m5[0]) == int(ms[0])


def test_batched_equals_single_and_permutes():
    K, X = workloads.random_tables(77, 25, 5, 3, hi=64)
    bi, bm, bp = oracle.oracle_map(K, X, threads=3)
    for e in range(25):
        si, sm, sp = oracle.oracle_map(K[e], X[e], threads=2)
        assert bi[e] == si[0] and bm[e] == sm[0] and (bp[e] == sp[0]).all()
    perm = np.random.default_rng(1).permutation(25)
    pi, pm, _ = oracle.oracle_map(K[perm], X[perm])
    assert (pi == bi[perm]).all() and (pm == bm[perm]).all()


@pytest.mark.parametrize("threads", [1, 2, 3, 5, 8])
def test_thread_split_invariance(threads):
    K, X = workloads.small_int_tables(8, 1, 9, 3, hi=4)  # heavy ties
    ref = oracle.oracle_map(K, X, threads=1)
    got = oracle.oracle_map(K, X, threads=threads)
    assert all((a == b).all() for a, b in zip(ref, got))


def test_subrange_merge():
    """min over shards [r*N/G, (r+1)*N/G) by (makespan, index) == full search."""
    K, X = workloads.small_int_tables(9, 1, 8, 3, hi=6)
    N = 3**8
    full = oracle.oracle_map(K, X)
    for G in (2, 3, 4, 7):
        best = None
        for r in range(G):
            lo, hi = r * N // G, (r + 1) * N // G
            i, m, _ = oracle.oracle_map(K, X, lo=lo, hi=hi)
            assert lo <= int(i[0]) < hi
            cand = (int(m[0]), int(i[0]))
            best = cand if best is None or cand < best else best
        assert best == (int(full[1][0]), int(full[0][0]))


def test_c_oracle_matches_definitional_oracle():
    """The pthread C brute force == itertools.product + min on random tiny instances,
    including many ties (small value ranges)."""
    rng = np.random.default_rng(5)
    n = 0
    for Q in range(1, 7):
        for D in range(1, 5):
            if D**Q > 4096:
                continue
            E = 40 if D**Q <= 256 else 8
            for hi in (3, 1 << 10):
                K = rng.integers(0, hi, size=(E, Q, D), dtype=np.uint64)
                X = rng.integers(0, hi, size=(E, Q, D), dtype=np.uint64)
                ci, cm, cp = oracle.oracle_map(K, X, threads=4)
                for e in range(E):
                    ti, tm, tp = tiny_map(K[e], X[e])
                    assert (int(ci[e]), int(cm[e]), tuple(cp[e])) == (ti, tm, tp)
                    n += 1
    assert n > 1000


def test_c_oracle_matches_tiny_on_10k_instances():
    """the C oracle equals tiny.py (itertools.product + min) on 10^4
    random cfg1-sized instances (Q <= 4, D <= 3, up to 81 mappings), a third of them with
    costs in {0, 1, 2} (heavy ties), all in one batched oracle call."""
    rng = np.random.default_rng(10_000)
    n = 0
    for Q, D in ((4, 3), (3, 3), (4, 2), (2, 3)):
        E = 2500
        hi = np.where(np.arange(E) % 3 == 0, 3, 1 << 30)[:, None, None]
        K = (rng.random((E, Q, D)) * hi).astype(np.uint64)
        X = (rng.random((E, Q, D)) * hi).astype(np.uint64)
        ci, cm, cp = oracle.oracle_map(K, X)
        for e in range(E):
            assert (int(ci[e]), int(cm[e]), tuple(cp[e])) == tiny_map(K[e], X[e]), (Q, D, e)
            n += 1
    assert n == 10_000


def test_error_conventions():
    K = np.zeros((1, 3, 2), np.uint64)
    with pytest.raises(oracle.OracleError) as e:
        oracle.oracle_map(K + np.uint64(1 << 48), K)
    assert e.value.code == -2
    with pytest.raises(oracle.OracleError) as e:
        oracle.oracle_map(np.zeros((1, 13, 16), np.uint64), np.zeros((1, 13, 16), np.uint64))
    assert e.value.code == -2  # 16^13 = 2^52 > 2^48
    with pytest.raises(oracle.OracleError) as e:
        oracle.oracle_map(np.zeros((1, 2, 17), np.uint64), np.zeros((1, 2, 17), np.uint64))
    assert e.value.code == -1


def test_cfg1_npb_outcomes():
    """Qualitative Fig. 5 outcomes on the SNU-NPB-like cfg1 tables:
    EP goes to the GPUs only; BT and MG keep at least half the queues on the CPU."""
    for name in workloads.NPB_RATIO:
        K, X = workloads.cfg1_npb(name)
        _, ms, mp = oracle.oracle_map(K, X)
        if name == "EP":
            assert (mp[0] != 0).all()
        if name in ("BT", "MG"):
            assert (mp[0] == 0).sum() >= 2
