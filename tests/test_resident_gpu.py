"""GPU parity of the resident mapper (include/mcl.h mcl_resident_*): one warp resident on
the device serving decisions from a pinned host mailbox, against the CPU oracle, bit-exact
(index, makespan, mapping) -- cfg1's shape and every other shape the mode accepts
(D^Q <= 8192, incl. the paper's FT-sized 8 x 3 decision), tie-heavy tables, back-to-back calls, the idle exit and relaunch, and the
error cases."""
from __future__ import annotations

import time

import numpy as np
import pytest

import oracle
from conftest import cuda_available
from paper_conf_cluster_ajipbf15_b200 import workloads
from paper_conf_cluster_ajipbf15_b200.mcl import MCL_E_INVAL, MCL_E_RANGE, Mapper, MclError

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def torch_cuda():
    if not cuda_available():
        pytest.fail("no CUDA device: the -m gpu tests must run on a GPU box")
    import torch

    return torch


def check(got, K, X, ctx=""):
    gi, gmp, gms = got
    wi, wms, wmp = oracle.oracle_map(K, X)
    bad = np.nonzero((gi != wi) | (gms != wms))[0]
    assert bad.size == 0, f"{ctx}: {bad.size} epochs differ, first {bad[:5]}"
    assert (gmp == wmp).all(), ctx


SHAPES = [(1, 1), (1, 5), (2, 2), (3, 4), (4, 3), (5, 5), (6, 4), (12, 2), (3, 16), (7, 3), (16, 1), (8, 3), (13, 2)]


@pytest.mark.parametrize("Q,D", SHAPES)
def test_resident_matches_oracle(torch_cuda, Q, D):
    with Mapper(0) as m:
        m.resident_start(Q, D, max_epochs=64)
        try:
            for seed, E in ((1, 1), (2, 7), (3, 64)):
                K, X = workloads.random_tables(seed * 100 + Q * 17 + D, E, Q, D, hi=1 << 20)
                check(m.resident_map(K, X), K, X, f"random Q={Q} D={D} E={E}")
                K, X = workloads.small_int_tables(seed * 100 + Q * 17 + D, E, Q, D, hi=3)
                check(m.resident_map(K, X), K, X, f"ties Q={Q} D={D} E={E}")
            # entries just below 2^48: makespans up to Q * 2^49
            K = np.full((2, Q, D), (1 << 48) - 1, np.uint64)
            X = np.zeros_like(K)
            X[1, :, 0] = 1 << 40
            K[1] -= 5
            check(m.resident_map(K, X), K, X, "top of range")
        finally:
            m.resident_stop()


def test_resident_cfg1_back_to_back(torch_cuda):
    """cfg1's shape, 2000 consecutive decisions on one resident warp (request numbers
    advance by one per call), each checked; pinned and pageable host buffers."""
    torch = torch_cuda
    K, X = workloads.random_tables(7, 2000, 4, 3, hi=1 << 30)
    want = oracle.oracle_map(K, X)
    Kp = torch.from_numpy(K).pin_memory()
    Xp = torch.from_numpy(X).pin_memory()
    with Mapper(0) as m:
        m.resident_start(4, 3)
        try:
            for e in range(K.shape[0]):
                src = (Kp[e], Xp[e]) if e % 2 else (K[e], X[e])
                gi, gmp, gms = m.resident_map(*src)
                assert gi[0] == want[0][e] and gms[0] == want[1][e] and (gmp[0] == want[2][e]).all(), e
        finally:
            m.resident_stop()


def test_resident_idle_exit_and_relaunch(torch_cuda):
    """With a 5 ms idle limit the warp exits between calls; the next call relaunches it
    and still answers correctly. Device-wide synchronisation completes once it has exited."""
    torch = torch_cuda
    K, X = workloads.random_tables(11, 3, 4, 3, hi=1 << 16)
    with Mapper(0) as m:
        m.resident_start(4, 3, max_epochs=3, idle_ms=5)
        try:
            for _ in range(4):
                check(m.resident_map(K, X), K, X, "after idle exit")
                time.sleep(0.03)
            torch.cuda.synchronize()  # the warp has exited idle: returns
            check(m.resident_map(K, X), K, X, "after a device sync")
        finally:
            m.resident_stop()
        m.resident_start(4, 3)  # start again on the same handle
        check(m.resident_map(K[:1], X[:1]), K[:1], X[:1], "restarted")
        # the handle's ordinary path still works beside a stopped resident mapper
        m.resident_stop()
        gi, gmp, gms = m.map_queues(K, X)
        check((gi, gmp, gms), K, X, "map_queues")


def test_resident_errors(torch_cuda):
    torch = torch_cuda
    with Mapper(0) as m:
        with pytest.raises(MclError) as ei:
            m.resident_start(14, 2)  # 2^14 > 8192
        assert ei.value.status == MCL_E_INVAL
        with pytest.raises(MclError):
            m.resident_start(4, 17)
        with pytest.raises(MclError):
            m.resident_start(4, 3, max_epochs=65)
        K, X = workloads.random_tables(3, 4, 4, 3, hi=100)
        with pytest.raises(MclError):
            m.resident_map(K, X)  # not started
        m.resident_start(4, 3, max_epochs=2)
        try:
            with pytest.raises(MclError) as ei:
                m.resident_map(K, X)  # 4 epochs > max_epochs
            assert ei.value.status == MCL_E_INVAL
            with pytest.raises(ValueError):
                m.resident_map(K[:, :3], X[:, :3])  # wrong Q
            Kd = torch.from_numpy(K[:1]).cuda()
            with pytest.raises(MclError) as ei:
                m.resident_map(Kd, torch.from_numpy(X[:1]).cuda())  # device buffers
            assert ei.value.status == MCL_E_INVAL
            Kr = K[:1].copy()
            Kr[0, 2, 1] = 1 << 48
            with pytest.raises(MclError) as ei:
                m.resident_map(Kr, X[:1])
            assert ei.value.status == MCL_E_RANGE
            check(m.resident_map(K[:2], X[:2]), K[:2], X[:2], "after errors")
            with pytest.raises(MclError):
                m.resident_start(4, 3)  # already started
        finally:
            m.resident_stop()


def test_resident_close_without_stop(torch_cuda):
    """Closing the handle while the warp is resident stops it (mcl_mapper_destroy); device-
    wide synchronisation afterwards returns at once."""
    torch = torch_cuda
    K, X = workloads.random_tables(13, 2, 4, 3, hi=1 << 16)
    m = Mapper(0)
    m.resident_start(4, 3, max_epochs=2, idle_ms=60000)
    check(m.resident_map(K, X), K, X, "before close")
    m.close()
    t0 = time.perf_counter()
    torch.cuda.synchronize()
    assert time.perf_counter() - t0 < 5.0


def test_resident_beside_searches(torch_cuda):
    """A resident warp and the handle's ordinary searches at the same time: decisions through
    the mailbox between (and during) full-GPU searches on the handle's stream, all exact."""
    torch = torch_cuda
    Kb, Xb = workloads.random_tables(21, 1, 10, 6, hi=1 << 20)  # 6^10 = 6e7 mappings
    want_b = oracle.oracle_map(Kb, Xb)
    Ks, Xs = workloads.random_tables(22, 50, 4, 3, hi=1 << 16)
    want_s = oracle.oracle_map(Ks, Xs)
    Kd, Xd = torch.from_numpy(Kb).cuda(), torch.from_numpy(Xb).cuda()
    with Mapper(0) as m, Mapper(0) as r:
        r.resident_start(4, 3)
        try:
            for e in range(Ks.shape[0]):
                gi, gmp, gms = m.map_queues(Kd, Xd)
                assert int(gi[0]) == want_b[0][0] and int(gms[0]) == want_b[1][0]
                ri, rmp, rms = r.resident_map(Ks[e], Xs[e])
                assert ri[0] == want_s[0][e] and rms[0] == want_s[1][e] and (rmp[0] == want_s[2][e]).all()
        finally:
            r.resident_stop()
