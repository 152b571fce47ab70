"""Pins for the cost-table construction oracle (NEXT-1, oracle/costs.c). CPU only."""
from __future__ import annotations

import math

import numpy as np
import pytest

import oracle
from paper_conf_cluster_ajipbf15_b200 import workloads


def model_one(Q=2, D=3, E=1, **over):
    """A tiny hand-made model: constant 4 bytes/ns H2D and 2 bytes/ns D2H curves."""
    m = dict(profile=np.array([[100, 10, 20], [7, 700, 70], [1, 2, 3]], np.uint64),
             offsets=np.array([0, 1, 3], np.uint64), kernel_ids=np.array([0, 1, 1], np.uint32),
             bytes=np.array([[4096, 1000]], np.uint64), source=np.array([[-1, 1]], np.int32),
             cached=None, sizes=np.array([1024, 1 << 20], np.uint64),
             h2d_bw=np.full((D, 2), 4.0), d2h_bw=np.full((D, 2), 2.0), host_shared=0)
    m.update(over)
    return m


def test_kernel_sums_are_multiset_sums():
    K, X = oracle.oracle_build_costs(2, 3, model_one())
    assert list(K[0, 0]) == [100, 10, 20]            # one invocation of kernel 0
    assert list(K[0, 1]) == [14, 1400, 140]          # kernel 1 invoked twice: counted twice


def test_transfer_closed_forms():
    K, X = oracle.oracle_build_costs(2, 3, model_one())
    # queue 0: data in host memory -> every device pays ceil(4096 / 4) = 1024 ns of H2D
    assert list(X[0, 0]) == [1024, 1024, 1024]
    # queue 1: data on device 1 -> device 1 pays nothing, the others D2H + H2D via the host
    assert list(X[0, 1]) == [math.ceil(1000 / 2) + math.ceil(1000 / 4), 0, 500 + 250]
    # a CPU device on host memory (host_shared bit 0) has no H2D / D2H leg
    K, X = oracle.oracle_build_costs(2, 3, model_one(host_shared=1))
    assert list(X[0, 0]) == [0, 1024, 1024] and list(X[0, 1]) == [500, 0, 750]
    # data already cached on a device: no transfer there
    K, X = oracle.oracle_build_costs(2, 3, model_one(cached=np.array([[0b100, 0b001]], np.uint16)))
    assert list(X[0, 0]) == [1024, 1024, 0] and list(X[0, 1]) == [0, 0, 750]


def test_interpolation_points_midpoints_and_clamping():
    """At a sample size the curve's own value is used; at the arithmetic midpoint of two
    sizes, the mean of their bandwidths; outside the sampled range, the end values."""
    sizes = np.array([1024, 3072, 5120], np.uint64)
    h2d = np.array([[1.0, 2.0, 8.0]])
    base = dict(profile=np.zeros((1, 1), np.uint64), offsets=np.array([0, 0], np.uint64),
                kernel_ids=np.zeros(0, np.uint32), source=np.array([[-1]], np.int32), cached=None,
                sizes=sizes, h2d_bw=h2d, d2h_bw=h2d, host_shared=0)
    for nbytes, bw in ((3072, 2.0), (1024, 1.0), (2048, 1.5), (4096, 5.0), (100, 1.0), (10**7, 8.0)):
        _, X = oracle.oracle_build_costs(1, 1, dict(base, bytes=np.array([[nbytes]], np.uint64)))
        assert int(X[0, 0, 0]) == math.ceil(nbytes / bw), nbytes
    # zero bytes move for free
    _, X = oracle.oracle_build_costs(1, 1, dict(base, bytes=np.array([[0]], np.uint64)))
    assert int(X[0, 0, 0]) == 0


@pytest.mark.parametrize("seed", range(5))
def test_device_to_device_is_d2h_plus_h2d(seed):
    """Moving data from GPU s costs the host->d leg plus one D2H leg that does not depend on
    the destination (L1293-1301: D2D as a D2H-H2D double operation)."""
    Q, D, E = 6, 5, 20
    m = workloads.cost_model(100 + seed, E, Q, D)
    m["cached"] = None
    m["host_shared"] = 0
    K, Xs = oracle.oracle_build_costs(Q, D, m)
    m_host = dict(m, source=np.full((E, Q), -1, np.int32))
    _, Xh = oracle.oracle_build_costs(Q, D, m_host)
    for e in range(E):
        for q in range(Q):
            s = int(m["source"][e, q])
            if s < 0:
                assert (Xs[e, q] == Xh[e, q]).all()
                continue
            legs = {int(Xs[e, q, d]) - int(Xh[e, q, d]) for d in range(D) if d != s}
            assert len(legs) == 1 and legs.pop() > 0 and Xs[e, q, s] == 0


@pytest.mark.parametrize("seed", range(5))
def test_monotone_in_bytes_and_kernels(seed):
    """More bytes never cost less to move (the curves are increasing with bytes/ns per
    byte... checked on the generated latency-bound curves), and adding an invocation adds
    exactly that kernel's profile row."""
    Q, D, E = 4, 3, 10
    m = workloads.cost_model(200 + seed, E, Q, D, cached_frac=0.0)
    K, X = oracle.oracle_build_costs(Q, D, m)
    m2 = dict(m, bytes=m["bytes"] * np.uint64(2))
    _, X2 = oracle.oracle_build_costs(Q, D, m2)
    assert (X2 >= X).all()
    # append kernel 3 to (e=0, q=0)
    off = m["offsets"].copy()
    off[1:] += np.uint64(1)
    ids = np.concatenate([m["kernel_ids"][:int(m["offsets"][1])], np.array([3], np.uint32),
                          m["kernel_ids"][int(m["offsets"][1]):]])
    K3, _ = oracle.oracle_build_costs(Q, D, dict(m, offsets=off, kernel_ids=ids))
    assert (K3[0, 0] == K[0, 0] + m["profile"][3]).all()
    assert (K3[1:] == K[1:]).all() and (K3[0, 1:] == K[0, 1:]).all()


def test_errors():
    with pytest.raises(oracle.OracleError):
        oracle.oracle_build_costs(2, 3, model_one(kernel_ids=np.array([0, 1, 9], np.uint32)))
    with pytest.raises(oracle.OracleError):
        oracle.oracle_build_costs(2, 3, model_one(source=np.array([[-1, 3]], np.int32)))
    with pytest.raises(oracle.OracleError):
        oracle.oracle_build_costs(2, 3, model_one(sizes=np.array([5, 5], np.uint64)))


# ------------------------------------------- per-socket curves (R19) and range (R10) ---
def model_two_sockets(**over):
    """model_one on a two-socket host: socket 0 keeps 4 / 2 bytes/ns (H2D / D2H), socket 1 is
    the far socket at 1 / 0.5 bytes/ns (the GPUs have affinity to one
    socket, so the host thread's socket changes the transfer cost)."""
    h2d = np.stack([np.full((3, 2), 4.0), np.full((3, 2), 1.0)])
    d2h = np.stack([np.full((3, 2), 2.0), np.full((3, 2), 0.5)])
    return model_one(h2d_bw=h2d, d2h_bw=d2h, **over)


def test_socket_curves_closed_forms():
    hs = np.array([[1, 1]], np.uint8)
    K, X = oracle.oracle_build_costs(2, 3, model_two_sockets(host_socket=hs))
    assert list(X[0, 0]) == [4096, 4096, 4096]                  # H2D from socket 1: 4096 / 1
    assert list(X[0, 1]) == [2000 + 1000, 0, 2000 + 1000]        # D2H + H2D both via socket 1
    K0, X0 = oracle.oracle_build_costs(2, 3, model_two_sockets(host_socket=np.zeros((1, 2), np.uint8)))
    K1, X1 = oracle.oracle_build_costs(2, 3, model_one())
    assert (X0 == X1).all() and (K0 == K1).all() and (K == K1).all()  # socket 0 = the plain model
    # mixed: queue 0 near, queue 1 far
    _, Xm = oracle.oracle_build_costs(2, 3, model_two_sockets(host_socket=np.array([[0, 1]], np.uint8)))
    assert list(Xm[0, 0]) == [1024, 1024, 1024] and list(Xm[0, 1]) == [3000, 0, 3000]


def test_one_socket_axis_is_the_plain_model():
    m = workloads.cost_model(7, 30, 5, 4)
    K, X = oracle.oracle_build_costs(5, 4, m)
    m3 = dict(m, h2d_bw=m["h2d_bw"][None], d2h_bw=m["d2h_bw"][None], host_socket=np.zeros((30, 5), np.uint8))
    K3, X3 = oracle.oracle_build_costs(5, 4, m3)
    assert (K == K3).all() and (X == X3).all()


@pytest.mark.parametrize("seed", range(4))
def test_socket_relabeling_invariance(seed):
    """Permuting the sockets (their curves and every queue's label alike) changes nothing."""
    rng = np.random.default_rng(seed)
    E, Q, D, S = 12, 4, 3, 3
    m = workloads.cost_model(300 + seed, E, Q, D)
    h2d = np.stack([m["h2d_bw"] * f for f in (1.0, 0.5, 0.25)])
    d2h = np.stack([m["d2h_bw"] * f for f in (1.0, 0.7, 0.3)])
    hs = rng.integers(0, S, size=(E, Q)).astype(np.uint8)
    K, X = oracle.oracle_build_costs(Q, D, dict(m, h2d_bw=h2d, d2h_bw=d2h, host_socket=hs))
    perm = rng.permutation(S)            # new socket i = old socket perm[i]
    inv = np.argsort(perm)
    Kp, Xp = oracle.oracle_build_costs(Q, D, dict(m, h2d_bw=h2d[perm], d2h_bw=d2h[perm],
                                                  host_socket=inv[hs].astype(np.uint8)))
    assert (K == Kp).all() and (X == Xp).all()
    # a slower socket never costs less
    _, Xs = oracle.oracle_build_costs(Q, D, dict(m, h2d_bw=h2d, d2h_bw=d2h, host_socket=np.full((E, Q), 2, np.uint8)))
    _, Xf = oracle.oracle_build_costs(Q, D, dict(m, h2d_bw=h2d, d2h_bw=d2h, host_socket=np.zeros((E, Q), np.uint8)))
    assert (Xs >= Xf).all() and (Xs > Xf).any()


def test_profile_and_sum_range():
    """Entries must be < 2^48 and a kernel sum that reaches 2^48 is out of range (checked as
    it grows, so it can never wrap around to a small accepted value)."""
    big = np.array([[1 << 47, 1, 1], [(1 << 47) - 1, 1, 1], [1 << 48, 1, 1]], np.uint64)
    ok = model_one(profile=big, offsets=np.array([0, 1, 2], np.uint64), kernel_ids=np.array([0, 1], np.uint32))
    K, _ = oracle.oracle_build_costs(2, 3, dict(ok, profile=big[:2]))
    assert int(K[0, 0, 0]) == 1 << 47
    two = dict(ok, profile=big[:2], offsets=np.array([0, 2, 2], np.uint64), kernel_ids=np.array([0, 1], np.uint32))
    K, _ = oracle.oracle_build_costs(2, 3, two)          # 2^47 + 2^47 - 1 = 2^48 - 1: fine
    assert int(K[0, 0, 0]) == (1 << 48) - 1
    with pytest.raises(oracle.OracleError):             # 2^47 + 2^47 = 2^48
        oracle.oracle_build_costs(2, 3, dict(two, kernel_ids=np.array([0, 0], np.uint32)))
    with pytest.raises(oracle.OracleError):             # an entry of 2^48, even if never invoked
        oracle.oracle_build_costs(2, 3, dict(ok, kernel_ids=np.array([0, 1], np.uint32)))
    many = dict(ok, profile=big[:2], offsets=np.array([0, 70000, 70000], np.uint64),
                kernel_ids=np.zeros(70000, np.uint32))   # 70000 x 2^47 would wrap a u64 sum
    with pytest.raises(oracle.OracleError):
        oracle.oracle_build_costs(2, 3, many)


def test_socket_out_of_range():
    with pytest.raises(oracle.OracleError):
        oracle.oracle_build_costs(2, 3, model_two_sockets(host_socket=np.array([[0, 2]], np.uint8)))
