"""GPU parity of cost-table construction (NEXT-1) and the fused profiles -> mapping
pipeline, against oracle/costs.c and the oracle search; bit-exact."""
from __future__ import annotations

import numpy as np
import pytest

import oracle
from conftest import cuda_available
from paper_conf_cluster_ajipbf15_b200 import workloads
from paper_conf_cluster_ajipbf15_b200.mcl import MCL_E_INVAL, Mapper, MclError

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def torch_cuda():
    if not cuda_available():
        pytest.fail("no CUDA device: the -m gpu tests must run on a GPU box")
    import torch

    return torch


@pytest.fixture(scope="module")
def mapper(torch_cuda):
    m = Mapper(0)
    yield m
    m.close()


def on_device(torch, model):
    return {k: (torch.from_numpy(np.ascontiguousarray(v)).cuda() if isinstance(v, np.ndarray) else v)
            for k, v in model.items()}


@pytest.mark.parametrize("E,Q,D", [(1, 4, 3), (50, 8, 4), (333, 2, 3), (7, 12, 8), (3, 5, 16), (20, 3, 1)])
def test_build_costs_host_and_device(torch_cuda, mapper, E, Q, D):
    m = workloads.cost_model(10 * E + Q + D, E, Q, D)
    want_k, want_x = oracle.oracle_build_costs(Q, D, m)
    K, X = mapper.build_costs(m, D)  # host arrays in and out
    assert (K == want_k).all() and (X == want_x).all()
    Kd, Xd = mapper.build_costs(on_device(torch_cuda, m), D, device_out=True)
    assert (Kd.cpu().numpy() == want_k).all() and (Xd.cpu().numpy() == want_x).all()


def test_build_costs_edge_models(torch_cuda, mapper):
    E, Q, D = 40, 6, 5
    m = workloads.cost_model(3, E, Q, D)
    variants = [
        dict(m, cached=None, host_shared=0),
        dict(m, bytes=np.zeros((E, Q), np.uint64)),                        # nothing to move
        dict(m, bytes=np.full((E, Q), 1 << 40, np.uint64)),                # beyond the last sample
        dict(m, bytes=np.full((E, Q), 100, np.uint64)),                    # below the first sample
        dict(m, bytes=m["sizes"][np.arange(E * Q) % len(m["sizes"])].reshape(E, Q)),  # exactly at samples
        dict(m, offsets=np.zeros(E * Q + 1, np.uint64), kernel_ids=np.zeros(0, np.uint32)),  # no kernels
        dict(m, sizes=m["sizes"][:1], h2d_bw=m["h2d_bw"][:, :1], d2h_bw=m["d2h_bw"][:, :1]),  # one sample
        dict(m, profile=m["profile"] * np.uint64(1 << 20)),               # entries >= 2^32: 64-bit rows
    ]
    for v in variants:
        want = oracle.oracle_build_costs(Q, D, v)
        got = mapper.build_costs(v, D)
        assert (got[0] == want[0]).all() and (got[1] == want[1]).all()


def test_bad_models(torch_cuda, mapper):
    E, Q, D = 4, 3, 3
    m = workloads.cost_model(5, E, Q, D)
    bad = [
        dict(m, kernel_ids=np.full_like(m["kernel_ids"], 10_000)),
        dict(m, source=np.full((E, Q), 7, np.int32)),
        dict(m, sizes=m["sizes"][::-1].copy()),
        dict(m, h2d_bw=np.zeros_like(m["h2d_bw"])),
    ]
    for v in bad:
        with pytest.raises(MclError) as e:
            mapper.build_costs(v, D)
        assert e.value.status == MCL_E_INVAL
    # still usable afterwards
    want = oracle.oracle_build_costs(Q, D, m)
    got = mapper.build_costs(m, D)
    assert (got[0] == want[0]).all()


@pytest.mark.parametrize("E,Q,D", [(200, 8, 4), (1, 10, 4), (5000, 2, 3)])
def test_map_from_profiles(torch_cuda, mapper, E, Q, D):
    m = workloads.cost_model(77 + E, E, Q, D)
    K, X = oracle.oracle_build_costs(Q, D, m)
    want = oracle.oracle_map(K, X)
    idx, mp, ms = mapper.map_from_profiles(m, D)
    assert (idx == want[0]).all() and (ms == want[1]).all() and (mp == want[2]).all()
    base, elig = workloads.constraints(5, E, Q, D)
    want = oracle.oracle_map_constrained(K, X, base, elig)
    idx, mp, ms = mapper.map_from_profiles(on_device(torch_cuda, m), D, base, elig)
    assert (idx == want[0]).all() and (ms == want[1]).all() and (mp == want[2]).all()


def test_build_costs_many_tiles_long_lists_misaligned(torch_cuda, mapper):
    """Many tiles per persistent CTA (E x Q pairs well above 256 x the resident CTAs), tiles
    whose invocation lists are long (~25k ids per 256-pair tile), a mix of long and short
    lists in one call, and an ids array that starts 4 bytes past a 16-byte boundary."""
    torch = torch_cuda
    cases = [
        workloads.cost_model(91, 40_000, 8, 4),                     # 1250 tiles, ~8.5 ids per pair
        workloads.cost_model(92, 700, 4, 3, max_kernels=200),       # ~25k ids per tile
    ]
    mixed = workloads.cost_model(93, 3000, 4, 3)
    counts = np.diff(mixed["offsets"].astype(np.int64))
    counts[: 256 * 3] = 60                                          # the first tiles: long lists
    mixed["offsets"] = np.concatenate([[0], np.cumsum(counts)]).astype(np.uint64)
    mixed["kernel_ids"] = np.random.default_rng(4).integers(0, 64, int(counts.sum())).astype(np.uint32)
    cases.append(mixed)
    for m in cases:
        Q, D = m["bytes"].shape[1], m["profile"].shape[1]
        want_k, want_x = oracle.oracle_build_costs(Q, D, m)
        Kd, Xd = mapper.build_costs(on_device(torch, m), D, device_out=True)
        assert (Kd.cpu().numpy() == want_k).all() and (Xd.cpu().numpy() == want_x).all()
    # misaligned ids: a device view starting one element into a 16-byte-aligned allocation
    m = workloads.cost_model(94, 5000, 8, 4)
    want_k, want_x = oracle.oracle_build_costs(8, 4, m)
    dm = on_device(torch, m)
    ids = m["kernel_ids"]
    padded = torch.zeros(ids.size + 1, dtype=torch.int32, device="cuda")
    padded[1:] = torch.from_numpy(ids.view(np.int32)).cuda()
    dm["kernel_ids"] = padded[1:].view(torch.uint32)
    assert dm["kernel_ids"].data_ptr() % 16 == 4
    Kd, Xd = mapper.build_costs(dm, 4, device_out=True)
    assert (Kd.cpu().numpy() == want_k).all() and (Xd.cpu().numpy() == want_x).all()


@pytest.mark.parametrize("E,Q,D,S", [(60, 8, 4, 2), (9, 5, 3, 3), (400, 2, 3, 2), (5, 12, 8, 4)])
def test_build_costs_per_socket_curves(torch_cuda, mapper, E, Q, D, S):
    """Per (socket, device) H2D / D2H curves and each queue's host socket (PAPER.md L897-901,
    L1349-1361; reading R19): bit-exact against oracle/costs.c, host and device buffers."""
    m = workloads.cost_model(7 * E + S, E, Q, D, sockets=S)
    want_k, want_x = oracle.oracle_build_costs(Q, D, m)
    K, X = mapper.build_costs(m, D)
    assert (K == want_k).all() and (X == want_x).all()
    Kd, Xd = mapper.build_costs(on_device(torch_cuda, m), D, device_out=True)
    assert (Kd.cpu().numpy() == want_k).all() and (Xd.cpu().numpy() == want_x).all()
    # the socket matters: every queue on socket 0 gives different (never larger) X here
    m0 = dict(m, host_socket=np.zeros((E, Q), np.uint8))
    _, X0 = mapper.build_costs(m0, D)
    assert (X0 == oracle.oracle_build_costs(Q, D, m0)[1]).all() and (X0 <= X).all() and (X0 < X).any()
    # a socket axis of one with no host_socket array is the plain model
    m1 = dict(workloads.cost_model(5, E, Q, D))
    m1s = dict(m1, h2d_bw=m1["h2d_bw"][None], d2h_bw=m1["d2h_bw"][None])
    assert all((a == b).all() for a, b in zip(mapper.build_costs(m1s, D), oracle.oracle_build_costs(Q, D, m1)))
    bad = dict(m, host_socket=np.full((E, Q), S, np.uint8))
    with pytest.raises(MclError) as e:
        mapper.build_costs(bad, D)
    assert e.value.status == MCL_E_INVAL


def test_build_costs_range_is_exact(torch_cuda, mapper):
    """A profile entry of 2^48 (even never invoked) and a kernel sum reaching 2^48 are range
    errors, like the oracle's running-sum check; a list of 70000 invocations (the checked
    accumulation path) sums exactly, and 70000 x 2^47 -- which would wrap a u64 -- is a range
    error, never a small wrapped cost."""
    from paper_conf_cluster_ajipbf15_b200.mcl import MCL_E_RANGE

    D = 3
    base = dict(bytes=np.array([[4096, 1000]], np.uint64), source=np.array([[-1, 1]], np.int32),
                cached=None, sizes=np.array([1024, 1 << 20], np.uint64), h2d_bw=np.full((D, 2), 4.0),
                d2h_bw=np.full((D, 2), 2.0), host_shared=0)
    prof = np.array([[1 << 47, 1, 1], [(1 << 47) - 1, 1, 1], [3, 5, 7]], np.uint64)
    two = dict(base, profile=prof, offsets=np.array([0, 2, 2], np.uint64), kernel_ids=np.array([0, 1], np.uint32))
    K, _ = mapper.build_costs(two, D)
    assert int(K[0, 0, 0]) == (1 << 48) - 1 == int(oracle.oracle_build_costs(2, D, two)[0][0, 0, 0])
    for bad in (dict(two, kernel_ids=np.array([0, 0], np.uint32)),
                dict(two, profile=np.vstack([prof, [[1 << 48, 0, 0]]]).astype(np.uint64)),
                dict(two, offsets=np.array([0, 70000, 70000], np.uint64), kernel_ids=np.zeros(70000, np.uint32))):
        with pytest.raises(MclError) as e:
            mapper.build_costs(bad, D)
        assert e.value.status == MCL_E_RANGE
    long_ok = dict(two, offsets=np.array([0, 70000, 70001], np.uint64),
                   kernel_ids=np.concatenate([np.full(70000, 2, np.uint32), [1]]).astype(np.uint32))
    K, X = mapper.build_costs(long_ok, D)
    wk, wx = oracle.oracle_build_costs(2, D, long_ok)
    assert (K == wk).all() and (X == wx).all() and int(K[0, 0, 2]) == 7 * 70000
