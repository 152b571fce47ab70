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
