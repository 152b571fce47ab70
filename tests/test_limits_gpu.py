"""Boundary sizes through the C ABI on the GPU: the largest index space (D^Q = 2^48), the
largest Q and D, epoch counts beyond one grid dimension, and randomized fuzz over every
kernel path. Results are checked against the oracle where it can enumerate, and against
properties that hold at any size where it cannot."""
from __future__ import annotations

import numpy as np
import pytest

import oracle
from conftest import cuda_available
from paper_conf_cluster_ajipbf15_b200 import workloads
from paper_conf_cluster_ajipbf15_b200.mcl import MCL_E_RANGE, Mapper, MclError

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


def dev(torch, a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def test_largest_index_space_2_pow_48(torch_cuda, mapper):
    """16^12 = 2^48 mappings is accepted (solved by the pruned search); 16^12 * ... > 2^48
    is rejected. The returned mapping re-scores to the returned makespan and respects the
    lower bounds; shard-style spot checks compare it with the exhaustive kernel on the
    sub-range that contains it."""
    torch = torch_cuda
    K, X = workloads.random_tables(48, 1, 12, 16, hi=1 << 24)
    i, mp, ms = mapper.map_queues_pruned(dev(torch, K), dev(torch, X))
    i, mp, ms = int(i[0]), mp.cpu().numpy()[0], int(ms[0])
    assert oracle.oracle_score(K[0], X[0], mp) == ms
    assert int(np.ravel_multi_index(tuple(int(v) for v in mp), (16,) * 12)) == i
    C = (K[0] + X[0]).astype(np.int64)
    assert ms >= int(C.min(axis=1).max()) and ms * 16 >= int(C.min(axis=1).sum())
    # the exhaustive GPU search on the index range around the answer agrees
    N = 16**12
    G = 1 << 15  # the largest world a handle accepts
    r = i * G // N
    with Mapper(0, rank=r, world=G) as m:
        ei, emp, ems = m.map_queues(dev(torch, K), dev(torch, X))
    assert int(ems[0]) >= ms
    if int(ems[0]) == ms:
        assert int(ei[0]) == i or int(ei[0]) > i
    with pytest.raises(MclError) as e:
        mapper.map_queues(np.zeros((1, 13, 16), np.uint64), np.zeros((1, 13, 16), np.uint64))
    assert e.value.status == MCL_E_RANGE


def test_max_queues_and_devices(torch_cuda, mapper):
    for Q, D in ((32, 1), (32, 2), (1, 16), (2, 16), (24, 2)):
        K, X = workloads.random_tables(Q * 100 + D, 2, Q, D, hi=1 << 20)
        if D**Q <= 1 << 26:
            want = oracle.oracle_map(K, X)
            i, mp, ms = mapper.map_queues(dev(torch_cuda, K), dev(torch_cuda, X))
            assert (i.cpu().numpy() == want[0]).all() and (ms.cpu().numpy() == want[1]).all()
        i2, mp2, ms2 = mapper.map_queues_pruned(dev(torch_cuda, K), dev(torch_cuda, X))
        for e in range(2):
            assert oracle.oracle_score(K[e], X[e], mp2.cpu().numpy()[e]) == int(ms2[e])
        if D**Q <= 1 << 26:
            assert (ms2.cpu().numpy() == want[1]).all() and (i2.cpu().numpy() == want[0]).all()


def test_epochs_beyond_one_grid_dimension(torch_cuda, mapper):
    """70,000 epochs (more than 65,535 CTAs in one grid dimension) on the blocked and
    generic kernels; 3 x 10^6 small epochs on the batched small kernel."""
    K, X = workloads.random_tables(7, 70_000, 3, 3, hi=1 << 16)
    want = oracle.oracle_map(K, X)
    for p in (1, 3):
        mapper.force_path(p)
        try:
            i, mp, ms = mapper.map_queues(dev(torch_cuda, K), dev(torch_cuda, X))
        finally:
            mapper.force_path(0)
        assert (i.cpu().numpy() == want[0]).all() and (ms.cpu().numpy() == want[1]).all(), p
    K, X = workloads.cfg3(E=3_000_000, seed=13)
    want = oracle.oracle_map(K, X)
    i, mp, ms = mapper.map_queues(dev(torch_cuda, K), dev(torch_cuda, X))
    assert (i.cpu().numpy() == want[0]).all() and (ms.cpu().numpy() == want[1]).all()


@pytest.mark.parametrize("seed", range(6))
def test_fuzz_every_path(torch_cuda, mapper, seed):
    """Random shapes, value ranges and batch sizes through every applicable path."""
    rng = np.random.default_rng(9000 + seed)
    for _ in range(8):
        D = int(rng.integers(1, 9))
        Q = int(rng.integers(1, 9))
        while D**Q > 2_000_000:
            Q -= 1
        E = int(rng.integers(1, 40))
        hi = int(rng.choice([4, 1 << 10, 1 << 30, 1 << 47]))
        K, X = workloads.random_tables(int(rng.integers(0, 1 << 30)), E, Q, D, hi=hi, x_cpu_zero=False)
        want = oracle.oracle_map(K, X)
        paths = [0, 3] + ([1, 2] if Q >= 3 and 2 <= D <= 8 else []) + ([5] if E > 1 and Q >= 3 and 2 <= D <= 8 and hi < (1 << 28) else [])
        for p in paths:
            mapper.force_path(p)
            try:
                i, mp, ms = mapper.map_queues(dev(torch_cuda, K), dev(torch_cuda, X))
            finally:
                mapper.force_path(0)
            ctx = f"Q={Q} D={D} E={E} hi={hi} path={p}"
            assert (i.cpu().numpy() == want[0]).all() and (ms.cpu().numpy() == want[1]).all(), ctx
            assert (mp.cpu().numpy() == want[2]).all(), ctx
        mapper.force_path(6)
        try:
            i, mp, ms = mapper.map_queues_pruned(dev(torch_cuda, K), dev(torch_cuda, X))
        finally:
            mapper.force_path(0)
        assert (i.cpu().numpy() == want[0]).all() and (ms.cpu().numpy() == want[1]).all()
        if E > 1:  # host buffers through the pipelined staging, a random chunk count
            mapper.set_pipeline_chunks(int(rng.integers(2, 6)))
            try:
                i, mp, ms = mapper.map_queues(K, X)
            finally:
                mapper.set_pipeline_chunks(0)
            ctx = f"Q={Q} D={D} E={E} hi={hi} pipelined"
            assert (i == want[0]).all() and (ms == want[1]).all() and (mp == want[2]).all(), ctx
