"""NEXT-4: the pruned exact search returns exactly the exhaustive result (lowest-index
minimum-makespan mapping) -- checked against the oracle and the full-size goldens."""
from __future__ import annotations

import json
import os

import numpy as np
import pytest

import oracle
from conftest import cuda_available
from paper_conf_cluster_ajipbf15_b200 import workloads
from paper_conf_cluster_ajipbf15_b200.mcl import MCL_E_INVAL, Mapper, MclError

pytestmark = pytest.mark.gpu
GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


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


def pruned(torch, m, K, X, base=None, elig=None, force=True):
    """Run the branch-and-bound kernel (forced even below the small-index-space cutover,
    where mcl_map_queues_pruned would otherwise score exhaustively)."""
    m.force_path(6 if force else 0)
    try:
        i, mp, ms = m.map_queues_pruned(dev(torch, K), dev(torch, X),
                                        None if base is None else dev(torch, base),
                                        None if elig is None else dev(torch, elig))
    finally:
        m.force_path(0)
    return i.cpu().numpy(), mp.cpu().numpy(), ms.cpu().numpy()


def check(got, want, ctx):
    gi, gmp, gms = got
    wi, wms, wmp = want
    bad = np.nonzero((gi != wi) | (gms != wms))[0]
    assert bad.size == 0, f"{ctx}: {bad[:5]} gpu {gi[bad[:5]]}/{gms[bad[:5]]} oracle {wi[bad[:5]]}/{wms[bad[:5]]}"
    assert (gmp == wmp).all(), ctx


SHAPES = [(q, d) for q in range(1, 8) for d in range(1, 9) if d**q <= 300_000]


@pytest.mark.parametrize("Q,D", SHAPES)
def test_pruned_random_and_ties(torch_cuda, mapper, Q, D):
    E = 48 if D**Q <= 5000 else 8
    for seed, maker in ((20 * Q + D, workloads.random_tables), (2000 + 10 * Q + D, workloads.small_int_tables)):
        K, X = maker(seed, E, Q, D)
        check(pruned(torch_cuda, mapper, K, X), oracle.oracle_map(K, X), f"Q={Q} D={D} {maker.__name__}")
    assert mapper.launch_info()["path"] == "pruned"


@pytest.mark.parametrize("Q,D", [(4, 3), (6, 4), (5, 5), (8, 2), (3, 13), (7, 3)])
def test_pruned_constrained(torch_cuda, mapper, Q, D):
    K, X = workloads.random_tables(70 + Q * D, 20, Q, D, hi=1 << 16)
    base, elig = workloads.constraints(80 + Q * D, 20, Q, D, base_hi=1 << 16)
    check(pruned(torch_cuda, mapper, K, X, base, elig), oracle.oracle_map_constrained(K, X, base, elig), "constrained")
    check(pruned(torch_cuda, mapper, K, X, None, elig), oracle.oracle_map_constrained(K, X, None, elig), "masks only")


def test_pruned_degenerate(torch_cuda, mapper):
    for Q, D in ((8, 4), (12, 3), (6, 8), (10, 2)):
        zeros = np.zeros((1, Q, D), np.uint64)
        eq = np.full((1, Q, D), 7, np.uint64)
        hot = np.full((1, Q, D), 1000, np.uint64)
        hot[0, :, D - 1] = 1
        for K in (zeros, eq, hot):
            check(pruned(torch_cuda, mapper, K, zeros), oracle.oracle_map(K, zeros), f"{Q}x{D}")


def test_pruned_batched_configs(torch_cuda, mapper):
    K, X = workloads.cfg2()
    check(pruned(torch_cuda, mapper, K, X), oracle.oracle_map(K, X), "cfg2")
    K, X = workloads.cfg3(E=100_000)
    check(pruned(torch_cuda, mapper, K, X), oracle.oracle_map(K, X), "cfg3")
    for name in workloads.NPB_RATIO:
        K, X = workloads.cfg1_npb(name)
        check(pruned(torch_cuda, mapper, K, X), oracle.oracle_map(K, X), name)


def _golden_full():
    path = os.path.join(GOLDEN, "full_configs.json")
    return json.load(open(path))["cases"] if os.path.exists(path) else {}


@pytest.mark.parametrize("key", sorted(_golden_full()))
def test_pruned_full_size(torch_cuda, mapper, key):
    case = _golden_full()[key]
    K, X = workloads.make(case["config"], seed=case["seed"])
    gi, gmp, gms = pruned(torch_cuda, mapper, K, X)
    assert int(gi[0]) == case["index"] and int(gms[0]) == case["makespan"]
    assert list(gmp[0]) == case["mapping"]
    assert 0 < mapper.launch_info()["nodes"] < 4**16  # far fewer nodes than mappings


def test_pruned_matches_exhaustive_gpu_beyond_oracle(torch_cuda, mapper):
    """Larger random searches (up to 8^13 = 5.5e11 mappings) where the exhaustive GPU kernel
    is the reference (itself pinned to the oracle at cfg5 scale)."""
    for seed, (Q, D) in enumerate(((13, 8), (18, 4), (9, 16))):
        K, X = workloads.random_tables(900 + seed, 1, Q, D, hi=1 << 22)
        a = pruned(torch_cuda, mapper, K, X)
        b = mapper.map_queues(dev(torch_cuda, K), dev(torch_cuda, X))
        b = tuple(t.cpu().numpy() for t in b)
        assert int(a[0][0]) == int(b[0][0]) and int(a[2][0]) == int(b[2][0]), (Q, D)


def test_pruned_small_cutover(torch_cuda, mapper):
    """Below 2^24 mappings the entry point scores exhaustively (same result)."""
    K, X = workloads.cfg2(E=50, seed=3)
    check(pruned(torch_cuda, mapper, K, X, force=False), oracle.oracle_map(K, X), "cutover")
    assert mapper.launch_info()["path"] != "pruned"


def test_pruned_errors(torch_cuda, mapper):
    K = np.ones((1, 4, 3), np.uint64)
    with pytest.raises(MclError) as e:
        mapper.map_queues_pruned(K, K, None, np.array([[0, 0b1000, 0, 0]], np.uint16))
    assert e.value.status == MCL_E_INVAL
    i, mp, ms = mapper.map_queues_pruned(K, K)  # host buffers, no constraints
    check((i, mp, ms), oracle.oracle_map(K, K), "host")
