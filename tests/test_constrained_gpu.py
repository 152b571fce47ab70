"""GPU parity of the constrained variant (NEXT-3) and of the scoring entry point, against
the constrained oracle; bit-exact. Run with ``pytest -m gpu``."""
from __future__ import annotations

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


@pytest.fixture(scope="module")
def mapper(torch_cuda):
    m = Mapper(0)
    yield m
    m.close()


def dev(torch, a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def run(torch, m, K, X, base, elig, path=0):
    m.force_path(path)
    try:
        i, mp, ms = m.map_queues_constrained(dev(torch, K), dev(torch, X),
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


def random_constraints(seed, E, Q, D, pin_frac=0.3):
    rng = np.random.default_rng(seed)
    base = rng.integers(0, 1 << 18, size=(E, D), dtype=np.uint64)
    elig = rng.integers(0, 1 << D, size=(E, Q)).astype(np.uint16)
    pins = rng.random((E, Q)) < pin_frac
    elig[pins] = (1 << rng.integers(0, D, size=int(pins.sum()))).astype(np.uint16)
    return base, elig


@pytest.mark.parametrize("Q,D", [(3, 2), (4, 3), (5, 4), (6, 5), (4, 8), (7, 3), (2, 3), (1, 4), (3, 11)])
def test_constrained_all_paths(torch_cuda, mapper, Q, D):
    K, X = workloads.random_tables(50 + Q * D, 24, Q, D, hi=1 << 20)
    base, elig = random_constraints(60 + Q * D, 24, Q, D)
    want = oracle.oracle_map_constrained(K, X, base, elig)
    paths = [0, 3] + ([1, 2] if Q >= 3 and 2 <= D <= 8 else [])
    for p in paths:
        for b, el in ((base, elig), (None, elig), (base, None)):
            w = want if (b is base and el is elig) else oracle.oracle_map_constrained(K, X, b, el)
            check(run(torch_cuda, mapper, K, X, b, el, p), w, f"Q={Q} D={D} path={p}")


def test_constrained_cfg4_scale_u64_fallback_and_shards(torch_cuda, mapper):
    """A full-size-shaped search (12 queues x 4 devices) with pins; large base loads force
    64-bit loads; shard-mode handles check the sub-ranges."""
    torch = torch_cuda
    K, X = workloads.cfg4(seed=9, Q=12)
    base, elig = random_constraints(9, 1, 12, 4, pin_frac=0.25)
    want = oracle.oracle_map_constrained(K, X, base, elig)
    check(run(torch, mapper, K, X, base, elig), want, "cfg4-12")
    big = base + np.uint64(1 << 40)
    check(run(torch, mapper, K, X, big, elig), oracle.oracle_map_constrained(K, X, big, elig), "u64")
    N = 4**12
    unit = 4**3
    nb = N // unit
    best = None
    G = 7
    for r in range(G):
        with Mapper(0, rank=r, world=G) as m:
            i, mp, ms = m.map_queues_constrained(dev(torch, K), dev(torch, X), dev(torch, base), dev(torch, elig))
        got = (int(ms.cpu().numpy()[0]), int(i.cpu().numpy()[0]))
        lo, hi = (nb * r // G) * unit, (nb * (r + 1) // G) * unit
        try:
            oi, oms, _ = oracle.oracle_map_constrained(K, X, base, elig, lo=lo, hi=hi)
            assert got == (int(oms[0]), int(oi[0])), f"shard {r}"
        except oracle.OracleError:  # no feasible mapping in this shard: (UINT64_MAX, UINT64_MAX)
            assert got == (2**64 - 1, 2**64 - 1), f"empty shard {r}"
            assert (mp.cpu().numpy() == 0xFF).all()
        best = got if best is None else min(best, got)
    assert best == (int(want[1][0]), int(want[0][0]))


def test_constrained_host_buffers(torch_cuda, mapper):
    K, X = workloads.cfg2(E=40, seed=5)
    base, elig = random_constraints(5, 40, 8, 4)
    i, mp, ms = mapper.map_queues_constrained(K, X, base, elig)
    check((i, mp, ms), oracle.oracle_map_constrained(K, X, base, elig), "host")


def test_constrained_errors(torch_cuda, mapper):
    K = np.ones((1, 4, 3), np.uint64)
    with pytest.raises(MclError) as e:
        mapper.map_queues_constrained(K, K, None, np.array([[0, 0b1000, 0, 0]], np.uint16))
    assert e.value.status == MCL_E_INVAL
    with pytest.raises(MclError) as e:
        mapper.map_queues_constrained(K, K, np.array([[0, 1 << 48, 0]], np.uint64), None)
    assert e.value.status == MCL_E_RANGE
    # all masks = all devices, zero base: the unconstrained answer
    full = np.full((1, 4), 0b111, np.uint16)
    got = mapper.map_queues_constrained(K, K, np.zeros((1, 3), np.uint64), full)
    check(got, oracle.oracle_map(K, K), "full masks")


def test_score_mappings(torch_cuda, mapper):
    """Round-robin and random mappings scored on the GPU == oracle scores; the optimum never
    exceeds them (round robin is not always optimal)."""
    torch = torch_cuda
    E, Q, D = 500, 8, 4
    K, X = workloads.cfg2(E=E, seed=8)
    base = np.random.default_rng(3).integers(0, 1 << 16, size=(E, D), dtype=np.uint64)
    rr = np.tile((np.arange(Q) % D).astype(np.uint8), (E, 1))
    rnd = np.random.default_rng(4).integers(0, D, size=(E, Q)).astype(np.uint8)
    opt_i, opt_ms, _ = oracle.oracle_map_constrained(K, X, base, None)
    for mps in (rr, rnd):
        got = mapper.score_mappings(dev(torch, K), dev(torch, X), dev(torch, mps), dev(torch, base)).cpu().numpy()
        want = np.array([oracle.oracle_score_base(K[e], X[e], base[e], mps[e]) for e in range(E)], np.uint64)
        assert (got == want).all()
        assert (opt_ms <= got).all()
    got = mapper.score_mappings(K, X, rr)  # host buffers, no base loads
    assert (got == np.array([oracle.oracle_score(K[e], X[e], rr[e]) for e in range(E)], np.uint64)).all()
    bad = rr.copy()
    bad[3, 2] = D
    with pytest.raises(MclError) as e:
        mapper.score_mappings(K, X, bad)
    assert e.value.status == MCL_E_INVAL


@pytest.mark.parametrize("Q,D", [(5, 1), (6, 3), (9, 7), (4, 16), (12, 5)])
def test_score_mappings_every_device_count(torch_cuda, mapper, Q, D):
    """The scoring kernel is compiled per device count: random mappings with and without
    base loads equal the oracle's scores for several D up to 16."""
    torch = torch_cuda
    E = 300
    K, X = workloads.random_tables(60 + D, E, Q, D)
    base = np.random.default_rng(D).integers(0, 1 << 20, size=(E, D), dtype=np.uint64)
    mps = np.random.default_rng(100 + D).integers(0, D, size=(E, Q)).astype(np.uint8)
    got = mapper.score_mappings(dev(torch, K), dev(torch, X), dev(torch, mps), dev(torch, base)).cpu().numpy()
    want = np.array([oracle.oracle_score_base(K[e], X[e], base[e], mps[e]) for e in range(E)], np.uint64)
    assert (got == want).all()
    got = mapper.score_mappings(K, X, mps)
    assert (got == np.array([oracle.oracle_score(K[e], X[e], mps[e]) for e in range(E)], np.uint64)).all()
