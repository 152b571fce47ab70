"""GPU parity of the warp-per-epoch batched kernel (search_batch.cu, force_path 7) against
the CPU oracle, bit-exact, on every (Q, D) it is instantiated for; plus its automatic
selection, the 64-bit rerun, range errors and ragged batches. Run with ``pytest -m gpu``.
"""
from __future__ import annotations

import numpy as np
import pytest

import oracle
from conftest import cuda_available
from paper_conf_cluster_ajipbf15_b200 import workloads
from paper_conf_cluster_ajipbf15_b200.mcl import MCL_E_RANGE, Mapper, MclError

pytestmark = pytest.mark.gpu

BATCH_SHAPES = [(8, 3), (9, 3), (10, 3), (11, 3), (8, 4), (9, 4), (10, 4), (11, 4), (8, 5), (9, 5)]


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


def run(torch, mp, K, X, path):
    mp.force_path(path)
    try:
        idx, mapping, ms = mp.map_queues(torch.from_numpy(np.ascontiguousarray(K)).cuda(),
                                         torch.from_numpy(np.ascontiguousarray(X)).cuda())
        info = mp.launch_info()
    finally:
        mp.force_path(0)
    return (idx.cpu().numpy(), mapping.cpu().numpy(), ms.cpu().numpy()), info


def check(got, want, ctx):
    gi, gmp, gms = got
    wi, wms, wmp = want
    bad = np.nonzero((gi != wi) | (gms != wms))[0]
    assert bad.size == 0, f"{ctx}: {bad.size} epochs differ, first {bad[:5]}: gpu {gi[bad[:5]]}/{gms[bad[:5]]} oracle {wi[bad[:5]]}/{wms[bad[:5]]}"
    assert (gmp == wmp).all(), ctx


@pytest.mark.parametrize("Q,D", BATCH_SHAPES)
def test_batch_kernel_shapes(torch_cuda, mapper, Q, D):
    # E not a multiple of the 4 warps per CTA; fewer epochs for the large index spaces
    E = 37 if D**Q <= 300_000 else 5
    for seed, maker in ((50 * Q + D, workloads.random_tables), (900 + 50 * Q + D, workloads.small_int_tables)):
        K, X = maker(seed, E, Q, D)
        got, info = run(torch_cuda, mapper, K, X, 7)
        assert info["path"] == "batch_u32"
        check(got, oracle.oracle_map(K, X), f"Q={Q} D={D} {maker.__name__}")


def test_batch_degenerate_ties(torch_cuda, mapper):
    """All-zero, all-equal and one-hot-cheap epochs side by side in one batch."""
    for Q, D in ((8, 4), (9, 3), (8, 5)):
        zeros = np.zeros((1, Q, D), np.uint64)
        eq = np.full((1, Q, D), 7, np.uint64)
        hot = np.full((1, Q, D), 1000, np.uint64)
        hot[0, :, D - 1] = 1
        K = np.concatenate([zeros, eq, hot, eq, zeros])
        X = np.zeros_like(K)
        got, _ = run(torch_cuda, mapper, K, X, 7)
        check(got, oracle.oracle_map(K, X), f"{Q}x{D} ties")


def test_batch_auto_selection_cfg2(torch_cuda, mapper):
    """cfg2 (10^4 epochs >= one per resident CTA) runs the batched kernel automatically and
    agrees with the CTA-per-epoch kernel and the oracle on every epoch."""
    K, X = workloads.cfg2()
    want = oracle.oracle_map(K, X)
    got, info = run(torch_cuda, mapper, K, X, 0)
    assert info["path"] == "batch_pool_u32", info
    check(got, want, "cfg2 auto")
    got, info = run(torch_cuda, mapper, K, X, 1)
    assert info["path"] == "blocked_u32"
    check(got, want, "cfg2 CTA per epoch")
    # a batch below one epoch per resident CTA keeps the CTA-per-epoch kernel
    got, info = run(torch_cuda, mapper, K[:100], X[:100], 0)
    assert info["path"] == "blocked_u32", info
    check(got, tuple(w[:100] for w in want), "cfg2[:100]")


def test_batch_u64_rerun(torch_cuda, mapper):
    """A batch whose bound needs 64-bit loads is detected on the device and rerun with the
    64-bit blocked kernel (mixed with ordinary epochs)."""
    K, X = workloads.random_tables(71, 9, 8, 4)
    K[4] = np.random.default_rng(1).integers(1 << 46, 1 << 47, size=(8, 4), dtype=np.uint64)
    got, info = run(torch_cuda, mapper, K, X, 7)
    assert info["path"] == "blocked_u64"
    check(got, oracle.oracle_map(K, X), "u64 rerun")


def test_batch_range_error(torch_cuda, mapper):
    """An entry >= 2^48 in a split epoch fails the call; the next call on the same shapes
    is exact."""
    K, X = workloads.random_tables(72, 6, 8, 4)
    X[3, 2, 1] = 1 << 48
    with pytest.raises(MclError) as ei:
        run(torch_cuda, mapper, K, X, 7)
    assert ei.value.status == MCL_E_RANGE
    X[3, 2, 1] = 5
    got, _ = run(torch_cuda, mapper, K, X, 7)
    check(got, oracle.oracle_map(K, X), "after range error")


@pytest.mark.parametrize("Q,D", [(9, 3), (8, 4), (8, 5)])
def test_batch_whole_and_split_epochs(torch_cuda, mapper, Q, D):
    """More epochs than resident warps: whole epochs (one warp each) plus a last partial
    wave of epochs split over the warps of a CTA, merged in shared memory; repeated and
    interleaved with other batch sizes (below one wave: one warp per epoch)."""
    E = 148 * 16 + 123
    K, X = workloads.small_int_tables(77 * Q + D, E, Q, D, hi=64)
    want = oracle.oracle_map(K, X)
    for rep in range(2):
        got, info = run(torch_cuda, mapper, K, X, 7)
        assert info["path"] == "batch_pool_u32"
        check(got, want, f"{Q}x{D} E={E} rep {rep}")
        sub = 3 + 40 * rep  # every epoch split, then whole + split again
        got, _ = run(torch_cuda, mapper, K[:sub], X[:sub], 7)
        check(got, tuple(w[:sub] for w in want), f"{Q}x{D} E={sub} after E={E}")


def test_batch_single_epoch_and_no_mapping_output(torch_cuda, mapper):
    torch = torch_cuda
    K, X = workloads.random_tables(73, 1, 9, 4)
    got, _ = run(torch, mapper, K, X, 7)
    check(got, oracle.oracle_map(K, X), "E=1")
    # mapping output optional (NULL): index and makespan only
    K, X = workloads.random_tables(74, 11, 8, 4)
    Kd, Xd = torch.from_numpy(K).cuda(), torch.from_numpy(X).cuda()
    idx = torch.empty(11, dtype=torch.uint64, device="cuda")
    ms = torch.empty(11, dtype=torch.uint64, device="cuda")
    mapper.force_path(7)
    try:
        mapper.map_queues_into(Kd, Xd, idx, None, ms)
    finally:
        mapper.force_path(0)
    wi, wms, _ = oracle.oracle_map(K, X)
    assert (idx.cpu().numpy() == wi).all() and (ms.cpu().numpy() == wms).all()


# ---- the SM-pooled form (path 12): batches of >= 2 epochs per SM ----
POOL_E = 148 * 2 + 37  # >= 2 epochs per SM, ragged over the 148 CTAs


@pytest.mark.parametrize("Q,D", BATCH_SHAPES)
def test_pool_kernel_shapes(torch_cuda, mapper, Q, D):
    """Every instantiated shape, random and tie-heavy tables, bit-exact vs the oracle."""
    E = POOL_E if D**Q <= 1_100_000 else 300
    for seed, maker in ((60 * Q + D, workloads.random_tables), (700 + 60 * Q + D, workloads.small_int_tables)):
        K, X = maker(seed, E, Q, D)
        got, info = run(torch_cuda, mapper, K, X, 7)
        assert info["path"] == "batch_pool_u32", info
        assert info["threads"] == 512
        check(got, oracle.oracle_map(K, X), f"pool Q={Q} D={D} {maker.__name__}")


def test_pool_degenerate_ties_and_sizes(torch_cuda, mapper):
    """All-zero / all-equal / one-hot epochs spread over a pooled batch, then the same
    handle at other batch sizes (pool state lives in shared memory: nothing carries over)."""
    Q, D = 8, 4
    K, X = workloads.small_int_tables(4242, 1200, Q, D, hi=3)
    K[::7] = 0
    X[::7] = 0
    K[3::11] = 9
    X[3::11] = 0
    K[5::13] = 1000
    K[5::13, :, 2] = 1
    X[5::13] = 0
    want = oracle.oracle_map(K, X)
    for E in (1200, 296, 297, 1199, 1200):
        got, info = run(torch_cuda, mapper, K[:E], X[:E], 7)
        assert info["path"] == "batch_pool_u32", (E, info)
        check(got, tuple(w[:E] for w in want), f"pool ties E={E}")


def test_pool_u64_rerun_and_range_error(torch_cuda, mapper):
    """An epoch of a pooled batch whose bound needs 64 bits reruns the batch on the 64-bit
    kernel; an entry >= 2^48 fails the call; the next pooled call is exact."""
    K, X = workloads.random_tables(81, POOL_E, 8, 4)
    K[200] = np.random.default_rng(2).integers(1 << 46, 1 << 47, size=(8, 4), dtype=np.uint64)
    got, info = run(torch_cuda, mapper, K, X, 7)
    assert info["path"] == "blocked_u64"
    check(got, oracle.oracle_map(K, X), "pool u64 rerun")
    K, X = workloads.random_tables(82, POOL_E, 8, 4)
    X[300, 2, 1] = 1 << 48
    with pytest.raises(MclError) as ei:
        run(torch_cuda, mapper, K, X, 7)
    assert ei.value.status == MCL_E_RANGE
    X[300, 2, 1] = 5
    got, info = run(torch_cuda, mapper, K, X, 7)
    assert info["path"] == "batch_pool_u32"
    check(got, oracle.oracle_map(K, X), "pool after range error")


def test_pool_repeatable_under_load(torch_cuda, mapper):
    """The pooled kernel's shared-memory hand-offs (claims, table slots, key merges, slot
    reuse) checked by repetition: 12 back-to-back launches of full cfg2 (10^4 epochs over
    148 CTAs, 16 slots recycled ~4 times per CTA) must all equal the oracle bit for bit.
    (compute-sanitizer is not available on this pool: repeated exact parity stands in.)"""
    torch = torch_cuda
    K, X = workloads.cfg2()
    wi, wms, wmp = oracle.oracle_map(K, X)
    Kd, Xd = torch.from_numpy(K).cuda(), torch.from_numpy(X).cuda()
    outs = []
    for _ in range(12):
        idx, mp, ms = mapper.map_queues(Kd, Xd)
        assert mapper.launch_info()["path"] == "batch_pool_u32"
        outs.append((idx, mp, ms))
    for idx, mp, ms in outs:
        assert (idx.cpu().numpy() == wi).all() and (ms.cpu().numpy() == wms).all()
        assert (mp.cpu().numpy() == wmp).all()


def test_pool_concurrent_handles_on_two_streams(torch_cuda):
    """Two handles on two CUDA streams, driven from two host threads, each repeating its
    own batch: the pooled kernel keeps all its state in shared memory and the handles'
    scratch is separate, so concurrent searches stay exact."""
    torch = torch_cuda
    K1, X1 = workloads.cfg2(E=3000, seed=31)
    K2, X2 = workloads.small_int_tables(32, 2000, 9, 4, hi=50)
    w1, w2 = oracle.oracle_map(K1, X1), oracle.oracle_map(K2, X2)
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    d1 = [torch.from_numpy(a).cuda() for a in (K1, X1)]
    d2 = [torch.from_numpy(a).cuda() for a in (K2, X2)]
    torch.cuda.synchronize()
    import threading

    results = {}

    def worker(name, stream, dK, dX, reps):
        with Mapper(0, stream=stream.cuda_stream) as m:
            outs = []
            for _ in range(reps):
                outs.append(m.map_queues(dK, dX))
                assert m.launch_info()["path"] == "batch_pool_u32"
            results[name] = [tuple(t.cpu().numpy() for t in o) for o in outs]

    t1 = threading.Thread(target=worker, args=("a", s1, *d1, 6))
    t2 = threading.Thread(target=worker, args=("b", s2, *d2, 6))
    t1.start(); t2.start(); t1.join(); t2.join()
    for gi, gmp, gms in results["a"]:
        check((gi, gmp, gms), w1, "handle a")
    for gi, gmp, gms in results["b"]:
        check((gi, gmp, gms), w2, "handle b")
