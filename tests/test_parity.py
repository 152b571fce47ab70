"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle, bit-exact.

Integer costs, so (index, makespan, mapping) must be identical for every epoch. Run on a
B200 with ``pytest -m gpu``.
"""
from __future__ import annotations

import json
import os

import numpy as np
import pytest

import oracle
from conftest import cuda_available
from paper_conf_cluster_ajipbf15_b200 import workloads
from paper_conf_cluster_ajipbf15_b200.mcl import MCL_E_INVAL, MCL_E_RANGE, Mapper, MclError

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


def to_dev(torch, a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def run_gpu(torch, mp, K, X, path=0):
    mp.force_path(path)
    try:
        idx, mapping, ms = mp.map_queues(to_dev(torch, K), to_dev(torch, X))
    finally:
        mp.force_path(0)
    return idx.cpu().numpy(), mapping.cpu().numpy(), ms.cpu().numpy()


def assert_same(got, want, ctx=""):
    gi, gmp, gms = got
    wi, wms, wmp = want
    bad = np.nonzero((gi != wi) | (gms != wms))[0]
    assert bad.size == 0, f"{ctx}: {bad.size} epochs differ, first {bad[:5]}: gpu {gi[bad[:5]]}/{gms[bad[:5]]} oracle {wi[bad[:5]]}/{wms[bad[:5]]}"
    assert (gmp == wmp).all(), ctx


# ------------------------------------------------------------------ hand cases ---------
def _hand_cases():
    with open(os.path.join(GOLDEN, "hand_cases.json")) as f:
        return json.load(f)["cases"]


@pytest.mark.parametrize("case", _hand_cases(), ids=lambda c: c["name"])
@pytest.mark.parametrize("path", [0, 1, 2, 3])
def test_hand_cases_gpu(torch_cuda, mapper, case, path):
    K = np.array(case["K"], dtype=np.uint64)[None]
    X = np.array(case["X"], dtype=np.uint64)[None]
    Q, D = K.shape[1:]
    if path in (1, 2) and not (Q >= 3 and 2 <= D <= 8):
        pytest.skip("blocked kernel needs Q >= 3, 2 <= D <= 8")
    gi, gmp, gms = run_gpu(torch_cuda, mapper, K, X, path)
    assert int(gi[0]) == case["index"] and int(gms[0]) == case["makespan"]
    assert list(gmp[0]) == case["mapping"]


# --------------------------------------------------- random shapes, every kernel path --
SHAPES = [(q, d) for q in range(1, 8) for d in range(1, 9) if d**q <= 300_000]


@pytest.mark.parametrize("Q,D", SHAPES)
def test_random_shapes_all_paths(torch_cuda, mapper, Q, D):
    E = 64 if D**Q <= 5000 else 8
    for seed, maker in ((10 * Q + D, workloads.random_tables), (1000 + 10 * Q + D, workloads.small_int_tables)):
        K, X = maker(seed, E, Q, D)
        want = oracle.oracle_map(K, X)
        paths = [0, 3]
        if Q >= 3 and 2 <= D <= 8:
            paths += [1, 2, 5]
        for p in paths:
            assert_same(run_gpu(torch_cuda, mapper, K, X, p), want, f"Q={Q} D={D} path={p} {maker.__name__}")


def test_generic_large_d(torch_cuda, mapper):
    for Q, D in ((2, 16), (3, 16), (4, 12), (5, 9), (4, 10)):
        K, X = workloads.random_tables(7 * Q + D, 3, Q, D)
        assert_same(run_gpu(torch_cuda, mapper, K, X), oracle.oracle_map(K, X), f"Q={Q} D={D}")


def test_batched_equals_single_and_permutation(torch_cuda, mapper):
    K, X = workloads.random_tables(99, 40, 6, 4, hi=1 << 10)
    gi, gmp, gms = run_gpu(torch_cuda, mapper, K, X)
    for e in (0, 7, 39):
        si, smp, sms = run_gpu(torch_cuda, mapper, K[e:e + 1], X[e:e + 1])
        assert si[0] == gi[e] and sms[0] == gms[e] and (smp[0] == gmp[e]).all()
    perm = np.random.default_rng(3).permutation(40)
    pi, _, pms = run_gpu(torch_cuda, mapper, K[perm], X[perm])
    assert (pi == gi[perm]).all() and (pms == gms[perm]).all()


# ------------------------------------------------------------- the five configs -------
@pytest.mark.parametrize("name", list(workloads.NPB_RATIO))
def test_cfg1_npb(torch_cuda, mapper, name):
    K, X = workloads.cfg1_npb(name)
    assert_same(run_gpu(torch_cuda, mapper, K, X), oracle.oracle_map(K, X), name)
    assert_same(run_gpu(torch_cuda, mapper, K, X, 1), oracle.oracle_map(K, X), name)


def test_cfg1_random_seeds(torch_cuda, mapper):
    Ks, Xs = zip(*(workloads.cfg1_random(s) for s in range(2000)))
    K, X = np.concatenate(Ks), np.concatenate(Xs)
    want = oracle.oracle_map(K, X)
    for p in (0, 1, 3, 5):
        assert_same(run_gpu(torch_cuda, mapper, K, X, p), want, f"cfg1 x2000 path {p}")


def test_cfg2_full(torch_cuda, mapper):
    K, X = workloads.cfg2()
    want = oracle.oracle_map(K, X)
    assert_same(run_gpu(torch_cuda, mapper, K, X), want, "cfg2")
    assert mapper.launch_info()["path"] == "batch_pool_u32"
    assert_same(run_gpu(torch_cuda, mapper, K, X, 5), want, "cfg2 flattened")
    assert_same(run_gpu(torch_cuda, mapper, K, X, 1), want, "cfg2 CTA per epoch")
    # repeated calls reuse the self-resetting per-epoch keys; a smaller batch after a larger one
    assert_same(run_gpu(torch_cuda, mapper, K[:37], X[:37]), tuple(w[:37] for w in want), "cfg2[:37]")
    assert_same(run_gpu(torch_cuda, mapper, K, X), want, "cfg2 again")


def test_cfg3_full(torch_cuda, mapper):
    K, X = workloads.cfg3()
    want = oracle.oracle_map(K, X)
    assert_same(run_gpu(torch_cuda, mapper, K, X), want, "cfg3")
    assert mapper.launch_info()["path"] == "small_batched"
    # the paper's two regimes (Fig. 9): column-major -> (C, C) always (the generator makes
    # every GPU at least 2.5x the CPU); row-major -> mostly split over the two GPUs
    _, mp, _ = run_gpu(torch_cuda, mapper, K[:1000], X[:1000])
    assert (mp[0::2] == 0).all()
    assert (np.sort(mp[1::2], axis=1) == [1, 2]).all(axis=1).mean() > 0.5


def test_cfg3_ragged_and_unaligned(torch_cuda, mapper):
    """Tail tiles (E not a multiple of the tile) and a 16-byte-misaligned base pointer take
    the plain-load path instead of cp.async.bulk."""
    torch = torch_cuda
    K, X = workloads.cfg3(E=4097, seed=11)
    want = oracle.oracle_map(K, X)
    assert_same(run_gpu(torch, mapper, K, X), want, "ragged")
    Kd = torch.zeros(4097 * 6 + 1, dtype=torch.uint64, device="cuda")
    Xd = torch.zeros(4097 * 6 + 1, dtype=torch.uint64, device="cuda")
    Kd[1:] = torch.from_numpy(K.reshape(-1)).cuda()
    Xd[1:] = torch.from_numpy(X.reshape(-1)).cuda()
    idx = torch.empty(4097, dtype=torch.uint64, device="cuda")
    ms = torch.empty_like(idx)
    mp = torch.empty((4097, 2), dtype=torch.uint8, device="cuda")
    mapper.map_queues_into(Kd[1:].view(4097, 2, 3), Xd[1:].view(4097, 2, 3), idx, mp, ms)
    assert_same((idx.cpu().numpy(), mp.cpu().numpy(), ms.cpu().numpy()), want, "unaligned")


def _golden_full():
    path = os.path.join(GOLDEN, "full_configs.json")
    return json.load(open(path))["cases"] if os.path.exists(path) else {}


@pytest.mark.parametrize("key", sorted(_golden_full()))
def test_full_single_epoch_configs(torch_cuda, mapper, key):
    """cfg4 / cfg5 at full size, in the launch configuration bench.py times, against the
    oracle's full run (tests/golden/full_configs.json, scripts/make_golden.py)."""
    case = _golden_full()[key]
    K, X = workloads.make(case["config"], seed=case["seed"])
    gi, gmp, gms = run_gpu(torch_cuda, mapper, K, X)
    assert int(gi[0]) == case["index"] and int(gms[0]) == case["makespan"]
    assert list(gmp[0]) == case["mapping"]


@pytest.mark.parametrize("name,G", [("cfg4", 3), ("cfg4", 8), ("cfg5", 7), ("cfg5", 4096)])
def test_full_size_shards_sampled(torch_cuda, name, G):
    """At full size, sampled shards: the GPU's shard-local argmin equals the oracle's on the
    same index sub-range (the oracle computes these one by one), and (when every shard is
    run) the min over all shards equals the unsharded result."""
    torch = torch_cuda
    K, X = workloads.make(name)
    Q, D = K.shape[1:]
    N = D**Q
    unit = D**3  # blocked kernel shards whole blocks of the 3 innermost digits
    nb = N // unit
    Kd, Xd = to_dev(torch, K), to_dev(torch, X)
    ranks = list(range(G)) if G <= 16 else sorted({0, 1, G // 2, G - 2, G - 1} |
                                                  set(np.random.default_rng(G).integers(0, G, 20).tolist()))
    results = []
    for r in ranks:
        with Mapper(0, rank=r, world=G) as m:
            idx, mp, ms = m.map_queues(Kd, Xd)
            assert m.launch_info()["path"] == "blocked_u32"
        results.append((int(ms[0].item()), int(idx[0].item())))
        lo, hi = (nb * r // G) * unit, (nb * (r + 1) // G) * unit
        assert lo <= results[-1][1] < hi
        if hi - lo <= 6 * 10**8 and (G > 16 or r in (0, G // 2, G - 1)):
            oi, oms, _ = oracle.oracle_map(K, X, lo=lo, hi=hi)
            assert (int(oms[0]), int(oi[0])) == results[-1], f"shard {r}/{G}"
    if len(ranks) == G:
        with Mapper(0) as m:
            idx, mp, ms = m.map_queues(Kd, Xd)
        assert min(results) == (int(ms[0].item()), int(idx[0].item()))


# ------------------------------------------------------------------- edge cases -------
def test_u64_fallback_and_max_entries(torch_cuda, mapper):
    """Bounds >= 2^32 need 64-bit loads: the u32 kernel detects it on the device and the
    call reruns with the 64-bit kernel. Entries up to 2^48 - 1 are accepted."""
    rng = np.random.default_rng(5)
    K = rng.integers((1 << 47), (1 << 48) - 1, size=(5, 6, 4), dtype=np.uint64)
    X = np.zeros_like(K)
    X[:, :, 1:] = rng.integers(0, 1 << 20, size=(5, 6, 3), dtype=np.uint64)
    want = oracle.oracle_map(K, X)
    for p in (0, 1, 3, 5):
        assert_same(run_gpu(torch_cuda, mapper, K, X, p), want, f"u64 path {p}")
    run_gpu(torch_cuda, mapper, K, X, 1)
    assert mapper.launch_info()["path"] == "blocked_u64"
    K = np.full((2, 5, 3), (1 << 48) - 1, dtype=np.uint64)
    assert_same(run_gpu(torch_cuda, mapper, K, np.zeros_like(K)), oracle.oracle_map(K, np.zeros_like(K)), "max")


U32_TOP = (1 << 32) - 1  # 0xFFFFFFFF: the all-ones "no candidate" start of the u32 minima


def _one_big_queue(E, Q, D, totals, big_q=0):
    """Epoch e: queue big_q costs totals[e] on every device, every other entry 0, so the
    bound UB = sum_q max_d C = totals[e] and EVERY mapping's makespan is totals[e]: the
    optimum equals UB (ms* = UB) and the lowest index 0 wins the all-way tie."""
    K = np.zeros((E, Q, D), np.uint64)
    for e, t in enumerate(totals):
        K[e, big_q, :] = t
    return K, np.zeros_like(K)


def _balanced_at(total, Q=4, D=3):
    """One epoch whose bound UB = sum_q max_d C equals `total` exactly: queue q costs r_q on
    device 0 and r_q + 1 on the others, with sum_q (r_q + 1) = total."""
    K = np.zeros((1, Q, D), np.uint64)
    base = total // Q - 1
    r = [base] * Q
    r[0] += total - Q * (base + 1)
    for q in range(Q):
        K[0, q, 0] = r[q]
        K[0, q, 1:] = r[q] + 1
    assert sum(int(K[0, q].max()) for q in range(Q)) == total
    return K, np.zeros_like(K)


@pytest.mark.parametrize("Q,D", [(5, 2), (6, 3), (8, 4)])
def test_u32_top_of_range_optimum_equals_bound(torch_cuda, mapper, Q, D):
    """ms* = UB = 2^32 - 1: the u32 kernels' running minima start at
    0xFFFFFFFF with a strict <, so this bound must take the 64-bit kernel (else the call
    returned index = makespan = UINT64_MAX). UB = 2^32 - 2 is the largest bound the u32
    kernels keep, and there the optimum equal to UB must still be found by them."""
    for total, want_path in ((U32_TOP, "blocked_u64"), (U32_TOP - 1, "blocked_u32")):
        K, X = _one_big_queue(1, Q, D, [total], big_q=1)
        want = oracle.oracle_map(K, X)
        assert int(want[1][0]) == total and int(want[0][0]) == 0
        for p in (0, 1):
            assert_same(run_gpu(torch_cuda, mapper, K, X, p), want, f"{Q}x{D} UB={total} path {p}")
            assert mapper.launch_info()["path"] == want_path, (total, p, mapper.launch_info())


@pytest.mark.parametrize("Q,D", [(6, 3), (8, 4)])
def test_u32_top_of_range_batched(torch_cuda, mapper, Q, D):
    """Three epochs in one call (UB = 2^32 - 1, an ordinary epoch, UB = 2^32 - 2): the whole
    call reruns on 64-bit loads when any epoch needs it; the flattened and warp-per-epoch
    batch kernels too."""
    K, X = _one_big_queue(3, Q, D, [U32_TOP, 0, U32_TOP - 1], big_q=Q - 1)
    rng = np.random.default_rng(Q * D)
    K[1] = rng.integers(0, 1 << 20, size=(Q, D), dtype=np.uint64)
    want = oracle.oracle_map(K, X)
    assert int(want[1][0]) == U32_TOP and int(want[1][2]) == U32_TOP - 1
    paths = [0, 1, 2, 3, 5] + ([7] if (Q, D) == (8, 4) else [])
    for p in paths:
        assert_same(run_gpu(torch_cuda, mapper, K, X, p), want, f"{Q}x{D} batched path {p}")
    # without the top epoch, the u32 kernels keep the call (UB = 2^32 - 2 at most)
    for p, name in ((1, "blocked_u32"), (5, "flat_u32")) + (((7, "batch_u32"),) if (Q, D) == (8, 4) else ()):
        assert_same(run_gpu(torch_cuda, mapper, K[1:], X[1:], p), tuple(w[1:] for w in want), f"path {p}")
        assert mapper.launch_info()["path"] == name


def test_u32_top_of_range_shards(torch_cuda):
    """Shard-mode handles (G = 3) at ms* = UB = 2^32 - 1 and 2^32 - 2: every shard's local
    argmin equals the oracle's on the same index sub-range."""
    torch = torch_cuda
    Q, D, G = 6, 3, 3
    nb = D ** (Q - 3)
    for total in (U32_TOP, U32_TOP - 1):
        K, X = _one_big_queue(1, Q, D, [total], big_q=2)
        Kd, Xd = to_dev(torch, K), to_dev(torch, X)
        for r in range(G):
            with Mapper(0, rank=r, world=G) as m:
                idx, _, ms = m.map_queues(Kd, Xd)
                path = m.launch_info()["path"]
            lo, hi = (nb * r // G) * D**3, (nb * (r + 1) // G) * D**3
            oi, oms, _ = oracle.oracle_map(K, X, lo=lo, hi=hi)
            assert (int(ms[0].item()), int(idx[0].item())) == (int(oms[0]), int(oi[0])), (total, r)
            assert path == ("blocked_u64" if total == U32_TOP else "blocked_u32")


def test_u32_boundary(torch_cuda, mapper):
    """Bounds UB = 2^32 - 2, 2^32 - 1 and 2^32 exactly (UB = sum_q max_d C, built to the
    unit), with a non-trivial optimum below UB: the u32 kernel keeps the first, the other two
    take the 64-bit rerun, and all three match the oracle."""
    for total, want_path in ((U32_TOP - 1, "blocked_u32"), (U32_TOP, "blocked_u64"), (1 << 32, "blocked_u64")):
        K, X = _balanced_at(total)
        want = oracle.oracle_map(K, X)
        assert_same(run_gpu(torch_cuda, mapper, K, X, 1), want, str(total))
        assert mapper.launch_info()["path"] == want_path


def test_degenerate_ties(torch_cuda, mapper):
    """All-equal (maximal ties), all-zero (every mapping ties at 0) and one-hot cheap device."""
    for Q, D in ((8, 4), (12, 3), (6, 8), (5, 5)):
        zeros = np.zeros((1, Q, D), np.uint64)
        eq = np.full((1, Q, D), 7, np.uint64)
        hot = np.full((1, Q, D), 1000, np.uint64)
        hot[0, :, D - 1] = 1
        for K in (zeros, eq, hot):
            assert_same(run_gpu(torch_cuda, mapper, K, zeros), oracle.oracle_map(K, zeros), f"{Q}x{D}")


def test_range_and_argument_errors(torch_cuda, mapper):
    torch = torch_cuda
    K = np.zeros((1, 4, 3), np.uint64)
    K[0, 2, 1] = 1 << 48
    for p in (0, 1, 3):
        with pytest.raises(MclError) as e:
            run_gpu(torch, mapper, K, np.zeros_like(K), p)
        assert e.value.status == MCL_E_RANGE
    # D^Q > 2^48
    with pytest.raises(MclError) as e:
        mapper.map_queues(np.zeros((1, 13, 16), np.uint64), np.zeros((1, 13, 16), np.uint64))
    assert e.value.status == MCL_E_RANGE
    with pytest.raises(MclError) as e:
        mapper.map_queues(np.zeros((1, 2, 17), np.uint64), np.zeros((1, 2, 17), np.uint64))
    assert e.value.status == MCL_E_INVAL
    with pytest.raises(MclError) as e:
        mapper.map_queues(np.zeros((1, 33, 1), np.uint64), np.zeros((1, 33, 1), np.uint64))
    assert e.value.status == MCL_E_INVAL
    # epochs == 0 is a no-op
    from paper_conf_cluster_ajipbf15_b200.mcl import mcl_map_queues

    assert mcl_map_queues(mapper.handle, 3, 3, 0, 0, 0, 0, None, 0) == 0
    # the mapper keeps working after errors
    K, X = workloads.cfg1_npb("FT")
    assert_same(run_gpu(torch, mapper, K, X), oracle.oracle_map(K, X), "after errors")
    # forced path that cannot run this shape
    with pytest.raises(MclError) as e:
        run_gpu(torch, mapper, np.zeros((1, 2, 3), np.uint64), np.zeros((1, 2, 3), np.uint64), 1)
    assert e.value.status == MCL_E_INVAL


def test_host_buffers_e2e(torch_cuda, mapper):
    """Host (numpy, pageable) and pinned torch buffers are staged inside the call."""
    torch = torch_cuda
    K, X = workloads.cfg2(E=300, seed=21)
    want = oracle.oracle_map(K, X)
    idx, mp, ms = mapper.map_queues(K, X)
    assert_same((idx, mp, ms), want, "numpy")
    Kp = torch.from_numpy(K).pin_memory()
    Xp = torch.from_numpy(X).pin_memory()
    idx, mp, ms = mapper.map_queues(Kp, Xp)
    assert_same((idx.numpy(), mp.numpy(), ms.numpy()), want, "pinned")
    # mixed: device inputs, host outputs
    i2 = np.empty(300, np.uint64)
    m2 = np.empty(300, np.uint64)
    p2 = np.empty((300, 8), np.uint8)
    mapper.map_queues_into(to_dev(torch, K), to_dev(torch, X), i2, p2, m2)
    assert_same((i2, p2, m2), want, "mixed")
    # mapping output is optional
    idx, mp, ms = mapper.map_queues(K, X, with_mapping=False)
    assert mp is None and (idx == want[0]).all()


def test_external_stream(torch_cuda):
    torch = torch_cuda
    s = torch.cuda.Stream()
    K, X = workloads.cfg2(E=50, seed=4)
    with Mapper(0, stream=s.cuda_stream) as m:
        got = m.map_queues(to_dev(torch, K), to_dev(torch, X))
    assert_same(tuple(t.cpu().numpy() for t in got), oracle.oracle_map(K, X), "stream")


def test_nccl_single_rank_collective_path(torch_cuda):
    """A 1-rank NCCL communicator runs the multi-GPU sequence (packed key, all-reduce,
    decode) on one GPU; large makespans take the two-step lexicographic reduce."""
    torch = torch_cuda
    from paper_conf_cluster_ajipbf15_b200 import mcl

    comm = mcl.mcl_comm_init(0, 1, 0, mcl.mcl_comm_unique_id())
    try:
        with Mapper(0, nccl_comm=comm, rank=0, world=1) as m:
            K, X = workloads.cfg4(seed=4, Q=12)
            got = m.map_queues(to_dev(torch, K), to_dev(torch, X))
            info = m.launch_info()
            assert info["allreduce"] and not info["two_step"]
            assert_same(tuple(t.cpu().numpy() for t in got), oracle.oracle_map(K, X), "packed")
            K = np.random.default_rng(1).integers(1 << 46, 1 << 47, size=(3, 9, 4), dtype=np.uint64)
            X = np.zeros_like(K)
            got = m.map_queues(to_dev(torch, K), to_dev(torch, X))
            assert m.launch_info()["two_step"]
            assert_same(tuple(t.cpu().numpy() for t in got), oracle.oracle_map(K, X), "two-step")
            # masked calls (mixed-radix kernel) through the same sequence, device and pinned
            K, X = workloads.cfg4(seed=5, Q=11)
            base, elig = workloads.constraints(12, 1, 11, 4)
            want = oracle.oracle_map_constrained(K, X, base, elig)
            got = m.map_queues_constrained(to_dev(torch, K), to_dev(torch, X), to_dev(torch, base), to_dev(torch, elig))
            assert m.launch_info()["allreduce"] and m.launch_info()["path"] == "mixed_u32"
            assert_same(tuple(t.cpu().numpy() for t in got), want, "constrained nccl")
            pin = [torch.from_numpy(a).pin_memory() for a in (K, X, base, elig)]
            got = m.map_queues_constrained(*pin)
            assert_same(tuple(t.numpy() for t in got), want, "constrained nccl pinned")
    finally:
        mcl.mcl_comm_destroy(comm)


def test_probe(torch_cuda):
    from paper_conf_cluster_ajipbf15_b200 import mcl

    for op in range(5):
        rate, per_clk, mhz = mcl.mcl_probe_int_rate(0, op)
        assert rate > 1e12 and 30 < per_clk < 140 and 500 < mhz < 2500


@pytest.mark.parametrize("Q,D", [(2, 2), (2, 3), (2, 4), (3, 2), (3, 3), (3, 4), (4, 2), (4, 3)])
def test_small_shapes_tiny_and_tiled(torch_cuda, mapper, Q, D):
    """The small shapes at both sides of the warp-per-epoch cut-over (<= 64 epochs: one warp
    per epoch; more: the thread-per-epoch TMA kernel), with random and tie-heavy tables and
    entries near 2^48 (the packed key's makespan field)."""
    for E in (1, 31, 64, 65):
        for seed, maker in ((E + 10 * Q + D, workloads.random_tables), (E + 500 + 10 * Q + D, workloads.small_int_tables)):
            K, X = maker(seed, E, Q, D)
            got_i, got_mp, got_ms = mapper.map_queues(to_dev(torch_cuda, K), to_dev(torch_cuda, X))
            assert mapper.launch_info()["path"] == "small_batched"
            wi, wms, wmp = oracle.oracle_map(K, X)
            ctx = f"Q={Q} D={D} E={E} {maker.__name__}"
            assert (got_i.cpu().numpy() == wi).all() and (got_ms.cpu().numpy() == wms).all(), ctx
            assert (got_mp.cpu().numpy() == wmp).all(), ctx
    K = np.full((3, Q, D), (1 << 48) - 1, np.uint64)
    X = np.zeros_like(K)
    got_i, _, got_ms = mapper.map_queues(to_dev(torch_cuda, K), to_dev(torch_cuda, X))
    wi, wms, _ = oracle.oracle_map(K, X)
    assert (got_i.cpu().numpy() == wi).all() and (got_ms.cpu().numpy() == wms).all()


def test_d5_single_epoch_lean_build(torch_cuda, mapper):
    """Single epochs with D = 5 run the one-CTA-per-SM (spill-free) build of the blocked
    kernel: whole index spaces and sharded sub-ranges equal the oracle."""
    for Q in (6, 8, 9):
        K, X = workloads.random_tables(700 + Q, 1, Q, 5)
        want = oracle.oracle_map(K, X)
        i, mp, ms = mapper.map_queues(to_dev(torch_cuda, K), to_dev(torch_cuda, X))
        assert mapper.launch_info()["path"] == "blocked_u32_lean"
        assert int(i[0]) == want[0][0] and int(ms[0]) == want[1][0] and (mp.cpu().numpy() == want[2]).all()
        N, unit = 5**Q, 125
        for r in range(3):
            with Mapper(0, rank=r, world=3) as m:
                si, _, sms = m.map_queues(to_dev(torch_cuda, K), to_dev(torch_cuda, X))
            nb = N // unit
            lo, hi = (nb * r // 3) * unit, (nb * (r + 1) // 3) * unit
            oi, oms, _ = oracle.oracle_map(K, X, lo=lo, hi=hi)
            assert (int(si[0]), int(sms[0])) == (int(oi[0]), int(oms[0])), f"Q={Q} shard {r}"
        # a batch of D = 5 epochs keeps the two-CTA build
        KB, XB = workloads.random_tables(710 + Q, 3, Q, 5)
        wb = oracle.oracle_map(KB, XB)
        assert_same(run_gpu(torch_cuda, mapper, KB, XB, 1), wb, f"Q={Q} batch")
        assert mapper.launch_info()["path"] == "blocked_u32"


def test_default_stream_follows_torch_current_stream(torch_cuda):
    """Mapper() without a stream runs on torch's current stream: inputs written
    on that stream after a 20+ ms spin are complete when the search reads them. (On a
    private non-blocking stream the search would read the zero tables.)"""
    torch = torch_cuda
    K, X = workloads.cfg2(E=300, seed=21)
    want = oracle.oracle_map(K, X)
    Ks, Xs = to_dev(torch, K), to_dev(torch, X)
    torch.cuda.synchronize()
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        Kd, Xd = torch.zeros_like(Ks), torch.zeros_like(Xs)
        torch.cuda._sleep(40_000_000)  # ~20 ms of device spin on s before the inputs land
        Kd.copy_(Ks)
        Xd.copy_(Xs)
        with Mapper(0) as m:
            i, mp, ms = m.map_queues(Kd, Xd)
    torch.cuda.synchronize()
    assert_same((i.cpu().numpy(), mp.cpu().numpy(), ms.cpu().numpy()), want, "torch stream order")


@pytest.mark.parametrize("Q,D", [(15, 4), (10, 8)])
def test_large_single_epoch_ties_and_shards(torch_cuda, mapper, Q, D):
    """Single epochs of ~1e9 mappings spread over every CTA: random, tie-heavy and all-equal
    tables, whole and in 3 shards, equal the oracle -- the CTA winner is the minimum holder
    with the lowest block, the rescan is the one-pass pair scan, and the CTAs merge through
    one packed per-epoch key (atomicMin) that the last CTA decodes and resets."""
    torch = torch_cuda
    cases = [workloads.random_tables(900 + Q, 1, Q, D, hi=1 << 20),
             workloads.small_int_tables(901 + Q, 1, Q, D, hi=3)]
    eq = np.full((1, Q, D), 11, np.uint64)
    cases.append((eq, np.zeros_like(eq)))
    nb = D ** (Q - 3)
    for K, X in cases:
        want = oracle.oracle_map(K, X)
        assert_same(run_gpu(torch, mapper, K, X), want, f"{Q}x{D}")
        Kd, Xd = to_dev(torch, K), to_dev(torch, X)
        for r in range(3):
            with Mapper(0, rank=r, world=3) as m:
                i, _, ms = m.map_queues(Kd, Xd)
            lo, hi = (nb * r // 3) * D**3, (nb * (r + 1) // 3) * D**3
            oi, oms, _ = oracle.oracle_map(K, X, lo=lo, hi=hi)
            assert (int(ms[0].item()), int(i[0].item())) == (int(oms[0]), int(oi[0])), f"{Q}x{D} shard {r}"


def test_small_pinned_calls_zero_copy(torch_cuda, mapper):
    """Small calls whose buffers are all pinned host memory run the kernels on them in place
    (zero-copy over PCIe, no staging copies): cfg1 decisions, a small batch, a constrained
    call with pinned base loads and masks, and a pinned call too large for zero-copy (staged)
    -- all equal the oracle."""
    torch = torch_cuda

    def pinned(a):
        return torch.from_numpy(np.ascontiguousarray(a)).pin_memory()

    def outs(E, Q):
        return (torch.empty(E, dtype=torch.uint64).pin_memory(), torch.empty((E, Q), dtype=torch.uint8).pin_memory(),
                torch.empty(E, dtype=torch.uint64).pin_memory())

    for name in workloads.NPB_RATIO:
        K, X = workloads.cfg1_npb(name)
        i, mp, ms = outs(1, 4)
        mapper.map_queues_into(pinned(K), pinned(X), i, mp, ms)
        assert_same((i.numpy(), mp.numpy(), ms.numpy()), oracle.oracle_map(K, X), name)
    for (E, Q, D) in ((40, 6, 4), (3, 8, 4), (2000, 8, 4)):  # the last one is staged
        K, X = workloads.random_tables(E + Q, E, Q, D)
        i, mp, ms = outs(E, Q)
        mapper.map_queues_into(pinned(K), pinned(X), i, mp, ms)
        assert_same((i.numpy(), mp.numpy(), ms.numpy()), oracle.oracle_map(K, X), f"{E}x{Q}x{D}")
    K, X = workloads.random_tables(77, 8, 7, 4)
    base, elig = workloads.constraints(77, 8, 7, 4)
    gi, gmp, gms = mapper.map_queues_constrained(pinned(K), pinned(X), pinned(base), pinned(elig))
    assert_same((gi.numpy(), gmp.numpy(), gms.numpy()), oracle.oracle_map_constrained(K, X, base, elig), "constrained")


def test_u32_top_of_range_pooled_batch(torch_cuda, mapper):
    """The SM-pooled batch kernel (path 12) at the top of the u32 range: a 400-epoch 8 x 4
    batch mixing random epochs with epochs whose optimum equals the bound UB = 2^32 - 2
    stays on the pooled u32 kernel and is exact; one more epoch at ms* = UB = 2^32 - 1 makes
    the device flag the batch and the call rerun on 64-bit loads, still exact."""
    Q, D, E = 8, 4, 400
    K, X = workloads.random_tables(4040, E, Q, D)
    for e in (0, 137, 399):
        K[e], X[e] = (a[0] for a in _one_big_queue(1, Q, D, [U32_TOP - 1], big_q=e % Q))
    want = oracle.oracle_map(K, X)
    assert int(want[1][137]) == U32_TOP - 1
    assert_same(run_gpu(torch_cuda, mapper, K, X, 7), want, "pooled, ms* = 2^32 - 2")
    assert mapper.launch_info()["path"] == "batch_pool_u32"
    K[250], X[250] = (a[0] for a in _one_big_queue(1, Q, D, [U32_TOP], big_q=3))
    want = oracle.oracle_map(K, X)
    assert int(want[1][250]) == U32_TOP
    assert_same(run_gpu(torch_cuda, mapper, K, X, 7), want, "pooled batch with ms* = 2^32 - 1")
    assert mapper.launch_info()["path"] == "blocked_u64"
