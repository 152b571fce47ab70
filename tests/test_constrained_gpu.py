"""GPU parity of the constrained variant (NEXT-3) and of the scoring entry point, against
the constrained oracle; bit-exact. Run with ``pytest -m gpu``."""
from __future__ import annotations

import numpy as np
import pytest

import oracle
from conftest import cuda_available
from paper_conf_cluster_ajipbf15_b200 import workloads
from paper_conf_cluster_ajipbf15_b200.mcl import MCL_E_INVAL, MCL_E_RANGE, Mapper, MclError
from shard_ranges import mixed_shard_ranges

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
    paths = [0, 3] + ([1, 2, 8] if Q >= 3 and 2 <= D <= 8 else [])
    for p in paths:
        for b, el in ((base, elig), (None, elig), (base, None)):
            if p == 8 and el is None:
                continue  # the mixed-radix kernel serves calls with eligible masks
            w = want if (b is base and el is elig) else oracle.oracle_map_constrained(K, X, b, el)
            check(run(torch_cuda, mapper, K, X, b, el, p), w, f"Q={Q} D={D} path={p}")


def test_mixed_shard_ranges_helper():
    """The test helper's ranges tile [first feasible block, D^Q) and grow monotonically."""
    rng = np.random.default_rng(0)
    for _ in range(50):
        Q, D, G = int(rng.integers(3, 9)), int(rng.integers(2, 7)), int(rng.integers(1, 9))
        _, elig = random_constraints(int(rng.integers(1 << 30)), 1, Q, D)
        rs = mixed_shard_ranges(elig[0], Q, D, G)
        assert rs[-1][1] == D**Q
        assert all(rs[i][1] == rs[i + 1][0] for i in range(G - 1))
        assert all(lo <= hi for lo, hi in rs)


def _shards_vs_oracle(torch, K, X, base, elig, G, ranges):
    best = None
    for r in range(G):
        with Mapper(0, rank=r, world=G) as m:
            i, mp, ms = m.map_queues_constrained(dev(torch, K), dev(torch, X), dev(torch, base), dev(torch, elig))
        got = (int(ms.cpu().numpy()[0]), int(i.cpu().numpy()[0]))
        lo, hi = ranges[r]
        try:
            if lo >= hi:
                raise oracle.OracleError(-1)
            oi, oms, _ = oracle.oracle_map_constrained(K, X, base, elig, lo=lo, hi=hi)
            assert got == (int(oms[0]), int(oi[0])), f"shard {r}/{G} [{lo}, {hi})"
        except oracle.OracleError:  # no feasible mapping in this shard: (UINT64_MAX, UINT64_MAX)
            assert got == (2**64 - 1, 2**64 - 1), f"empty shard {r}"
            assert (mp.cpu().numpy() == 0xFF).all()
        best = got if best is None else min(best, got)
    return best


def test_constrained_cfg4_scale_u64_fallback_and_shards(torch_cuda, mapper):
    """A full-size-shaped search (12 queues x 4 devices) with pins; large base loads force
    64-bit loads; shard-mode handles check the sub-ranges (the mixed-radix kernel's shards
    of the feasible enumeration, and the INF-masked blocked kernel's full-space shards)."""
    torch = torch_cuda
    K, X = workloads.cfg4(seed=9, Q=12)
    base, elig = random_constraints(9, 1, 12, 4, pin_frac=0.25)
    want = oracle.oracle_map_constrained(K, X, base, elig)
    check(run(torch, mapper, K, X, base, elig), want, "cfg4-12")
    assert mapper.launch_info()["path"] == "mixed_u32"
    check(run(torch, mapper, K, X, base, elig, 1), want, "cfg4-12 full space")
    big = base + np.uint64(1 << 40)
    check(run(torch, mapper, K, X, big, elig), oracle.oracle_map_constrained(K, X, big, elig), "u64")
    assert mapper.launch_info()["path"] == "mixed_u64"
    G = 7
    best = _shards_vs_oracle(torch, K, X, base, elig, G, mixed_shard_ranges(elig[0], 12, 4, G))
    assert best == (int(want[1][0]), int(want[0][0]))
    # 64-bit loads: no super-block, every outer queue over its eligible devices only
    wide = _shards_vs_oracle(torch, K, X, big, elig, 5, mixed_shard_ranges(elig[0], 12, 4, 5, wide=True))
    wb = oracle.oracle_map_constrained(K, X, big, elig)
    assert wide == (int(wb[1][0]), int(wb[0][0]))
    # the INF-masked blocked kernel (force 1) shards the full index space
    N = 4**12
    unit = 4**3
    nb = N // unit
    best = None
    for r in range(G):
        with Mapper(0, rank=r, world=G) as m:
            m.force_path(1)
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


# ------------------------------------------------- mixed radix (feasible mappings only) --
@pytest.mark.parametrize("Q,D", [(3, 2), (4, 3), (5, 4), (6, 5), (7, 3), (6, 6), (5, 7), (5, 8), (8, 4), (9, 3)])
def test_mixed_radix_random_and_ties(torch_cuda, mapper, Q, D):
    """The mixed-radix kernel (auto for masked calls) == the constrained oracle, bit-exact,
    on random and tie-heavy tables, with pins / masks / bits >= D / zero masks, batched."""
    torch = torch_cuda
    E = 40
    for seed, maker in ((Q * 100 + D, workloads.random_tables), (Q * 100 + D + 1, workloads.small_int_tables)):
        K, X = maker(seed, E, Q, D)
        base, elig = random_constraints(seed + 7, E, Q, D, pin_frac=0.35)
        elig[::5, 0] = np.where(elig[::5, 0] != 0, elig[::5, 0] | np.uint16(1 << 15), 0)  # bits >= D: ignored
        elig[1::7, :] = 0                   # every queue on any device
        for b in (base, None):
            want = oracle.oracle_map_constrained(K, X, b, elig)
            check(run(torch, mapper, K, X, b, elig), want, f"Q={Q} D={D} {maker.__name__}")
            assert mapper.launch_info()["path"] == "mixed_u32"


@pytest.mark.parametrize("Q,D", [(4, 3), (6, 4), (9, 5), (8, 8)])
def test_mixed_radix_pins_everywhere(torch_cuda, mapper, Q, D):
    """Every pinned-queue count, including all queues pinned (a single feasible mapping: the
    reduced problem is padded with zero-cost virtual inner queues) and pins after the inner
    queues (their digits are the least significant)."""
    torch = torch_cuda
    rng = np.random.default_rng(Q * D)
    K, X = workloads.random_tables(Q + D, Q + 1, Q, D, hi=1 << 16)
    base = rng.integers(0, 1 << 16, size=(Q + 1, D), dtype=np.uint64)
    elig = np.zeros((Q + 1, Q), np.uint16)
    for e in range(Q + 1):  # epoch e pins e queues (a random subset), masks two more
        pin = rng.permutation(Q)[:e]
        elig[e, pin] = (1 << rng.integers(0, D, size=e)).astype(np.uint16)
        rest = [q for q in range(Q) if q not in set(pin.tolist())][:2]
        for q in rest:
            elig[e, q] = np.uint16(int(rng.integers(1, 1 << D)) | (1 << int(rng.integers(0, D))))
    want = oracle.oracle_map_constrained(K, X, base, elig)
    check(run(torch, mapper, K, X, base, elig), want, f"pins Q={Q} D={D}")
    check(run(torch, mapper, K, X, base, elig, 8), want, f"pins Q={Q} D={D} forced")


def test_mixed_radix_cfg5_feasible_work(torch_cuda, mapper):
    """cfg5 (12 x 8) with 3 pinned and 3 masked queues: the mixed-radix kernel scores the
    feasible space (<= 8^9 leaves here instead of 8^12) and equals the oracle (which also
    enumerates only what the masks allow, one by one) and the INF-masked full-space kernel."""
    torch = torch_cuda
    K, X = workloads.cfg5()
    base, elig = workloads.constraints(77, 1, 12, 8)
    elig[0] = 0
    elig[0, [1, 5, 10]] = [1 << 3, 1 << 0, 1 << 6]          # pinned
    elig[0, [2, 7, 11]] = [0b00110110, 0b11000001, 0b0111]  # masked (queue 11 is inner)
    want = pinned_reduced_oracle(K, X, base, elig)
    check(run(torch, mapper, K, X, base, elig), want, "cfg5 constrained")
    assert mapper.launch_info()["path"] == "mixed_u32"
    check(run(torch, mapper, K, X, base, elig, 1), want, "cfg5 constrained full space")
    # a smaller space the oracle enumerates in full (10 x 8 = 1.1e9 mappings, one by one)
    K10, X10, b10, e10 = K[:, :10], X[:, :10], base, elig[:, :10].copy()
    want10 = oracle.oracle_map_constrained(K10, X10, b10, e10)
    check(run(torch, mapper, K10, X10, b10, e10), want10, "10 x 8 constrained")
    assert (pinned_reduced_oracle(K10, X10, b10, e10)[0] == want10[0]).all()


def pinned_reduced_oracle(K, X, base, elig):
    """The constrained oracle on the reduced problem of one epoch: every pinned queue's cost
    moved into its device's base load and the queue removed (test_oracle_constrained.py pins
    this equivalence, P12), then its digit re-inserted into the returned index. Lets the
    oracle check full cfg5-sized constrained searches in a fraction of a second."""
    E, Q, D = K.shape
    assert E == 1
    full = (1 << D) - 1
    m = [(int(v) & full) if int(v) else full for v in elig[0]]
    pins = {q: m[q].bit_length() - 1 for q in range(Q) if bin(m[q]).count("1") == 1}
    keep = [q for q in range(Q) if q not in pins]
    b = (np.zeros(D, np.uint64) if base is None else base[0].astype(np.uint64)).copy()
    for q, d in pins.items():
        b[d] += K[0, q, d] + X[0, q, d]
    if keep:
        i, ms, mp = oracle.oracle_map_constrained(K[:, keep], X[:, keep], b[None], elig[:, keep])
        sub = list(mp[0])
    else:
        ms = np.array([int(b.max())], np.uint64)
        sub = []
    digits = np.zeros(Q, np.uint8)
    it = iter(sub)
    for q in range(Q):
        digits[q] = pins[q] if q in pins else next(it)
    idx = sum(int(digits[q]) * D ** (Q - 1 - q) for q in range(Q))
    return np.array([idx], np.uint64), np.asarray(ms, np.uint64).reshape(1), digits[None]


def test_static_policy_baseline(torch_cuda, mapper):
    """SCHED_AUTO_STATIC: the GPU's hint-based mappings equal the
    policy oracle's (with and without eligible masks); scored through mcl_score_mappings they
    never beat the mapper's optimum, and do worse on most epochs."""
    from oracle import policies

    torch = torch_cuda
    K, X = workloads.cfg2(E=2000, seed=31)
    E, Q, D = K.shape
    hints = workloads.static_hints(K, X)
    score = workloads.static_device_scores(D)
    _, elig = random_constraints(31, E, Q, D, pin_frac=0.0)
    for el in (None, elig):
        want = policies.static_mapping(hints, score, el)
        got = mapper.static_mappings(dev(torch, hints), dev(torch, score), None if el is None else dev(torch, el))
        assert (got.cpu().numpy() == want).all()
        assert (mapper.static_mappings(hints, score, el) == want).all()  # host buffers
    st = mapper.score_mappings(dev(torch, K), dev(torch, X), dev(torch, want)).cpu().numpy()
    assert (st == np.array([oracle.oracle_score(K[e], X[e], want[e]) for e in range(E)], np.uint64)).all()
    opt = oracle.oracle_map(K, X)[1]
    assert (opt <= st).all() and (opt < st).mean() > 0.5
    with pytest.raises(MclError):
        mapper.static_mappings(np.full((1, Q), 3, np.uint8), score)  # hint >= classes
    with pytest.raises(MclError):
        mapper.static_mappings(hints[:1], score, np.full((1, Q), 1 << 15, np.uint16))  # no device


@pytest.mark.parametrize("D", [6, 7, 8])
def test_mixed_radix_u64_wide_devices(torch_cuda, mapper, D):
    """64-bit loads on the mixed-radix kernel for D = 6..8 (the builds with register
    spills): base loads near 2^40 force the rerun; every epoch equals the oracle."""
    torch = torch_cuda
    Q = 6
    K, X = workloads.random_tables(90 + D, 12, Q, D, hi=1 << 20)
    base, elig = random_constraints(91 + D, 12, Q, D, pin_frac=0.3)
    big = base + np.uint64(1 << 40)
    want = oracle.oracle_map_constrained(K, X, big, elig)
    check(run(torch, mapper, K, X, big, elig), want, f"u64 D={D}")
    assert mapper.launch_info()["path"] == "mixed_u64"


def test_mixed_radix_batches_beyond_one_wave(torch_cuda, mapper):
    """Batches larger than one wave of CTAs (whole-CTA epochs, then the tail epochs split over
    several CTAs merged through scratch) on the mixed-radix kernel == the oracle."""
    torch = torch_cuda
    E, Q, D = 700, 7, 4
    K, X = workloads.random_tables(123, E, Q, D, hi=1 << 18)
    base, elig = random_constraints(124, E, Q, D, pin_frac=0.3)
    want = oracle.oracle_map_constrained(K, X, base, elig)
    check(run(torch, mapper, K, X, base, elig, 8), want, "mixed E=700")
    assert mapper.launch_info()["path"] == "mixed_u32"


# ------------------------------- mixed radix, one warp per epoch (batched constrained) ----
@pytest.mark.parametrize("Q,D", [(3, 2), (4, 3), (5, 4), (6, 5), (7, 3), (6, 6), (5, 7), (5, 8), (8, 4), (9, 3),
                                 (12, 3), (10, 4), (18, 2)])
def test_mixed_warp_random_and_ties(torch_cuda, mapper, Q, D):
    """The warp-per-epoch mixed-radix kernel (forced, path 9) == the constrained oracle,
    bit-exact, on random and tie-heavy tables with pins, masks, bits >= D and zero masks."""
    torch = torch_cuda
    E = 70
    for seed, maker in ((Q * 100 + D + 5, workloads.random_tables), (Q * 100 + D + 6, workloads.small_int_tables)):
        K, X = maker(seed, E, Q, D)
        base, elig = random_constraints(seed + 9, E, Q, D, pin_frac=0.35)
        elig[::5, 0] = np.where(elig[::5, 0] != 0, elig[::5, 0] | np.uint16(1 << 15), 0)
        elig[1::7, :] = 0
        for b in (base, None):
            want = oracle.oracle_map_constrained(K, X, b, elig)
            check(run(torch, mapper, K, X, b, elig, 9), want, f"warp Q={Q} D={D} {maker.__name__}")
            assert mapper.launch_info()["path"] == "mixed_warp_u32"


@pytest.mark.parametrize("Q,D", [(4, 3), (6, 4), (9, 5), (8, 8)])
def test_mixed_warp_pins_everywhere(torch_cuda, mapper, Q, D):
    """Every pinned-queue count on the warp kernel, including all queues pinned."""
    torch = torch_cuda
    rng = np.random.default_rng(Q * D + 1)
    K, X = workloads.random_tables(Q + D + 1, Q + 1, Q, D, hi=1 << 16)
    base = rng.integers(0, 1 << 16, size=(Q + 1, D), dtype=np.uint64)
    elig = np.zeros((Q + 1, Q), np.uint16)
    for e in range(Q + 1):
        pin = rng.permutation(Q)[:e]
        elig[e, pin] = (1 << rng.integers(0, D, size=e)).astype(np.uint16)
    want = oracle.oracle_map_constrained(K, X, base, elig)
    check(run(torch, mapper, K, X, base, elig, 9), want, f"warp pins Q={Q} D={D}")


def test_mixed_warp_auto_batch_u64_and_errors(torch_cuda, mapper):
    """A cfg2-shaped constrained batch (8 x 4, 25 % pinned + 25 % masked) takes the warp
    kernel automatically; an epoch whose bound needs 64 bits reruns the call on the 64-bit
    CTA kernel; input errors raise as on every path."""
    torch = torch_cuda
    E, Q, D = 1000, 8, 4
    K, X = workloads.random_tables(131, E, Q, D, hi=1 << 18)
    base, elig = workloads.constraints(132, E, Q, D, pin_frac=0.25, mask_frac=0.25)
    want = oracle.oracle_map_constrained(K, X, base, elig)
    check(run(torch, mapper, K, X, base, elig), want, "auto warp")
    assert mapper.launch_info()["path"] == "mixed_warp_u32"
    big = base.copy()
    big[E // 2] += np.uint64(1 << 40)  # one epoch over 2^32: the whole call reruns wide
    want_big = oracle.oracle_map_constrained(K, X, big, elig)
    check(run(torch, mapper, K, X, big, elig), want_big, "auto warp -> u64")
    assert mapper.launch_info()["path"] == "mixed_u64"
    Kr = K.copy()
    Kr[E - 1, 3, 2] = 1 << 48
    with pytest.raises(MclError) as e:
        run(torch, mapper, Kr, X, base, elig)
    assert e.value.status == MCL_E_RANGE
    bad = elig.copy()
    bad[7, 2] = 1 << 5  # no eligible device below D
    with pytest.raises(MclError) as e:
        run(torch, mapper, K, X, base, bad)
    assert e.value.status == MCL_E_INVAL
