"""CPU model check of the fused cross-GPU exchange protocol (peer.cuh).

The device code cannot run here, so its protocol -- per-rank slabs with a signal counter, a
round counter and two alternating regions; rounds of "atomicMin into every rank's region,
signal every rank, wait for world * (R + 1) signals, read-and-reset own region"; a packed-key
round followed, when some reduced key is empty, by the two-step lexicographic rounds -- is
replayed step by step with `world` simulated ranks under random interleavings of every
shared-memory access, over sequences of calls with varying epoch counts. Every rank must get
the lexicographic minimum over ranks of (makespan, index) for every epoch of every call.

A deliberately broken variant (resetting the region when a round STARTS instead of after it
is read) must be caught, which shows the interleavings reach the races the design avoids.
"""
from __future__ import annotations

import random

import pytest

NONE = (1 << 64) - 1


class Slab:
    def __init__(self, cap):
        self.sig = 0
        self.rounds = 0
        self.reg = [[NONE] * cap, [NONE] * cap]


def rank_program(me, world, slabs, calls, ibits, out, reset_early=False):
    """Generator: one rank's sequence of calls. Yields before every shared access."""
    fit = 1 << (64 - ibits)
    for call in calls:
        cand = call[me]  # [(ms, idx)] per epoch; ms == NONE: no candidate
        E = len(cand)
        R = slabs[me].rounds

        def round_(values):
            nonlocal R
            region = R & 1
            if reset_early:  # BROKEN variant: clear own region at the start of the round
                for e in range(E):
                    yield
                    slabs[me].reg[region][e] = NONE
            for e in range(E):
                for r in range(world):
                    v = values[e]
                    if v != NONE:
                        yield
                        cur = slabs[r].reg[region][e]
                        slabs[r].reg[region][e] = min(cur, v)  # atomicMin_system
            for r in range(world):
                yield
                slabs[r].sig += 1  # atomicAdd_system after the system fence
            while True:
                yield
                if slabs[me].sig >= world * (R + 1):
                    break
            got = []
            for e in range(E):
                yield
                got.append(slabs[me].reg[region][e])
                if not reset_early:
                    slabs[me].reg[region][e] = NONE  # read-and-reset (peer_take)
            R += 1
            return got

        keys = [((ms << ibits) | idx) if ms != NONE and ms < fit else NONE for ms, idx in cand]
        got = yield from round_(keys)
        res = [None] * E
        for e, k in enumerate(got):
            if k != NONE:
                res[e] = (k >> ibits, k & ((1 << ibits) - 1))
        if any(k == NONE for k in got):
            gms = yield from round_([ms for ms, _ in cand])
            gidx = yield from round_([idx if ms == gms[e] else NONE for e, (ms, idx) in enumerate(cand)])
            res = [(gms[e], gidx[e]) for e in range(E)]
        yield
        slabs[me].rounds = R
        out[me].append(res)


def run(world, calls, ibits, seed, reset_early=False, cap=8):
    slabs = [Slab(cap) for _ in range(world)]
    out = [[] for _ in range(world)]
    progs = [rank_program(r, world, slabs, calls, ibits, out, reset_early) for r in range(world)]
    rng = random.Random(seed)
    live = list(range(world))
    steps = 0
    while live:
        i = rng.choice(live)
        try:
            next(progs[i])
        except StopIteration:
            live.remove(i)
        steps += 1
        if steps > 500_000:
            return None  # no progress: the ranks' round counts diverged (a hang on hardware)
    return out


def make_calls(seed, world, ncalls, ibits):
    rng = random.Random(seed)
    fit = 1 << (64 - ibits)
    calls = []
    for _ in range(ncalls):
        E = rng.randint(1, 6)
        big = rng.random() < 0.4  # some makespans do not fit beside the index
        call = []
        for r in range(world):
            row = []
            for e in range(E):
                if rng.random() < 0.1:
                    row.append((NONE, NONE))  # e.g. an infeasible sub-range
                    continue
                ms = rng.randint(0, 3 * fit if big else fit - 1)
                idx = r * 1000 + rng.randint(0, 999)  # disjoint shards
                row.append((ms, idx))
            call.append(row)
        calls.append(call)
    return calls


def expected(calls):
    res = []
    for call in calls:
        E = len(call[0])
        res.append([min(call[r][e] for r in range(len(call))) for e in range(E)])
    return res


@pytest.mark.parametrize("world", [1, 2, 3, 4])
def test_fused_protocol_interleavings(world):
    ibits = 60  # makespans >= 16 do not pack: the two-step rounds run often
    for seed in range(12):
        calls = make_calls(seed, world, 10, ibits)
        want = expected(calls)
        out = run(world, calls, ibits, seed)
        assert out is not None, (world, seed, "deadlock")
        for r in range(world):
            assert out[r] == want, (world, seed, r)


def test_broken_reset_is_caught():
    """Resetting a region at the start of its round (before the other ranks are known to be
    in it) loses contributions of faster ranks: some interleaving must give a wrong result,
    or ranks that disagree on the two-step decision and then wait on each other forever."""
    ibits = 60
    bad = 0
    for seed in range(40):
        calls = make_calls(seed, 3, 8, ibits)
        out = run(3, calls, ibits, seed, reset_early=True)
        if out is None or any(o != expected(calls) for o in out):
            bad += 1
    assert bad > 0
