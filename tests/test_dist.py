"""Multi-process (gloo, world 2 and 3) check of the sharded search protocol on CPU.

The product's N > 1 path (include/mcl.h "Sharding"): every rank searches the contiguous
block range [floor(r*nb/G), floor((r+1)*nb/G)) of every epoch's index space, packs
key = makespan << ceil(log2 N) | index, and one all-reduce(MIN) gives every rank the global
lexicographic minimum. Here the per-rank search is the oracle on that index range and the
collective is gloo, so the protocol (ranges, packing, min-reduce, bit-identical results
for every world size, max-over-ranks timing) is exercised without a GPU.
"""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _index_bits(n):
    return int(n - 1).bit_length()


def _worker(rank, world, port, K, X, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle

    E, Q, D = K.shape
    N = D**Q
    unit = D**3
    nb = N // unit
    lo, hi = (nb * rank // world) * unit, (nb * (rank + 1) // world) * unit
    ib = _index_bits(N)
    keys = []
    for e in range(E):
        idx, ms, _ = oracle.oracle_map(K[e], X[e], lo=lo, hi=hi, threads=1)
        assert lo <= int(idx[0]) < hi
        keys.append((int(ms[0]) << ib) | int(idx[0]))
    t = torch.tensor(keys, dtype=torch.int64)
    dist.all_reduce(t, op=dist.ReduceOp.MIN)
    elapsed = torch.tensor([float(rank + 1)], dtype=torch.float64)  # stand-in per-rank time
    dist.all_reduce(elapsed, op=dist.ReduceOp.MAX)
    q.put((rank, t.tolist(), float(elapsed[0])))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_sharded_protocol_gloo(world):
    from paper_conf_cluster_ajipbf15_b200 import workloads

    K, X = workloads.small_int_tables(31, 3, 8, 3, hi=5)  # heavy ties across shard borders
    K2, X2 = workloads.random_tables(32, 2, 8, 3, hi=1 << 16)
    K, X = np.concatenate([K, K2]), np.concatenate([X, X2])
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, K, X, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    import oracle

    idx, ms, _ = oracle.oracle_map(K, X)
    ib = _index_bits(3**8)
    want = [(int(m) << ib) | int(i) for i, m in zip(idx, ms)]
    for rank, keys, elapsed in out:
        assert keys == want  # every rank holds the identical global result
        assert elapsed == float(world)  # max over ranks


def test_shard_ranges_cover_exactly():
    for nb in (1, 5, 64, 4**13, 8**9):
        for world in (1, 2, 3, 7, 8, 4096):
            cuts = [nb * r // world for r in range(world + 1)]
            assert cuts[0] == 0 and cuts[-1] == nb
            assert all(a <= b for a, b in zip(cuts, cuts[1:]))
            sizes = [b - a for a, b in zip(cuts, cuts[1:])]
            assert max(sizes) - min(sizes) <= 1


def _worker_constrained(rank, world, port, K, X, base, elig, q):
    """A masked call's shard: the oracle on this rank's range of the FEASIBLE enumeration
    (tests/shard_ranges.py; include/mcl.h, reading R21), then the same packed-key min."""
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle
    from shard_ranges import mixed_shard_ranges

    E, Q, D = K.shape
    ib = _index_bits(D**Q)
    keys = []
    for e in range(E):
        lo, hi = mixed_shard_ranges(elig[e], Q, D, world)[rank]
        key = (1 << 63) - 1  # no feasible mapping in this shard
        if lo < hi:
            try:
                idx, ms, _ = oracle.oracle_map_constrained(K[e], X[e], base[e], elig[e], lo=lo, hi=hi, threads=1)
                key = (int(ms[0]) << ib) | int(idx[0])
            except oracle.OracleError:
                pass
        keys.append(key)
    t = torch.tensor(keys, dtype=torch.int64)
    dist.all_reduce(t, op=dist.ReduceOp.MIN)
    q.put((rank, t.tolist()))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_sharded_feasible_enumeration_gloo(world):
    """Masked calls shard the feasible (mixed-radix) enumeration: the min over ranks of the
    shards' (makespan, full index) keys is the global constrained optimum, on tie-heavy and
    random tables with pinned and masked queues."""
    import sys

    sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
    from paper_conf_cluster_ajipbf15_b200 import workloads

    K, X = workloads.small_int_tables(41, 3, 8, 4, hi=4)
    K2, X2 = workloads.random_tables(42, 3, 8, 4, hi=1 << 16)
    K, X = np.concatenate([K, K2]), np.concatenate([X, X2])
    base, elig = workloads.constraints(43, 6, 8, 4, pin_frac=0.3, mask_frac=0.3)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker_constrained, args=(r, world, port, K, X, base, elig, q))
             for r in range(world)]
    for p in procs:
        p.start()
    out = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    import oracle

    idx, ms, _ = oracle.oracle_map_constrained(K, X, base, elig)
    ib = _index_bits(4**8)
    want = [(int(m) << ib) | int(i) for i, m in zip(idx, ms)]
    for rank, keys in out:
        assert keys == want
