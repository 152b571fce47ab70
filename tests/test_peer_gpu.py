"""Fused cross-GPU exchange (include/mcl.h mcl_peer_export / mcl_peer_import)
on the GPU box's single B200.

* world = 1: the handle exchanges with its own slab, so every exchange round (atomicMin into
  the slab, system fence, signal, acquire-wait, read-and-reset) runs on real hardware inside
  the search kernel; results must equal the oracle's, across many consecutive calls (the
  round counter and the two alternating regions), through the packed-key round and the
  two-step rounds, the 64-bit rerun, the generic kernel and the constrained variant.
* world = 2 on ONE GPU: two processes, each a rank with its own slab mapped into the other
  through CUDA IPC; their kernels time-slice on the device, and the in-kernel barrier must
  still complete (it has a timeout, so a failure reports an error instead of hanging).
"""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest

import oracle
from conftest import cuda_available
from paper_conf_cluster_ajipbf15_b200 import workloads
from paper_conf_cluster_ajipbf15_b200.mcl import Mapper, MclError

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def torch_cuda():
    if not cuda_available():
        pytest.fail("no CUDA device: the -m gpu tests must run on a GPU box")
    import torch

    return torch


def dev(torch, a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def _cases():
    rng = np.random.default_rng(77)
    big = rng.integers(1 << 46, 1 << 47, size=(3, 9, 4), dtype=np.uint64)  # no key packs
    wide = rng.integers(1 << 34, 1 << 36, size=(2, 8, 4), dtype=np.uint64)  # 64-bit loads, packs
    return [
        ("cfg4 Q=12 blocked u32", *workloads.cfg4(seed=4, Q=12)),
        ("two-step", big, np.zeros_like(big)),
        ("u64 rerun", wide, np.zeros_like(wide)),
        ("generic D=10", *workloads.random_tables(5, 2, 5, 10, hi=1 << 20)),
        ("generic Q=2", *workloads.random_tables(6, 7, 2, 3, hi=1 << 20)),
        ("batch of 64 ties", *workloads.small_int_tables(8, 64, 7, 3, hi=4)),
    ]


def test_fused_exchange_single_rank(torch_cuda):
    torch = torch_cuda
    with Mapper(0, rank=0, world=1) as m:
        m.peer_import([m.peer_export(max_epochs=64)], timeout_ms=10_000)
        cases = _cases()
        for rep in range(3):  # consecutive calls: round counter, alternating regions
            for name, K, X in cases:
                want = oracle.oracle_map(K, X)
                i, mp, ms = m.map_queues(dev(torch, K), dev(torch, X))
                info = m.launch_info()
                assert info["fused_exchange"] and info["launches"] == 1, (name, info)
                assert info["two_step"] == (name == "two-step"), (name, info)
                assert (i.cpu().numpy() == want[0]).all(), (name, rep)
                assert (ms.cpu().numpy() == want[1]).all(), (name, rep)
                assert (mp.cpu().numpy() == want[2]).all(), (name, rep)
        # constrained variant through the same exchange
        K, X = workloads.cfg2(E=16, seed=9)
        base, elig = workloads.constraints(3, *K.shape)
        want = oracle.oracle_map_constrained(K, X, base, elig)
        i, mp, ms = m.map_queues_constrained(dev(torch, K), dev(torch, X), dev(torch, base), dev(torch, elig))
        assert m.launch_info()["fused_exchange"]
        assert (i.cpu().numpy() == want[0]).all() and (ms.cpu().numpy() == want[1]).all()
        # more epochs than the slabs hold: plain single-GPU path (no communicator)
        K, X = workloads.cfg2(E=65, seed=10)
        i, mp, ms = m.map_queues(dev(torch, K), dev(torch, X))
        assert not m.launch_info()["fused_exchange"]
        assert (i.cpu().numpy() == oracle.oracle_map(K, X)[0]).all()


def test_fused_exchange_errors(torch_cuda):
    with Mapper(0, rank=0, world=1) as m:
        with pytest.raises(MclError):
            m.peer_import([bytes(64)])  # before export
        with pytest.raises(MclError):
            m.peer_export(max_epochs=0)
        m.peer_import([m.peer_export(max_epochs=4)])
        # an input error skips the exchange on every rank; the next call still works
        K = np.full((1, 4, 3), 1 << 50, np.uint64)
        with pytest.raises(MclError):
            m.map_queues(K, np.zeros_like(K))
        K, X = workloads.cfg1_npb("FT")
        i, mp, ms = m.map_queues(K, X)
        assert int(i[0]) == int(oracle.oracle_map(K, X)[0][0])
        # pinned host buffers of a small call are used in place (zero-copy) by the search
        # kernel and its in-kernel exchange / decode
        import torch

        Kp, Xp = torch.from_numpy(K).pin_memory(), torch.from_numpy(X).pin_memory()
        ip = torch.empty(1, dtype=torch.uint64).pin_memory()
        mp_ = torch.empty((1, 4), dtype=torch.uint8).pin_memory()
        msp = torch.empty(1, dtype=torch.uint64).pin_memory()
        m.map_queues_into(Kp, Xp, ip, mp_, msp)
        want = oracle.oracle_map(K, X)
        assert m.launch_info()["fused_exchange"]
        assert int(ip[0]) == int(want[0][0]) and int(msp[0]) == int(want[1][0]) and (mp_.numpy() == want[2]).all()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _rank(rank, world, port, q):
    try:
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        import torch
        import torch.distributed as dist

        dist.init_process_group("gloo", rank=rank, world_size=world)
        out = []
        with Mapper(0, rank=rank, world=world) as m:
            m.connect_peers(max_epochs=8, timeout_ms=60_000)
            for name, K, X in _cases():
                if K.shape[0] > 8:
                    continue
                i, mp, ms = m.map_queues(dev(torch, K), dev(torch, X))
                out.append((name, i.cpu().numpy(), ms.cpu().numpy(), mp.cpu().numpy(),
                            m.launch_info()["fused_exchange"]))
            # masked calls: each rank searches its piece of the FEASIBLE enumeration
            # (mixed-radix kernel) and the fused exchange combines them
            Kc, Xc = workloads.cfg4(seed=6, Q=11)
            bc, ec = workloads.constraints(21, 1, 11, 4)
            i, mp, ms = m.map_queues_constrained(dev(torch, Kc), dev(torch, Xc), dev(torch, bc), dev(torch, ec))
            out.append(("constrained", i.cpu().numpy(), ms.cpu().numpy(), mp.cpu().numpy(),
                        m.launch_info()["fused_exchange"] and m.launch_info()["path"] == "mixed_u32"))
            # more epochs than the slabs hold and no communicator: an error, never this
            # rank's shard-local argmin presented as the global result
            K, X = workloads.small_int_tables(8, 64, 7, 3, hi=4)
            try:
                m.map_queues(dev(torch, K), dev(torch, X))
                over = "returned"
            except MclError as exc:
                over = exc.status
            out.append(("over max_epochs", over))
            dist.barrier()
        dist.destroy_process_group()
        q.put((rank, out, None))
    except Exception as e:  # report instead of hanging the parent
        q.put((rank, None, repr(e)))


def test_fused_exchange_two_ranks_one_gpu(torch_cuda):
    import torch.multiprocessing as mp

    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_rank, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=600) for _ in range(2)]
    for p in procs:
        p.join(timeout=120)
    errs = [e for _, _, e in res if e]
    if errs and all("cudaIpcOpenMemHandle" in e for e in errs):
        pytest.skip(f"CUDA IPC between two processes on one device unavailable: {errs[0]}")
    assert not errs, errs
    want = {name: oracle.oracle_map(K, X) for name, K, X in _cases() if K.shape[0] <= 8}
    Kc, Xc = workloads.cfg4(seed=6, Q=11)
    bc, ec = workloads.constraints(21, 1, 11, 4)
    want["constrained"] = oracle.oracle_map_constrained(Kc, Xc, bc, ec)
    from paper_conf_cluster_ajipbf15_b200.mcl import MCL_E_INVAL

    for rank, out, _ in res:
        assert out[-1] == ("over max_epochs", MCL_E_INVAL), (rank, out[-1])
        out = out[:-1]
        assert len(out) == len(want)
        for name, i, ms, mp_, fused in out:
            assert fused, (rank, name)
            assert (i == want[name][0]).all() and (ms == want[name][1]).all(), (rank, name)
            assert (mp_ == want[name][2]).all(), (rank, name)
