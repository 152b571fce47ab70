"""GPU parity of the pipelined staging of host-resident batches (include/mcl_ext.h
mcl_set_pipeline_chunks): every chunk's H2D copy, search and D2H copy on rotating streams.
The results must equal the oracle's (and the unpipelined call's) bit for bit, for any chunk
count, ragged chunk sizes, every batched kernel path, with and without the mapping output,
and through the 64-bit rerun and range errors. Run with ``pytest -m gpu``.
"""
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


def host_call(torch, m, K, X, with_mapping=True, pinned=True):
    E, Q, _ = K.shape
    Kh, Xh = torch.from_numpy(np.ascontiguousarray(K)), torch.from_numpy(np.ascontiguousarray(X))
    idx = torch.empty(E, dtype=torch.uint64)
    ms = torch.empty(E, dtype=torch.uint64)
    mp = torch.empty((E, Q), dtype=torch.uint8) if with_mapping else None
    if pinned:
        Kh, Xh, idx, ms = Kh.pin_memory(), Xh.pin_memory(), idx.pin_memory(), ms.pin_memory()
        mp = mp.pin_memory() if mp is not None else None
    m.map_queues_into(Kh, Xh, idx, mp, ms)
    return idx.numpy(), (mp.numpy() if mp is not None else None), ms.numpy()


def check(got, want, ctx, with_mapping=True):
    gi, gmp, gms = got
    wi, wms, wmp = want
    bad = np.nonzero((gi != wi) | (gms != wms))[0]
    assert bad.size == 0, f"{ctx}: {bad.size} epochs differ, first {bad[:5]}"
    if with_mapping:
        assert (gmp == wmp).all(), ctx


@pytest.mark.parametrize("chunks", [2, 3, 5, 7])
def test_pipelined_chunks_cfg2_shape(torch_cuda, mapper, chunks):
    """8 x 4 batches (warp-per-epoch / CTA-per-epoch kernels per chunk), ragged chunk sizes."""
    K, X = workloads.cfg2(E=3001, seed=31)
    want = oracle.oracle_map(K, X)
    mapper.set_pipeline_chunks(chunks)
    try:
        got = host_call(torch_cuda, mapper, K, X)
        assert mapper.launch_info()["chunks"] == chunks
    finally:
        mapper.set_pipeline_chunks(0)
    check(got, want, f"chunks={chunks}")


def test_pipelined_small_kernel_and_pageable(torch_cuda, mapper):
    """2 x 3 batches (thread-per-epoch kernel per chunk); pageable host buffers too."""
    K, X = workloads.cfg3(E=200_003, seed=32)
    want = oracle.oracle_map(K, X)
    mapper.set_pipeline_chunks(6)
    try:
        for pinned in (True, False):
            got = host_call(torch_cuda, mapper, K, X, pinned=pinned)
            assert mapper.launch_info()["chunks"] == 6
            check(got, want, f"cfg3 pinned={pinned}")
    finally:
        mapper.set_pipeline_chunks(0)


def test_pipelined_auto_matches_unpipelined(torch_cuda, mapper):
    """The automatic chunking of a full cfg2 batch from pageable buffers (4 chunks of one
    wave or more), the unpipelined staged call, and the zero-copy call from pinned buffers
    (the warp-per-epoch kernel reads them in place) return identical outputs; no mapping
    output (NULL) works."""
    K, X = workloads.cfg2()
    got_auto = host_call(torch_cuda, mapper, K, X, pinned=False)
    assert mapper.launch_info()["chunks"] > 1
    mapper.set_pipeline_chunks(1)
    try:
        got_off = host_call(torch_cuda, mapper, K, X, pinned=False)
        assert mapper.launch_info()["chunks"] == 0
    finally:
        mapper.set_pipeline_chunks(0)
    got_zc = host_call(torch_cuda, mapper, K, X, pinned=True)
    assert mapper.launch_info()["chunks"] == 0 and mapper.launch_info()["path"] == "batch_u32"
    for a, b, c in zip(got_auto, got_off, got_zc):
        assert (a == b).all() and (a == c).all()
    check(got_auto, oracle.oracle_map(K, X), "cfg2 auto")
    gi, _, gms = host_call(torch_cuda, mapper, K, X, with_mapping=False)
    assert (gi == got_auto[0]).all() and (gms == got_auto[2]).all()


def test_pipelined_u64_rerun_and_range_error(torch_cuda, mapper):
    """A chunk whose bound needs 64-bit loads makes the whole call rerun unpipelined (same
    outputs as the oracle); an entry >= 2^48 in any chunk fails the call, and the next call
    is exact."""
    K, X = workloads.random_tables(33, 64, 8, 4)
    K[50] = np.random.default_rng(2).integers(1 << 46, 1 << 47, size=(8, 4), dtype=np.uint64)
    mapper.set_pipeline_chunks(4)
    try:
        got = host_call(torch_cuda, mapper, K, X)
        assert mapper.launch_info()["path"] == "blocked_u64"
        assert mapper.launch_info()["chunks"] == 0
        check(got, oracle.oracle_map(K, X), "u64 rerun")
        K2, X2 = workloads.random_tables(34, 64, 8, 4)
        X2[40, 1, 2] = 1 << 48
        with pytest.raises(MclError) as ei:
            host_call(torch_cuda, mapper, K2, X2)
        assert ei.value.status == MCL_E_RANGE
        X2[40, 1, 2] = 9
        got = host_call(torch_cuda, mapper, K2, X2)
        check(got, oracle.oracle_map(K2, X2), "after range error")
    finally:
        mapper.set_pipeline_chunks(0)


def test_pipelined_more_chunks_than_epochs(torch_cuda, mapper):
    K, X = workloads.random_tables(35, 3, 9, 3)
    mapper.set_pipeline_chunks(16)
    try:
        got = host_call(torch_cuda, mapper, K, X)
        assert mapper.launch_info()["chunks"] == 3
    finally:
        mapper.set_pipeline_chunks(0)
    check(got, oracle.oracle_map(K, X), "E=3, 16 chunks requested")


def test_pipelined_on_external_stream_with_timing(torch_cuda):
    """A handle on a caller's stream: pipelined host calls interleaved with device calls on
    the same handle, kernel timing on (the span from the first chunk's search to the last's
    is reported), every result exact."""
    torch = torch_cuda
    stream = torch.cuda.Stream()
    K, X = workloads.cfg2(E=2600, seed=36)
    want = oracle.oracle_map(K, X)
    Kd, Xd = torch.from_numpy(K).cuda(), torch.from_numpy(X).cuda()
    with Mapper(0, stream=stream.cuda_stream) as m:
        m.set_timing(True)
        m.set_pipeline_chunks(3)
        for rep in range(3):
            got = host_call(torch, m, K, X)
            assert m.launch_info()["chunks"] == 3
            assert m.last_kernel_time_ms()[0] > 0
            check(got, want, f"pipelined rep {rep}")
            with torch.cuda.stream(stream):
                idx, mp, ms = m.map_queues(Kd, Xd)
                stream.synchronize()
            assert (idx.cpu().numpy() == want[0]).all() and (ms.cpu().numpy() == want[1]).all()


@pytest.mark.parametrize("path", [1, 3])
def test_pipelined_chunks_share_scratch(torch_cuda, mapper, path):
    """Chunk searches that use the handle's scratch (split-epoch slots and done counters of
    the CTA-per-epoch and generic kernels) must not overlap: many small chunks, forced
    kernel path, every epoch exact."""
    K, X = workloads.cfg2(E=1500, seed=37) if path == 1 else workloads.random_tables(38, 400, 6, 3)
    want = oracle.oracle_map(K, X)
    mapper.set_pipeline_chunks(9)
    mapper.force_path(path)
    try:
        for rep in range(3):
            got = host_call(torch_cuda, mapper, K, X)
            check(got, want, f"path {path} rep {rep}")
    finally:
        mapper.force_path(0)
        mapper.set_pipeline_chunks(0)
