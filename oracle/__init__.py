"""CPU oracle for MultiCL's device-mapper search -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package. The product package
(``paper_conf_cluster_ajipbf15_b200``) never imports it, and it imports nothing from the
product: the two share no code. See ``oracle/oracle.c`` for the definition it follows
(PAPER.md L1042-1056 SS V.A "Device Mapper"; L2106-2118 SS VI.B.1 aggregate cost).

Parity status: pinned. ``tests/test_oracle.py`` pins it against the hand-solved cases in
``tests/golden/hand_cases.json``, closed forms (D=1, Q=1, all-equal),
a subset-sum DP (D=2 identical devices), a load-vector DP (D<=3), lower/upper bounds,
metamorphic relations and ``oracle.tiny`` (``itertools.product`` + ``min`` semantics).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRCS = [os.path.join(_HERE, "oracle.c"), os.path.join(_HERE, "costs.c")]
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile oracle.c + costs.c into oracle/liboracle.so with gcc (plain C11 + pthreads;
    no fused multiply-add, so the fp64 cost-model arithmetic is rounded as written)."""
    stale = not os.path.exists(_LIB) or any(os.path.getmtime(_LIB) < os.path.getmtime(s) for s in _SRCS)
    if force or stale:
        subprocess.check_call(
            ["gcc", "-O2", "-std=c11", "-ffp-contract=off", "-fPIC", "-shared", "-pthread", "-o", _LIB]
            + _SRCS + ["-lm"]
        )
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        lib.oracle_map.restype = ctypes.c_int
        lib.oracle_map.argtypes = [
            ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint64,
            ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_int,
            ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
        ]
        lib.oracle_score.restype = ctypes.c_uint64
        lib.oracle_score.argtypes = [
            ctypes.c_uint32, ctypes.c_uint32, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
        ]
        lib.oracle_map_constrained.restype = ctypes.c_int
        lib.oracle_map_constrained.argtypes = [
            ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_void_p, ctypes.c_void_p,
            ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_int,
            ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
        ]
        lib.oracle_build_costs.restype = ctypes.c_int
        lib.oracle_build_costs.argtypes = [
            ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_uint32,
            ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
            ctypes.c_void_p, ctypes.c_uint32, ctypes.c_void_p, ctypes.c_uint32, ctypes.c_void_p,
            ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint32, ctypes.c_void_p, ctypes.c_void_p,
        ]
        lib.oracle_score_base.restype = ctypes.c_uint64
        lib.oracle_score_base.argtypes = [
            ctypes.c_uint32, ctypes.c_uint32, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
            ctypes.c_void_p,
        ]
        _lib = lib
    return _lib


class OracleError(RuntimeError):
    def __init__(self, code: int):
        super().__init__(f"oracle_map returned {code}")
        self.code = code


def default_threads() -> int:
    return len(os.sched_getaffinity(0))


def oracle_map(K, X, lo: int = 0, hi: int = 0, threads: int | None = None):
    """Brute-force argmin per epoch.

    K, X: integer arrays of shape [E, Q, D] or [Q, D] (ns). Returns (index[E], makespan[E],
    mapping[E, Q]) as numpy arrays (uint64, uint64, uint8). ``lo``/``hi`` restrict the search
    to mapping indices [lo, hi) in every epoch (hi == 0: full range).
    """
    K = np.ascontiguousarray(K, dtype=np.uint64)
    X = np.ascontiguousarray(X, dtype=np.uint64)
    single = K.ndim == 2
    if single:
        K = K[None]
        X = X[None]
    if K.shape != X.shape or K.ndim != 3:
        raise ValueError("K and X must both be [E, Q, D]")
    E, Q, D = K.shape
    idx = np.zeros(E, dtype=np.uint64)
    ms = np.zeros(E, dtype=np.uint64)
    mp = np.zeros((E, Q), dtype=np.uint8)
    rc = _load().oracle_map(
        Q, D, E, K.ctypes.data, X.ctypes.data, lo, hi,
        threads if threads else default_threads(),
        idx.ctypes.data, ms.ctypes.data, mp.ctypes.data,
    )
    if rc != 0:
        raise OracleError(rc)
    return idx, ms, mp


def oracle_score(K, X, mapping) -> int:
    """Makespan of one mapping (device tuple) for one epoch's [Q, D] tables."""
    K = np.ascontiguousarray(K, dtype=np.uint64)
    X = np.ascontiguousarray(X, dtype=np.uint64)
    m = np.ascontiguousarray(mapping, dtype=np.uint8)
    Q, D = K.shape
    return int(_load().oracle_score(Q, D, K.ctypes.data, X.ctypes.data, m.ctypes.data))


def oracle_map_constrained(K, X, base=None, elig=None, lo: int = 0, hi: int = 0,
                           threads: int | None = None):
    """Constrained brute force (NEXT-3): ``base`` [E, D] pre-existing device loads (or None),
    ``elig`` [E, Q] uint16 eligible-device masks (bit d = device d, 0 = any; or None).
    Returns (index[E], makespan[E], mapping[E, Q]); raises OracleError(-1) if an epoch has
    no feasible mapping."""
    K = np.ascontiguousarray(K, dtype=np.uint64)
    X = np.ascontiguousarray(X, dtype=np.uint64)
    if K.ndim == 2:
        K, X = K[None], X[None]
        base = None if base is None else np.asarray(base)[None]
        elig = None if elig is None else np.asarray(elig)[None]
    E, Q, D = K.shape
    b = None if base is None else np.ascontiguousarray(base, dtype=np.uint64).reshape(E, D)
    m = None if elig is None else np.ascontiguousarray(elig, dtype=np.uint16).reshape(E, Q)
    idx = np.zeros(E, dtype=np.uint64)
    ms = np.zeros(E, dtype=np.uint64)
    mp = np.zeros((E, Q), dtype=np.uint8)
    rc = _load().oracle_map_constrained(
        Q, D, E, K.ctypes.data, X.ctypes.data, None if b is None else b.ctypes.data,
        None if m is None else m.ctypes.data, lo, hi, threads if threads else default_threads(),
        idx.ctypes.data, ms.ctypes.data, mp.ctypes.data,
    )
    if rc != 0:
        raise OracleError(rc)
    return idx, ms, mp


def oracle_score_base(K, X, base, mapping) -> int:
    """Makespan of one mapping for one epoch's [Q, D] tables with device base loads [D]."""
    K = np.ascontiguousarray(K, dtype=np.uint64)
    X = np.ascontiguousarray(X, dtype=np.uint64)
    mpg = np.ascontiguousarray(mapping, dtype=np.uint8)
    Q, D = K.shape
    b = None if base is None else np.ascontiguousarray(base, dtype=np.uint64)
    return int(_load().oracle_score_base(Q, D, K.ctypes.data, X.ctypes.data,
                                         None if b is None else b.ctypes.data, mpg.ctypes.data))


def oracle_build_costs(Q: int, D: int, model: dict):
    """Cost tables (NEXT-1) from a cost model dict with keys: profile [n_kernels, D] u64,
    offsets [E*Q+1] u64, kernel_ids [nnz] u32, bytes [E, Q] u64, source [E, Q] i32
    (-1 = host), cached [E, Q] u16 or None, sizes [M] u64, h2d_bw / d2h_bw [D, M] or
    [S, D, M] f64 (per host socket), host_socket [E, Q] u8 or None (socket 0), host_shared
    (int bit mask). Returns (K, X) uint64 [E, Q, D]."""
    prof = np.ascontiguousarray(model["profile"], dtype=np.uint64)
    off = np.ascontiguousarray(model["offsets"], dtype=np.uint64)
    ids = np.ascontiguousarray(model["kernel_ids"], dtype=np.uint32)
    nbytes = np.ascontiguousarray(model["bytes"], dtype=np.uint64)
    src = np.ascontiguousarray(model["source"], dtype=np.int32)
    cached = model.get("cached")
    cached = None if cached is None else np.ascontiguousarray(cached, dtype=np.uint16)
    sizes = np.ascontiguousarray(model["sizes"], dtype=np.uint64)
    h2d = np.ascontiguousarray(model["h2d_bw"], dtype=np.float64)
    d2h = np.ascontiguousarray(model["d2h_bw"], dtype=np.float64)
    S = 1 if h2d.ndim == 2 else int(h2d.shape[0])
    hs = model.get("host_socket")
    hs = None if hs is None else np.ascontiguousarray(hs, dtype=np.uint8)
    E = nbytes.shape[0]
    K = np.zeros((E, Q, D), dtype=np.uint64)
    X = np.zeros((E, Q, D), dtype=np.uint64)
    ids_ptr = ids.ctypes.data if ids.size else None
    rc = _load().oracle_build_costs(
        Q, D, E, prof.shape[0], prof.ctypes.data, off.ctypes.data, ids_ptr, nbytes.ctypes.data,
        src.ctypes.data, None if cached is None else cached.ctypes.data, sizes.shape[0],
        sizes.ctypes.data, S, None if hs is None else hs.ctypes.data,
        h2d.ctypes.data, d2h.ctypes.data, int(model.get("host_shared", 0)),
        K.ctypes.data, X.ctypes.data,
    )
    if rc != 0:
        raise OracleError(rc)
    return K, X
