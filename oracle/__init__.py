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
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile oracle.c into oracle/liboracle.so with gcc (plain C11 + pthreads)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(
            ["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-pthread", "-o", _LIB, _SRC]
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
