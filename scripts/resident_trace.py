"""Phases of the resident warp per request (a -DMCL_RESIDENT_TRACE build of resident.cu and
mcl.cpp, scripts/build_variant.py): inputs read over PCIe, scoring, result fence; host wall
time per call beside them. Measurement only.

    python scripts/resident_trace.py build/ab/libmcl_restrace.so
"""
import ctypes
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_cluster_ajipbf15_b200 import mcl, workloads  # noqa: E402

lib = mcl.load_library(os.path.abspath(sys.argv[1]))
lib.mcl_resident_trace.argtypes = [ctypes.c_void_p, ctypes.POINTER(ctypes.c_uint64)]
K, X = workloads.make("cfg1")
Kp, Xp = torch.from_numpy(K).pin_memory(), torch.from_numpy(X).pin_memory()
tr = (ctypes.c_uint64 * 4)()
rows = []
with mcl.Mapper(0) as m:
    m.resident_start(K.shape[1], K.shape[2])
    out = (np.empty(1, np.uint64), np.empty((1, K.shape[1]), np.uint8), np.empty(1, np.uint64))
    for i in range(3000):
        t0 = time.perf_counter()
        m.resident_map(Kp, Xp, out=out)
        dt = (time.perf_counter() - t0) * 1e6
        lib.mcl_resident_trace(m.handle, tr)
        if i >= 100:
            rows.append((dt, (tr[1] - tr[0]) / 1e3, (tr[2] - tr[1]) / 1e3, (tr[3] - tr[2]) / 1e3))
    # the bare C call through ctypes (pointers prepared once): the binding's own overhead
    pk, px = Kp.data_ptr(), Xp.data_ptr()
    pi, pmap, pm = (o.ctypes.data for o in out)
    f = lib.mcl_resident_map
    raw = []
    for r in range(5):
        t0 = time.perf_counter()
        for _ in range(1000):
            f(m.handle, 1, pk, px, pi, pmap, pm)
        raw.append((time.perf_counter() - t0) / 1000 * 1e6)
    m.resident_stop()
    t0 = time.perf_counter()
    for _ in range(1000):
        f(None, 1, pk, px, pi, pmap, pm)  # returns MCL_E_INVAL at once: ctypes call cost
    empty = (time.perf_counter() - t0) / 1000 * 1e6
med = [statistics.median(c) for c in zip(*rows)]
print(json.dumps({"measure": "resident phases (us, median of 2900 calls)", "host_call": med[0],
                  "inputs_read": med[1], "score": med[2], "release_store": med[3],
                  "unaccounted (poll + done + host)": med[0] - sum(med[1:]),
                  "bare_ctypes_call": statistics.median(raw), "ctypes_noop_call": empty}))
