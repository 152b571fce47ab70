"""Per-decision latency of cfg1-sized searches (4 queues x 3 devices, one epoch) through the
three public ways of calling the mapper (measurement only; prints one JSON line each):
  resident     : mcl_resident_map, the warp resident on the GPU (host buffers)
  launch_host  : mcl_map_queues with pinned host buffers (zero-copy launch per call)
  launch_dev   : mcl_map_queues with device-resident buffers (launch + sync per call)
Wall-clock per call from Python (ctypes), median of rounds of 500 calls, results checked.

    python scripts/resident_latency.py [calls] [--lib path/to/libmcl.so]
"""
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_cluster_ajipbf15_b200 import Mapper, mcl, workloads  # noqa: E402

argv = sys.argv[1:]
if "--lib" in argv:
    i = argv.index("--lib")
    mcl.load_library(os.path.abspath(argv[i + 1]))
    del argv[i:i + 2]
shape = None
if "--shape" in argv:  # e.g. --shape 8x3: the paper's FT-sized decision (8 queues, 3 devices)
    i = argv.index("--shape")
    shape = tuple(int(v) for v in argv[i + 1].split("x"))
    del argv[i:i + 2]
calls = int(argv[0]) if argv else 500
K, X = workloads.make("cfg1") if shape is None else workloads.cfg1_random(11, Q=shape[0], D=shape[1])
label = "cfg1 decision latency" if shape is None else f"{shape[0]}x{shape[1]} decision latency"
Kp, Xp = torch.from_numpy(K).pin_memory(), torch.from_numpy(X).pin_memory()
Kd, Xd = Kp.cuda(), Xp.cuda()
out = []
with Mapper(0) as m:
    ref = m.map_queues(Kd, Xd)
    ref = (ref[0].cpu().numpy(), ref[1].cpu().numpy(), ref[2].cpu().numpy())
    idx = torch.empty(1, dtype=torch.uint64).pin_memory()
    mp = torch.empty((1, K.shape[1]), dtype=torch.uint8).pin_memory()
    ms = torch.empty(1, dtype=torch.uint64).pin_memory()
    idx_d, mp_d, ms_d = idx.cuda(), mp.cuda(), ms.cuda()

    def per_call(fn):
        rounds = []
        for _ in range(5):
            t0 = time.perf_counter()
            for _ in range(calls):
                fn()
            rounds.append((time.perf_counter() - t0) / calls * 1e6)
        return statistics.median(rounds), min(rounds)

    r_out = (np.empty(1, np.uint64), np.empty((1, K.shape[1]), np.uint8), np.empty(1, np.uint64))
    Kn, Xn = Kp.numpy(), Xp.numpy()  # numpy views of the pinned buffers
    m.resident_start(K.shape[1], K.shape[2])
    try:
        m.resident_map(Kn, Xn, out=r_out)
        assert r_out[0][0] == ref[0][0] and r_out[2][0] == ref[2][0] and (r_out[1] == ref[1]).all()
        med, best = per_call(lambda: m.resident_map(Kn, Xn, out=r_out))
        out.append({"measure": label, "path": "resident", "lib": os.path.basename(mcl.LIB_PATH if not "--lib" in sys.argv else sys.argv[sys.argv.index("--lib") + 1]), "us_per_call_median": med,
                    "us_per_call_best_round": best})
    finally:
        m.resident_stop()
    med, best = per_call(lambda: m.map_queues_into(Kp, Xp, idx, mp, ms))
    assert idx[0] == ref[0][0] and ms[0] == ref[2][0]
    out.append({"measure": label, "path": "launch_host_pinned", "us_per_call_median": med,
                "us_per_call_best_round": best})
    med, best = per_call(lambda: m.map_queues_into(Kd, Xd, idx_d, mp_d, ms_d))
    out.append({"measure": label, "path": "launch_device_resident", "us_per_call_median": med,
                "us_per_call_best_round": best})
for o in out:
    print(json.dumps(o), flush=True)
