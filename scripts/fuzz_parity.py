"""Randomised parity sweep on the GPU (test aid, complements tests/): random shapes, batch
sizes, value ranges and forced kernel paths through mcl_map_queues, every result compared
with the CPU oracle bit for bit. Runs for a time budget and prints one JSON summary line.

    python scripts/fuzz_parity.py [seconds] [seed]
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402  (test infrastructure: the checker)
from paper_conf_cluster_ajipbf15_b200 import Mapper  # noqa: E402

budget = float(sys.argv[1]) if len(sys.argv) > 1 else 240.0
rng = np.random.default_rng(int(sys.argv[2]) if len(sys.argv) > 2 else 12345)
BATCH = [(8, 3), (9, 3), (10, 3), (11, 3), (8, 4), (9, 4), (10, 4), (8, 5), (9, 5)]
cases = fails = 0
paths = {}
t0 = time.time()
with Mapper(0) as m:
    while time.time() - t0 < budget:
        kind = rng.integers(0, 6)
        if kind >= 4:  # constrained (mixed-radix kernels) and pruned calls vs the constrained oracle
            Q, D = int(rng.integers(3, 11)), int(rng.integers(2, 9))
            while D ** Q > 3e5:
                Q -= 1
            E = int(rng.choice([1, 4, 50, 700]))
            hi = int(rng.choice([8, 1 << 12, 1 << 22]))
            K = rng.integers(0, hi, size=(E, Q, D), dtype=np.uint64)
            X = rng.integers(0, hi, size=(E, Q, D), dtype=np.uint64)
            base = rng.integers(0, hi, size=(E, D), dtype=np.uint64)
            elig = np.zeros((E, Q), np.uint16)
            r = rng.random((E, Q))
            elig[r < 0.25] = (1 << rng.integers(0, D, size=(E, Q))).astype(np.uint16)[r < 0.25]
            sub = rng.integers(1, 1 << D, size=(E, Q)).astype(np.uint16)
            elig[(r >= 0.25) & (r < 0.5)] = sub[(r >= 0.25) & (r < 0.5)]
            args = [torch.from_numpy(a).cuda() for a in (K, X, base, elig)]
            fn = m.map_queues_constrained if kind == 4 else m.map_queues_pruned
            gi, gmp, gms = fn(*args)
            path = ("constrained:" if kind == 4 else "pruned:") + m.launch_info()["path"]
            wi, wms, wmp = oracle.oracle_map_constrained(K, X, base, elig)
            ok = bool((gi.cpu().numpy() == wi).all() and (gms.cpu().numpy() == wms).all()
                      and (gmp.cpu().numpy() == wmp).all())
            cases += 1
            paths[path] = paths.get(path, 0) + 1
            if not ok:
                fails += 1
                print(json.dumps({"FAIL": True, "Q": Q, "D": D, "E": E, "hi": hi, "kind": int(kind), "path": path}), flush=True)
            continue
        if kind == 0:  # batch shapes, pooled / warp / CTA kernels
            Q, D = BATCH[rng.integers(0, len(BATCH))]
            E = int(rng.choice([1, 5, 37, 150, 296, 333, 600, 1000]))
            if D ** Q * E > 4e8:
                E = max(1, int(4e8 // D ** Q))
            force = int(rng.choice([0, 0, 7, 1]))
        elif kind == 1:  # small shapes (thread / warp per epoch)
            Q, D = int(rng.integers(1, 5)), int(rng.integers(1, 4))
            E = int(rng.choice([1, 64, 1000, 20000]))
            force = 0
        else:  # general shapes: blocked / generic / flat
            Q, D = int(rng.integers(1, 8)), int(rng.integers(1, 9))
            while D ** Q > 3e5:
                Q -= 1
            E = int(rng.choice([1, 3, 17, 200]))
            force = int(rng.choice([0, 1, 2, 3, 5])) if Q >= 3 and D >= 2 else 0
            if force == 5 and E == 1:
                force = 0
        hi = int(rng.choice([2, 8, 1 << 10, 1 << 20, 1 << 28]))
        K = rng.integers(0, hi, size=(E, Q, D), dtype=np.uint64)
        X = rng.integers(0, hi, size=(E, Q, D), dtype=np.uint64)
        if rng.random() < 0.3:  # equal rows / zero epochs: heavy ties
            K[:: max(1, E // 3)] = K[0, 0, 0]
            X[:: max(1, E // 3)] = 0
        m.force_path(force)
        try:
            gi, gmp, gms = m.map_queues(torch.from_numpy(K).cuda(), torch.from_numpy(X).cuda())
            path = m.launch_info()["path"]
        except Exception as exc:  # a forced path that does not apply to the shape
            m.force_path(0)
            if "forced kernel path" in str(exc):
                continue
            raise
        m.force_path(0)
        wi, wms, wmp = oracle.oracle_map(K, X)
        ok = bool((gi.cpu().numpy() == wi).all() and (gms.cpu().numpy() == wms).all()
                  and (gmp.cpu().numpy() == wmp).all())
        cases += 1
        paths[path] = paths.get(path, 0) + 1
        if not ok:
            fails += 1
            print(json.dumps({"FAIL": True, "Q": Q, "D": D, "E": E, "hi": hi, "force": force, "path": path}), flush=True)
print(json.dumps({"fuzz_parity": True, "cases": cases, "failures": fails, "paths": paths,
                  "seconds": round(time.time() - t0, 1)}))
