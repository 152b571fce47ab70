"""Write tests/golden/full_configs.json: the oracle's answer on the full-size single-epoch
configs (cfg4: 16 queues x 4 devices, seeds 4-6; cfg5: 12 queues x 8 devices, seed 7).

Calls ONLY oracle/ (plus the seeded generators); no value here comes from the CUDA path.
Run:  python scripts/make_golden.py [cfg4] [cfg5]
"""
from __future__ import annotations

import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
from paper_conf_cluster_ajipbf15_b200 import workloads  # noqa: E402

OUT = os.path.join(ROOT, "tests", "golden", "full_configs.json")


def main(which):
    data = json.load(open(OUT)) if os.path.exists(OUT) else {"_about": (
        "Oracle (oracle/oracle.c brute force) results on the full-size BASELINE configs, written by "
        "scripts/make_golden.py which calls only oracle/ and the seeded generators in "
        "paper_conf_cluster_ajipbf15_b200/workloads.py."), "cases": {}}
    jobs = []
    if "cfg4" in which:
        jobs += [("cfg4", dict(seed=s)) for s in (4, 5, 6)]
    if "cfg5" in which:
        jobs += [("cfg5", dict(seed=7))]
    for name, kw in jobs:
        K, X = workloads.make(name, **kw)
        t0 = time.time()
        idx, ms, mp = oracle.oracle_map(K, X)
        dt = time.time() - t0
        key = f"{name}_seed{kw['seed']}"
        data["cases"][key] = {
            "config": name, "seed": kw["seed"], "Q": int(K.shape[1]), "D": int(K.shape[2]),
            "index": int(idx[0]), "makespan": int(ms[0]), "mapping": [int(v) for v in mp[0]],
            "oracle_seconds": round(dt, 2), "oracle_threads": oracle.default_threads(),
        }
        print(key, data["cases"][key], flush=True)
        json.dump(data, open(OUT, "w"), indent=1)


if __name__ == "__main__":
    main(sys.argv[1:] or ["cfg4", "cfg5"])
