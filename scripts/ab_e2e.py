"""A/B of the host-buffer (e2e) call of the batched configs between builds of libmcl.so
(measurement only): each round runs every library in a fresh subprocess and times
map_queues_into on pinned host buffers (wall clock, median of 30 calls after warm-up), with
the buffers pinned separately and as views into one pinned arena (as bench.py's e2e leg).

    python scripts/ab_e2e.py build/ab/libA.so build/ab/libB.so [rounds]
"""
import json
import os
import subprocess
import sys

CHILD = r'''
import json, os, statistics, sys, time
sys.path.insert(0, os.environ["REPO"])
import torch
from paper_conf_cluster_ajipbf15_b200 import mcl, workloads
mcl.load_library(os.environ["LIB"])
out = {}
for name in os.environ.get("AB_WORKLOADS", "cfg2").split(","):
    K, X = workloads.make(name)
    E, Q, D = K.shape
    sizes = [K.nbytes, X.nbytes, E * 8, E * 8, E * Q]
    offs = [0]
    for n in sizes:
        offs.append(offs[-1] + (n + 255) // 256 * 256)
    arena = torch.empty(offs[-1], dtype=torch.uint8).pin_memory()
    views = [arena[offs[i]:offs[i] + sizes[i]] for i in range(5)]
    bufs = {"separate": [torch.from_numpy(K).pin_memory(), torch.from_numpy(X).pin_memory(),
                         torch.empty(E, dtype=torch.uint64).pin_memory(), torch.empty(E, dtype=torch.uint64).pin_memory(),
                         torch.empty((E, Q), dtype=torch.uint8).pin_memory()],
            "arena": [views[0].view(torch.uint64).view(K.shape), views[1].view(torch.uint64).view(X.shape),
                      views[2].view(torch.uint64), views[3].view(torch.uint64), views[4].view(E, Q)]}
    bufs["arena"][0].copy_(torch.from_numpy(K)); bufs["arena"][1].copy_(torch.from_numpy(X))
    with mcl.Mapper(0) as m:
        for kind, (Kh, Xh, ih, mh, ph) in bufs.items():
            for _ in range(3):
                m.map_queues_into(Kh, Xh, ih, ph, mh)
            ts = []
            for _ in range(30):
                t0 = time.perf_counter(); m.map_queues_into(Kh, Xh, ih, ph, mh); ts.append(time.perf_counter() - t0)
            out[f"{name}/{kind}"] = round(statistics.median(ts) * 1e3, 4)
            out[f"{name}/{kind}/path"] = m.launch_info()["path"]
print(json.dumps(out))
'''

args = sys.argv[1:]
rounds = int(args.pop()) if args and args[-1].isdigit() else 3
repo = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
for r in range(rounds):
    for lib in (args if r % 2 == 0 else args[::-1]):
        env = dict(os.environ, REPO=repo, LIB=os.path.abspath(lib))
        res = subprocess.run([sys.executable, "-c", CHILD], env=env, capture_output=True, text=True)
        line = res.stdout.strip().splitlines()[-1] if res.stdout.strip() else res.stderr[-400:]
        print(json.dumps({"round": r, "lib": os.path.basename(lib), "result": line}), flush=True)
