"""A/B kernel timing of several builds of libmcl.so on the same GPU (not the bench line).

    python scripts/ab_kernel.py --libs ab/libmcl_head.so paper_conf_cluster_ajipbf15_b200/libmcl.so \
        --workloads cfg5 cfg4 cfg2 --rounds 3

A workload may carry generator / path options: `cfg2:E=600:path=7`.
A library may carry environment settings for its subprocess: `lib.so@MCL_BATCH_PIECES=1`.
Each (round, library) pair runs in its own subprocess (the binding loads one library per
process); libraries alternate within a round so clock drift hits them alike. Prints the
median kernel time (CUDA events around the search launch) per library and workload, and
checks that every build returns the same result.
"""
import argparse
import json
import os
import statistics
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CHILD = r"""
import json, sys, statistics
sys.path.insert(0, {root!r})
import torch
from paper_conf_cluster_ajipbf15_b200 import mcl, Mapper, workloads
mcl.load_library({lib!r})
out = {{}}
with Mapper(0) as m:
    m.set_timing(1)
    for spec in {wls!r}:
        name, *opts = spec.split(":")
        kw = {{k: int(v) for k, v in (o.split("=") for o in opts)}}
        m.force_path(kw.pop("path", 0))
        K, X = workloads.make(name, **kw)
        Kd, Xd = torch.from_numpy(K).cuda(), torch.from_numpy(X).cuda()
        reps = 5 if name == "cfg5" else 20
        for _ in range(3):
            idx, mp, ms = m.map_queues(Kd, Xd)
        ts = []
        for _ in range(reps):
            idx, mp, ms = m.map_queues(Kd, Xd)
            ts.append(m.last_kernel_time_ms()[0])
        out[spec] = {{"ms": statistics.median(ts), "min": min(ts),
                      "res": [int(idx[:64].sum()), int(ms[:64].sum())]}}
print(json.dumps(out))
"""


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--libs", nargs="+", required=True)
    ap.add_argument("--workloads", nargs="+", default=["cfg5", "cfg4", "cfg2"])
    ap.add_argument("--rounds", type=int, default=3)
    args = ap.parse_args()
    res = {lib: {w: [] for w in args.workloads} for lib in args.libs}
    results = {}
    for r in range(args.rounds):
        for lib in (args.libs if r % 2 == 0 else args.libs[::-1]):
            path, _, envs = lib.partition("@")
            env = dict(os.environ)
            for kv in filter(None, envs.split(",")):
                k, _, v = kv.partition("=")
                env[k] = v
            code = CHILD.format(root=ROOT, lib=os.path.abspath(path), wls=args.workloads)
            p = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, env=env)
            if p.returncode:
                print(lib, "failed:", p.stderr[-2000:])
                continue
            d = json.loads(p.stdout.strip().splitlines()[-1])
            for w, v in d.items():
                res[lib][w].append(v["ms"])
                results.setdefault(w, set()).add(tuple(v["res"]))
    for w in args.workloads:
        line = {"workload": w, "same_result": len(results.get(w, ())) == 1}
        for lib in args.libs:
            line[os.path.basename(lib)] = {"median_ms": statistics.median(res[lib][w]) if res[lib][w] else None,
                                           "all": [round(x, 4) for x in res[lib][w]]}
        print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
