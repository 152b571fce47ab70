"""A/B kernel timing of two builds of libmcl.so on one GPU (measurement only):

    python scripts/ab_lib.py build/ab/libmcl_old.so build/ab/libmcl_new.so [more.so ...] [rounds]

Each round runs every library in a fresh subprocess (alternating order) and prints the
median (AB_STAT=mean: mean; AB_N launches, default 9) kernel time (CUDA events, 200 us spin hold, L2 flushed) of the single-epoch configs
at G = 1 and of rank 0 at G = 8, and of cfg2.
"""
import json
import os
import subprocess
import sys

CHILD = r'''
import json, os, statistics, sys
sys.path.insert(0, os.environ["REPO"])
import torch
from paper_conf_cluster_ajipbf15_b200 import mcl, workloads
mcl.load_library(os.environ["LIB"])
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
st = torch.cuda.Stream(); torch.cuda.set_stream(st)
out = {}
for name in os.environ.get("AB_WORKLOADS", "cfg5,cfg4,cfg2").split(","):
    cons = name.endswith("c")  # e.g. cfg2c: 25 % pinned + 25 % masked queues (NEXT-3)
    K, X = workloads.make(name.rstrip("c")); Kd, Xd = torch.from_numpy(K).cuda(), torch.from_numpy(X).cuda()
    if cons:
        base, elig = workloads.constraints(77, *K.shape)
        Bd, Ed = torch.from_numpy(base).cuda(), torch.from_numpy(elig).cuda()
    for G in ((1, 8) if name in ("cfg4", "cfg5") else (1,)):
        with mcl.Mapper(0, stream=st.cuda_stream, rank=0, world=G) as m:
            m.set_timing(True, hold_us=200); ts = []
            for i in range(int(os.environ.get("AB_N", "9"))):
                flush.fill_(i); flush.view(torch.int64).sum()
                if cons: m.map_queues_constrained(Kd, Xd, Bd, Ed)
                else: m.map_queues(Kd, Xd)
                ts.append(m.last_kernel_time_ms()[0])
        # AB_STAT=mean: the CUDA-event clock of some boxes ticks in ~1 us steps, so a mean
        # over many launches resolves differences a median of a few cannot
        stat = statistics.mean if os.environ.get("AB_STAT") == "mean" else statistics.median
        out[f"{name}/G{G}"] = round(stat(ts[2:]), 5)
print(json.dumps(out))
'''

args = sys.argv[1:]
rounds = int(args.pop()) if args and args[-1].isdigit() else 3
libs = args
repo = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
for r in range(rounds):
    for lib in (libs if r % 2 == 0 else libs[::-1]):
        env = dict(os.environ, REPO=repo, LIB=os.path.abspath(lib))
        res = subprocess.run([sys.executable, "-c", CHILD], env=env, capture_output=True, text=True)
        line = res.stdout.strip().splitlines()[-1] if res.stdout.strip() else res.stderr[-400:]
        print(json.dumps({"round": r, "lib": os.path.basename(lib), "result": line}), flush=True)
