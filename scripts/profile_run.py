"""Run one workload through the mapper a few times (for ncu / compute-sanitizer runs)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_cluster_ajipbf15_b200 import Mapper, workloads  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "cfg5"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
kw = {}
if len(sys.argv) > 3:  # optional epochs override for batched configs (sanitizer runs)
    kw["E"] = int(sys.argv[3])
constrained = name.endswith("c")  # e.g. cfg5c: cfg5 with 3 pinned + 3 masked queues (NEXT-3)
K, X = workloads.make(name.rstrip("c"), **kw)
Kd, Xd = torch.from_numpy(K).cuda(), torch.from_numpy(X).cuda()
if constrained:
    base, elig = workloads.constraints(77, *K.shape)
    if K.shape[1] == 12:  # cfg5c: 3 pinned + 3 masked queues
        elig[:] = 0
        elig[:, [1, 5, 10]] = [1 << 3, 1 << 0, 1 << 6]
        elig[:, [2, 7, 11]] = [0b00110110, 0b11000001, 0b0111]
    # else (e.g. cfg2c): 25 % pinned + 25 % masked queues per epoch (workloads.constraints)
    Bd, Ed = torch.from_numpy(base).cuda(), torch.from_numpy(elig).cuda()
with Mapper(0) as m:
    for _ in range(reps):
        if constrained:
            idx, mp, ms = m.map_queues_constrained(Kd, Xd, Bd, Ed)
        else:
            idx, mp, ms = m.map_queues(Kd, Xd)
    torch.cuda.synchronize()
    print(name, m.launch_info(), int(idx[0]), int(ms[0]))
