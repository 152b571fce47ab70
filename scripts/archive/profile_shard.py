"""One shard-mode launch of a single-epoch config (rank r of G), for ncu captures."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_cluster_ajipbf15_b200 import Mapper, workloads  # noqa: E402

name, G, r = sys.argv[1], int(sys.argv[2]), int(sys.argv[3])
K, X = workloads.make(name)
Kd, Xd = torch.from_numpy(K).cuda(), torch.from_numpy(X).cuda()
with Mapper(0, rank=r, world=G) as m:
    for _ in range(3):
        m.map_queues(Kd, Xd)
    torch.cuda.synchronize()
