"""Run the warp-per-epoch kernel on the first E epochs of a cfg2-shaped batch (for ncu)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_cluster_ajipbf15_b200 import Mapper, workloads  # noqa: E402

E = int(sys.argv[1])
K, X = workloads.cfg2(E=E)
Kd, Xd = torch.from_numpy(K).cuda(), torch.from_numpy(X).cuda()
with Mapper(0) as m:
    m.force_path(7)
    for _ in range(3):
        m.map_queues(Kd, Xd)
    torch.cuda.synchronize()
