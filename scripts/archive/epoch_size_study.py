"""cfg2-like batches with the same total mappings but bigger epochs: how much of the
batched time is per-epoch overhead?"""
import os, sys, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_cluster_ajipbf15_b200 import Mapper, workloads
with Mapper(0) as m:
    m.set_timing(1)
    for Q, E in ((8, 10000), (9, 2500), (10, 625), (11, 157), (12, 40)):
        K, X = workloads.cfg2(E=E, Q=Q, seed=2)
        Kd, Xd = torch.from_numpy(K).cuda(), torch.from_numpy(X).cuda()
        ts = []
        for i in range(12):
            m.map_queues(Kd, Xd)
            if i >= 2:
                ts.append(m.last_kernel_time_ms()[0])
        t = statistics.median(ts)
        n = E * 4**Q
        print(f"Q={Q} E={E} mappings={n:.3g} kernel {t:.4f} ms -> {n / t / 1e9:.3g} mappings/s, frac {1.5 * n / (t / 1e3) / 18.61e12:.3f}, ctas {m.launch_info()['ctas']} thr {m.launch_info()['threads']}")
