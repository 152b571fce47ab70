import sys, statistics, torch
sys.path.insert(0, '.')
from paper_conf_cluster_ajipbf15_b200 import Mapper, workloads
K, X = workloads.cfg2()
with Mapper(0) as m:
    m.set_timing(1)
    for E in (2368, 4736, 7104, 9472, 10000, 11840):
        Kd, Xd = torch.from_numpy(K[:E] if E <= 10000 else __import__('numpy').concatenate([K, K[:E-10000]])).cuda(), torch.from_numpy(X[:E] if E <= 10000 else __import__('numpy').concatenate([X, X[:E-10000]])).cuda()
        ts = []
        for i in range(12):
            m.map_queues(Kd, Xd)
            if i >= 2: ts.append(m.last_kernel_time_ms()[0])
        t = statistics.median(ts)
        print(E, "%.4f ms" % t, "%.2f us/epoch-wave-unit" % (t * 1e3 / (E / 2368)), m.launch_info()["ctas"])
