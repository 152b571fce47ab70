"""Host-side overhead of one synchronous mcl_map_queues call (tiny workload)."""
import ctypes
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch  # noqa: E402

from paper_conf_cluster_ajipbf15_b200 import Mapper, mcl, workloads  # noqa: E402

K, X = workloads.cfg1_npb("FT")
Kd, Xd = torch.from_numpy(K).cuda(), torch.from_numpy(X).cuda()
idx = torch.empty(1, dtype=torch.uint64, device="cuda")
ms = torch.empty_like(idx)
mp = torch.empty((1, 4), dtype=torch.uint8, device="cuda")
lib = mcl.load_library()
for timing in (False, True):
    with Mapper(0) as m:
        m.set_timing(timing)
        for _ in range(100):
            m.map_queues_into(Kd, Xd, idx, mp, ms)
        n = 2000
        t0 = time.perf_counter()
        for _ in range(n):
            m.map_queues_into(Kd, Xd, idx, mp, ms)
        t1 = time.perf_counter()
        args = (m.handle, 4, 3, 1, Kd.data_ptr(), Xd.data_ptr(), idx.data_ptr(), mp.data_ptr(), ms.data_ptr())
        f = lib.mcl_map_queues
        t2 = time.perf_counter()
        for _ in range(n):
            f(*args)
        t3 = time.perf_counter()
        print(f"timing={timing}: python binding {1e6 * (t1 - t0) / n:.1f} us/call, raw ctypes {1e6 * (t3 - t2) / n:.1f} us/call")
# bare launch + sync floor
s = torch.cuda.current_stream()
t0 = time.perf_counter()
for _ in range(2000):
    mp.zero_()
    torch.cuda.synchronize()
print(f"torch tiny kernel + synchronize: {1e6 * (time.perf_counter() - t0) / 2000:.1f} us")
