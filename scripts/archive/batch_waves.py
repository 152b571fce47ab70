"""cfg2-shaped batches of E epochs on the warp-per-epoch kernel: kernel time vs E (whole
waves of 148 SMs x 16 warps and partial ones), to separate per-wave time from the fixed
launch / ramp cost and the last partial wave. Device time via the timing hold."""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_cluster_ajipbf15_b200 import Mapper, workloads  # noqa: E402

K, X = workloads.cfg2(E=12_000)
Kd, Xd = torch.from_numpy(K).cuda(), torch.from_numpy(X).cuda()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
with Mapper(0, stream=torch.cuda.current_stream().cuda_stream) as m:
    m.set_timing(True, hold_us=200)
    m.force_path(7)
    for E in (592, 1184, 2368, 2960, 3552, 4736, 7104, 9472, 10000, 11840):
        ts = []
        for i in range(12):
            flush.fill_(i)
            flush.view(torch.int64).sum()
            m.map_queues(Kd[:E], Xd[:E])
            if i >= 2:
                ts.append(m.last_kernel_time_ms()[0])
        t = statistics.median(ts)
        print(f"E={E:6d} waves={E / 2368:5.2f} kernel_ms={t:.4f} us/epoch={t * 1e3 / E:.4f}", flush=True)
