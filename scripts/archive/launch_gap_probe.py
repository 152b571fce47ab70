"""Event-timed duration of a tiny shard of the blocked kernel (cfg5 / cfg4, rank 0 of 4096:
almost no scoring) under different preceding work on the stream, to separate the kernel's
own fixed cost from what the previous kernel leaves behind (measurement only):
  hold+flush : L2 flush, then the 200 us spin kernel, then the search (bench.py's pass)
  hold       : spin kernel only
  b2b        : the previous search call only (back to back)
  b2b_dev    : the previous search call only, events bracketing 10 launches (per launch)
"""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch  # noqa: E402

from paper_conf_cluster_ajipbf15_b200 import Mapper, workloads  # noqa: E402

flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
st = torch.cuda.Stream()
torch.cuda.set_stream(st)
for name in ("cfg5", "cfg4"):
    K, X = workloads.make(name)
    Kd, Xd = torch.from_numpy(K).cuda(), torch.from_numpy(X).cuda()
    for G in (4096, 8):
        res = {"workload": name, "G": G}
        with Mapper(0, stream=st.cuda_stream, rank=0, world=G) as m:
            for mode in ("hold+flush", "hold", "b2b"):
                ts = []
                for i in range(12):
                    if mode == "hold+flush":
                        flush.fill_(i)
                        flush.view(torch.int64).sum()
                    m.set_timing(True, hold_us=200 if mode != "b2b" else 0)
                    m.map_queues(Kd, Xd)
                    ts.append(m.last_kernel_time_ms()[0] * 1e3)
                res[mode] = statistics.median(ts[2:])
            m.set_timing(False)
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            for _ in range(3):
                m.map_queues(Kd, Xd)
            a.record(st)
            for _ in range(10):
                m.map_queues(Kd, Xd)
            b.record(st)
            b.synchronize()
            res["b2b_call_us"] = a.elapsed_time(b) * 1e3 / 10
        print(json.dumps(res), flush=True)
