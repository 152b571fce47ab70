import json, statistics, sys, os
sys.path.insert(0, "/root/repo")
import torch
from paper_conf_cluster_ajipbf15_b200 import Mapper, workloads
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
stream = torch.cuda.Stream(); torch.cuda.set_stream(stream)
def kms(m, Kd, Xd, reps=7):
    m.set_timing(True, hold_us=200); ts=[]
    for i in range(reps):
        flush.fill_(i & 0xFF); m.map_queues(Kd, Xd); ts.append(m.last_kernel_time_ms()[0])
    m.set_timing(False); return statistics.median(ts[1:])
for name in ("cfg5", "cfg4"):
    K, X = workloads.make(name); Kd, Xd = torch.from_numpy(K).cuda(), torch.from_numpy(X).cuda()
    for G in (1, 8, 64, 512, 4096, 32768):
        with Mapper(0, stream=stream.cuda_stream, rank=0, world=G) as m:
            k = kms(m, Kd, Xd); info = m.launch_info()
        print(json.dumps({"w": name, "G": G, "kernel_ms": k, "ctas": info["ctas"], "threads": info["threads"]}), flush=True)
