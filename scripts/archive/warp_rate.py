import json, os, statistics, sys
sys.path.insert(0, "/root/repo")
import torch
from paper_conf_cluster_ajipbf15_b200 import mcl, workloads
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
st = torch.cuda.Stream(); torch.cuda.set_stream(st)
E = int(os.environ["E"])
K, X = workloads.cfg2(E=E, seed=2)
Kd, Xd = torch.from_numpy(K).cuda(), torch.from_numpy(X).cuda()
with mcl.Mapper(0, stream=st.cuda_stream) as m:
    m.force_path(7)
    m.set_timing(True, hold_us=200); ts = []
    for i in range(9):
        flush.fill_(i); m.map_queues(Kd, Xd); ts.append(m.last_kernel_time_ms()[0])
    info = m.launch_info()
k = statistics.median(ts[2:])
print(json.dumps({"E": E, "cap": os.environ.get("MCL_BATCH_CTAS_PER_SM"), "split": os.environ.get("MCL_BATCH_SPLIT_PCT"), "kernel_us": k * 1e3, "ctas": info["ctas"], "us_per_epoch_per_warp": k * 1e3 * info["ctas"] * 4 / E}))
