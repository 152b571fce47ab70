#!/bin/bash
# cfg2: CTA-per-epoch (path 1) vs flattened (path 5) kernel time
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
python - <<'PY'
import sys, torch
sys.path.insert(0, '.')
from paper_conf_cluster_ajipbf15_b200 import Mapper, workloads
K, X = workloads.cfg2()
Kd, Xd = torch.from_numpy(K).cuda(), torch.from_numpy(X).cuda()
with Mapper(0) as m:
    m.set_timing(1)
    for path in (1, 5, 1, 5):
        m.force_path(path)
        ts = []
        for _ in range(12):
            m.map_queues(Kd, Xd)
            ts.append(m.last_kernel_time_ms()[0])
        ts = sorted(ts[2:])
        print("path", path, m.launch_info()["path"], "kernel ms median %.4f min %.4f" % (ts[len(ts)//2], ts[0]), m.launch_info()["ctas"])
PY
