#!/bin/bash
# cfg3 small-kernel tuning sweep: tile threads x stages x CTAs per SM (kernel time, ms)
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
for th in 128 256; do for stg in 2 4 6 8 12; do for cps in 1 2 4 32; do
  r=$(MCL_SMALL_THREADS=$th MCL_SMALL_STAGES=$stg MCL_SMALL_CTAS_PER_SM=$cps python - <<'PY'
import sys, statistics, torch
sys.path.insert(0, '.')
from paper_conf_cluster_ajipbf15_b200 import Mapper, workloads
K, X = workloads.cfg3()
Kd, Xd = torch.from_numpy(K).cuda(), torch.from_numpy(X).cuda()
with Mapper(0) as m:
    m.set_timing(1)
    ts = []
    for i in range(15):
        m.map_queues(Kd, Xd)
        if i >= 3: ts.append(m.last_kernel_time_ms()[0])
    print("%.4f %s" % (statistics.median(ts), m.launch_info()["ctas"]))
PY
)
  echo "threads=$th stages=$stg ctas_per_sm=$cps kernel_ms/ctas=$r"
done; done; done
