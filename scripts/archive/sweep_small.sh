#!/bin/bash
# cfg3 small-kernel tuning sweep: tile threads x stages x CTAs per SM. Kernel time (ms,
# median) measured as bench.py does: L2 flushed (write + read-back of 256 MiB) before each
# launch, spin-kernel hold so the events bracket device execution only.
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
for th in ${SWEEP_THREADS:-64 128 256}; do for stg in ${SWEEP_STAGES:-1 2 3 4 6 8}; do for cps in ${SWEEP_CPS:-2 4 8 16}; do
  r=$(MCL_SMALL_THREADS=$th MCL_SMALL_STAGES=$stg MCL_SMALL_CTAS_PER_SM=$cps python - <<'PY'
import sys, statistics, torch
sys.path.insert(0, '.')
from paper_conf_cluster_ajipbf15_b200 import Mapper, workloads
K, X = workloads.cfg3()
Kd, Xd = torch.from_numpy(K).cuda(), torch.from_numpy(X).cuda()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
with Mapper(0, stream=torch.cuda.current_stream().cuda_stream) as m:
    m.set_timing(True, hold_us=200)
    ts = []
    for i in range(15):
        flush.fill_(i)
        flush.view(torch.int64).sum()
        m.map_queues(Kd, Xd)
        if i >= 3: ts.append(m.last_kernel_time_ms()[0])
    print("%.4f %s" % (statistics.median(ts), m.launch_info()["ctas"]))
PY
)
  echo "threads=$th stages=$stg ctas_per_sm=$cps kernel_ms/ctas=$r"
done; done; done
