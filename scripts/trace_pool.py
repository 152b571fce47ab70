"""Per-CTA timeline of the SM-pooled batch kernel (cfg2) from a -DMCL_TRACE build
(measurement only):

    python scripts/build_variant.py build/trace/libmcl_btrace.so search_batch.cu -DMCL_TRACE
    python scripts/trace_pool.py build/trace/libmcl_btrace.so

Per CTA (= SM): entry, the first part with its tables ready, the first failed claim (no
work left) and the last warp's exit, relative to the earliest entry; prints quantiles.
"""
import ctypes
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_cluster_ajipbf15_b200 import mcl, workloads  # noqa: E402

lib = mcl.load_library(os.path.abspath(sys.argv[1]))
lib.mcl_ptrace_read.argtypes = [ctypes.c_void_p]
buf = np.zeros((1024, 4), np.uint64)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
E = int(os.environ.get("E", "10000"))
K, X = workloads.cfg2(E=E, seed=2)
Kd, Xd = torch.from_numpy(K).cuda(), torch.from_numpy(X).cuda()
with mcl.Mapper(0) as m:
    m.force_path(7)
    m.set_timing(True, hold_us=200)
    for i in range(4):
        flush.fill_(i)
        flush.view(torch.int64).sum()
        torch.cuda.synchronize()
        m.map_queues(Kd, Xd)
    kms = m.last_kernel_time_ms()[0]
    info = m.launch_info()
lib.mcl_ptrace_read(buf.ctypes.data)
t = buf[: info["ctas"]].astype(np.int64)
t0 = t[:, 0].min()
r = (t - t0) / 1e3
q = lambda v: [round(float(np.quantile(v, x)), 2) for x in (0, 0.5, 0.9, 1)]
print(json.dumps({"E": E, "path": info["path"], "ctas": info["ctas"], "kernel_us_events": round(kms * 1e3, 2),
                  "span_us": round(float(r[:, 3].max()), 2),
                  "entry_us_q0_50_90_100": q(r[:, 0]), "first_ready_us": q(r[:, 1]),
                  "work_exhausted_us": q(r[:, 2]), "last_exit_us": q(r[:, 3]),
                  "drain_us (exit - exhausted)": q(r[:, 3] - r[:, 2])}))
