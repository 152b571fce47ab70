"""Per-CTA phase timing of the blocked kernel from a -DMCL_TRACE build (measurement only):

    python scripts/build_variant.py build/trace/libmcl_trace.so search_blocked.cu -DMCL_TRACE
    python scripts/trace_phases.py build/trace/libmcl_trace.so

For cfg5 / cfg4 at several shard counts G (rank 0's kernel, as on each of G GPUs), prints
the launch ramp (spread of the CTAs' start), the prologue (tables), the walk (min / median /
max over CTAs), the reduction tail, and the SM clock during the walk (clock64 / globaltimer).
"""
import ctypes
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_cluster_ajipbf15_b200 import mcl, workloads  # noqa: E402

lib = mcl.load_library(os.path.abspath(sys.argv[1]))
lib.mcl_trace_read.argtypes = [ctypes.c_void_p, ctypes.c_int]
buf = np.zeros((4096, 8), np.uint64)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for name, Gs in (("cfg5", (1, 8, 64)), ("cfg4", (1, 8, 64))):
    K, X = workloads.make(name)
    Kd, Xd = torch.from_numpy(K).cuda(), torch.from_numpy(X).cuda()
    for G in Gs:
        with mcl.Mapper(0, rank=0, world=G) as m:
            for i in range(3):
                flush.fill_(i)
                torch.cuda.synchronize()
                m.map_queues(Kd, Xd)
            n = m.launch_info()["ctas"]
        lib.mcl_trace_read(buf.ctypes.data, 4096)
        t = buf[:n].astype(np.int64)
        t0, c0, t1, c1, t2, c2, t3, c3 = (t[:, k] for k in range(8))
        base = t0.min()
        walk = (t2 - t1) / 1e3
        mhz = (c2 - c1) / np.maximum(1, (t2 - t1)) * 1e3
        print(json.dumps({
            "workload": name, "G": G, "ctas": int(n),
            "kernel_span_us": float((t3.max() - base) / 1e3),
            "start_spread_us": float((t0.max() - base) / 1e3),
            "prologue_us_median": float(np.median((t1 - t0) / 1e3)),
            "walk_us_min": float(walk.min()), "walk_us_median": float(np.median(walk)), "walk_us_max": float(walk.max()),
            "walk_end_spread_us": float((t2.max() - t2.min()) / 1e3),
            "tail_us_max": float(((t3 - t2) / 1e3).max()),
            "sm_mhz_walk_median": float(np.median(mhz)), "sm_mhz_walk_min": float(mhz.min()),
        }), flush=True)
