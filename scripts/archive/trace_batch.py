"""Per-warp timeline of the warp-per-epoch batch kernel (cfg2) from a -DMCL_TRACE build
(measurement only):

    python scripts/build_variant.py build/trace/libmcl_btrace.so search_batch.cu -DMCL_TRACE
    python scripts/trace_batch.py build/trace/libmcl_btrace.so

Prints the kernel span, per-unit phase durations (setup / walk / finish, medians), the
spread of the warps' finish times, and how busy the SMs are over time (warps still working
in each 5 us window).
"""
import ctypes
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_cluster_ajipbf15_b200 import mcl, workloads  # noqa: E402

lib = mcl.load_library(os.path.abspath(sys.argv[1]))
lib.mcl_btrace_read.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int]
NW = 4096 * 4
buf = np.zeros((NW, 8, 4), np.uint64)
sm = np.zeros(NW, np.uint32)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
E = int(os.environ.get("E", "10000"))
K, X = workloads.cfg2(E=E, seed=2)
Kd, Xd = torch.from_numpy(K).cuda(), torch.from_numpy(X).cuda()
with mcl.Mapper(0) as m:
    m.force_path(7)
    for i in range(3):
        flush.fill_(i)
        torch.cuda.synchronize()
        m.map_queues(Kd, Xd)
    ctas = m.launch_info()["ctas"]
lib.mcl_btrace_read(buf.ctypes.data, sm.ctypes.data, NW)
nw = ctas * 4
t = buf[:nw].astype(np.int64)
valid = t[:, :, 0] > 0
t0 = t[valid][:, 0].min()
starts, setup, walk, fin, ends = [], [], [], [], []
for w in range(nw):
    for u in range(8):
        if not valid[w, u]:
            continue
        s0, s1, s2, s3 = t[w, u]
        if s2 == 0:  # split epoch: walk recorded, finish in slot 3
            s2 = s1
        setup.append(s1 - s0)
        walk.append(s2 - s1)
        fin.append(s3 - s2)
    us = [u for u in range(8) if valid[w, u]]
    if us:
        ends.append(t[w, us[-1], 3] - t0)
        starts.append(t[w, 0, 0] - t0)
ends = np.array(ends) / 1e3
span = ends.max()
hist = [int((ends > x).sum()) for x in np.arange(0, span + 5, 5)]
by_unit = {}
for u in range(5):
    w = [(t[x, u, 2] - t[x, u, 1]) / 1e3 for x in range(nw) if valid[x, u] and t[x, u, 2] > 0]
    if w:
        by_unit[u] = [float(np.percentile(w, 10)), float(np.median(w)), float(np.percentile(w, 90))]
print(json.dumps({
    "walk_us_by_unit_p10_p50_p90": by_unit,
    "E": E, "env": {k: v for k, v in os.environ.items() if k.startswith("MCL_")}, "warps": nw, "kernel_span_us": float(span), "first_start_spread_us": float(np.max(starts) / 1e3),
    "setup_us_median": float(np.median(setup) / 1e3), "walk_us_median": float(np.median(walk) / 1e3),
    "walk_us_p10_p90": [float(np.percentile(walk, 10) / 1e3), float(np.percentile(walk, 90) / 1e3)],
    "finish_us_median": float(np.median(fin) / 1e3),
    "warp_end_us_p0_p50_p100": [float(ends.min()), float(np.median(ends)), float(ends.max())],
    "warps_busy_per_5us": hist,
}), flush=True)
