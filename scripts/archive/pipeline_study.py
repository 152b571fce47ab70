"""Pipelined staging study: wall time of one host-resident mcl_map_queues call per chunk
count, next to the raw pinned copy rates (H2D, D2H, both at once) on this box."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch  # noqa: E402

from paper_conf_cluster_ajipbf15_b200 import Mapper, workloads  # noqa: E402


def wall(fn, reps=30):
    """Median over `reps` of the mean time of 5 back-to-back calls (ms)."""
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        t0 = time.perf_counter()
        for _ in range(5):
            fn()
        torch.cuda.synchronize()
        ts.append((time.perf_counter() - t0) / 5)
    ts.sort()
    return ts[len(ts) // 2] * 1e3


nb = 96 * 2**20
hs = torch.empty(nb, dtype=torch.uint8).pin_memory()
hd = torch.empty(nb, dtype=torch.uint8).pin_memory()
d1 = torch.empty(nb, dtype=torch.uint8, device="cuda")
d2 = torch.empty(nb, dtype=torch.uint8, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()


def both():
    with torch.cuda.stream(s1):
        d1.copy_(hs, non_blocking=True)
    with torch.cuda.stream(s2):
        hd.copy_(d2, non_blocking=True)
    s1.synchronize()
    s2.synchronize()


h2d = wall(lambda: d1.copy_(hs, non_blocking=True))
d2h = wall(lambda: hd.copy_(d2, non_blocking=True))
bi = wall(both)
print(json.dumps({"copy_96MiB_ms": {"h2d": h2d, "d2h": d2h, "both_directions": bi},
                  "GB_per_s": {"h2d": nb / h2d / 1e6, "d2h": nb / d2h / 1e6, "both_each": nb / bi / 1e6}}), flush=True)

for name in ("cfg2", "cfg3"):
    K, X = workloads.make(name)
    E, Q, D = K.shape
    Kh, Xh = torch.from_numpy(K).pin_memory(), torch.from_numpy(X).pin_memory()
    ih = torch.empty(E, dtype=torch.uint64).pin_memory()
    mh = torch.empty(E, dtype=torch.uint64).pin_memory()
    ph = torch.empty((E, Q), dtype=torch.uint8).pin_memory()
    with Mapper(0) as m:
        row = {"workload": name}
        for nc in (1, 2, 3, 4, 6, 8, 16, 0, 1, 2, 4):
            m.set_pipeline_chunks(nc)
            row[f"chunks={nc or 'auto'}" + ("" if f"chunks={nc or 'auto'}" not in row else "_again")] = round(wall(lambda: m.map_queues_into(Kh, Xh, ih, ph, mh)), 4)
        row["auto_chunks"] = m.launch_info()["chunks"]
        print(json.dumps(row), flush=True)
