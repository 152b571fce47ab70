"""Host-buffer (e2e) call time of the batched configs, pinned buffers, as bench.py's e2e leg
times it (wall clock over 20 calls after warm-up); MCL_ZERO_COPY_MAX decides whether the
kernels use the pinned buffers in place (zero-copy) or the call stages them (pipelined
copies). Prints one JSON line per config; checks the results against a device-resident call.

    MCL_ZERO_COPY_MAX=1073741824 python scripts/e2e_study.py
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_cluster_ajipbf15_b200 import Mapper, workloads  # noqa: E402

for name in ("cfg2", "cfg3", "cfg1"):
    K, X = workloads.make(name)
    E, Q, D = K.shape
    Kh, Xh = torch.from_numpy(K).pin_memory(), torch.from_numpy(X).pin_memory()
    ih = torch.empty(E, dtype=torch.uint64).pin_memory()
    mh = torch.empty(E, dtype=torch.uint64).pin_memory()
    ph = torch.empty((E, Q), dtype=torch.uint8).pin_memory()
    with Mapper(0) as m:
        i_d, p_d, m_d = m.map_queues(torch.from_numpy(K).cuda(), torch.from_numpy(X).cuda())
        for _ in range(3):
            m.map_queues_into(Kh, Xh, ih, ph, mh)
        same = bool((ih == i_d.cpu()).all() and (mh == m_d.cpu()).all() and (ph == p_d.cpu()).all())
        reps = 20
        t0 = time.perf_counter()
        for _ in range(reps):
            m.map_queues_into(Kh, Xh, ih, ph, mh)
        dt = (time.perf_counter() - t0) / reps
        info = m.launch_info()
    print(json.dumps({"workload": name, "zero_copy_max": os.environ.get("MCL_ZERO_COPY_MAX", "default"),
                      "e2e_ms": dt * 1e3, "mappings_per_s": E * D**Q / dt, "chunks": info["chunks"],
                      "path": info["path"], "identical": same}), flush=True)
