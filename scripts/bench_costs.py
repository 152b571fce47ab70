"""Cost-table construction (NEXT-1) kernel time and algorithmic HBM fraction, measured as
bench.py measures the search: L2 flushed (256 MiB write + read-back) before each launch,
spin-kernel hold so the events bracket device execution. Prints one JSON line per shape.

    python scripts/bench_costs.py [--lib path/to/libmcl.so] [--reps 10]
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_cluster_ajipbf15_b200 import Mapper, mcl, workloads  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--lib", default=None)
ap.add_argument("--reps", type=int, default=10)
args = ap.parse_args()
if args.lib:
    mcl.load_library(os.path.abspath(args.lib))


def hbm_peak():
    try:
        return float(json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"])
    except Exception:
        return 6650.0


peak = hbm_peak()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
with Mapper(0, stream=torch.cuda.current_stream().cuda_stream) as m:
    m.set_timing(True, hold_us=200)
    for E, Q, D, S in ((100_000, 8, 4, 1), (1_000_000, 2, 3, 1), (100_000, 8, 4, 2)):
        model = workloads.cost_model(42, E, Q, D, sockets=S)
        dm = {k: (torch.from_numpy(np.ascontiguousarray(v)).cuda() if isinstance(v, np.ndarray) else v)
              for k, v in model.items()}
        EQ = E * Q
        nnz = int(model["kernel_ids"].shape[0])
        # ids + offsets + bytes + source + cached in, K and X out
        alg = 4 * nnz + 8 * (EQ + 1) + 8 * EQ + 4 * EQ + 2 * EQ + 2 * 8 * D * EQ + (EQ if S > 1 else 0)
        for _ in range(3):
            m.build_costs(dm, D, device_out=True)
        ks = []
        for i in range(args.reps):
            flush.fill_(i)
            flush.view(torch.int64).sum()
            m.build_costs(dm, D, device_out=True)
            ks.append(m.last_kernel_time_ms()[0])
        k = statistics.median(ks)
        print(json.dumps({"measure": "build_costs", "lib": args.lib or "in-tree", "E": E, "Q": Q, "D": D, "sockets": S,
                          "invocations": nnz, "kernel_ms": k, "algorithmic_bytes": alg,
                          "GB_per_s": alg / (k / 1e3) / 1e9, "frac_of_hbm": alg / (k / 1e3) / 1e9 / peak,
                          "hbm_peak_gbs": peak}), flush=True)
