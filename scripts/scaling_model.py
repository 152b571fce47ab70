"""Projected strong scaling of the single-epoch searches (cfg4, cfg5) from one GPU.

This run has one B200, so N-GPU steps cannot be timed. What can be measured here is the
compute side of every rank: shard-mode handles (rank r of G, no communicator) run exactly
the kernel rank r would run on its own GPU over its contiguous index range. For G = 1, 2,
4, 8 this script times every rank's kernel (CUDA events, spin-kernel hold, L2 flushed) and
the per-call host overhead at G = 1 (step time minus kernel time), and projects

    T(G) = max_r kernel_r(G) + host + exchange(G)

with exchange(G) an ASSUMED cost of the cross-GPU combine (default: the fused tail's
measured ~6 us at world 1 plus 2 us per extra rank, --exchange-us overrides). Efficiency is
T(1) / (G * T(G)). A projection, not a measurement: it bounds what load balance and the
per-rank kernel allow; the collective's real latency at N > 1 is the unmeasured term.

    python scripts/scaling_model.py [--reps 5] [--exchange-us 6] [--per-rank-us 2]
"""
import argparse
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_cluster_ajipbf15_b200 import Mapper, workloads  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--reps", type=int, default=5)
ap.add_argument("--exchange-us", type=float, default=6.0)
ap.add_argument("--per-rank-us", type=float, default=2.0)
args = ap.parse_args()

flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
stream = torch.cuda.Stream()
torch.cuda.set_stream(stream)


def kernel_ms(m, Kd, Xd, hold=200):
    m.set_timing(True, hold_us=hold)
    ts = []
    for i in range(args.reps + 1):
        flush.fill_(i & 0xFF)
        m.map_queues(Kd, Xd)
        ts.append(m.last_kernel_time_ms()[0])
    m.set_timing(False)
    return statistics.median(ts[1:])


def step_ms(m, Kd, Xd):
    ts = []
    for i in range(args.reps + 1):
        flush.fill_(i & 0xFF)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        m.map_queues(Kd, Xd)
        b.record(stream)
        b.synchronize()
        ts.append(a.elapsed_time(b))
    return statistics.median(ts[1:])


for name in ("cfg4", "cfg5"):
    K, X = workloads.make(name)
    Kd, Xd = torch.from_numpy(K).cuda(), torch.from_numpy(X).cuda()
    with Mapper(0, stream=stream.cuda_stream) as m:
        k1 = kernel_ms(m, Kd, Xd)
        s1 = step_ms(m, Kd, Xd)
    host = max(0.0, s1 - k1)
    t1 = s1
    for G in (1, 2, 4, 8):
        ks = []
        for r in range(G):
            with Mapper(0, stream=stream.cuda_stream, rank=r, world=G) as m:
                ks.append(kernel_ms(m, Kd, Xd))
        exch = 0.0 if G == 1 else (args.exchange_us + args.per_rank_us * (G - 1)) / 1e3
        tg = max(ks) + host + exch
        print(json.dumps({
            "workload": name, "G": G, "kernel_ms_per_rank_max": max(ks), "kernel_ms_per_rank_min": min(ks),
            "host_ms": host, "exchange_ms_assumed": exch, "projected_step_ms": tg,
            "projected_mappings_per_s": K.shape[2] ** K.shape[1] / (tg / 1e3),
            "projected_efficiency": t1 / (G * tg), "kind": "projection (per-rank kernels measured on one B200)",
        }), flush=True)
