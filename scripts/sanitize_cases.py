"""Small runs of the round-2 paths for compute-sanitizer (memcheck / racecheck / synccheck):
the mixed-radix constrained kernels (single epoch spread over CTAs, batched, one warp per
epoch, sharded, u64),
the blocked kernel's packed-key merge of a split epoch, the static policy and scoring
kernels, per-socket cost tables, and zero-copy small calls on pinned host buffers.

    compute-sanitizer --tool memcheck python scripts/sanitize_cases.py
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_cluster_ajipbf15_b200 import Mapper, workloads  # noqa: E402


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


with Mapper(0) as m:
    # mixed radix: one 10 x 6 epoch with pins and masks, a batch of 24, a 64-bit rerun
    K, X = workloads.random_tables(1, 1, 10, 6)
    base, elig = workloads.constraints(1, 1, 10, 6)
    m.map_queues_constrained(dev(K), dev(X), dev(base), dev(elig))
    K, X = workloads.cfg2(E=24, seed=3)
    base, elig = workloads.constraints(2, 24, 8, 4)
    m.map_queues_constrained(dev(K), dev(X), dev(base), dev(elig))
    m.map_queues_constrained(dev(K), dev(X), dev(base + np.uint64(1 << 40)), dev(elig))
    # the warp-per-epoch mixed-radix kernel (forced; a batch of 40 epochs), and its u64 rerun
    K, X = workloads.cfg2(E=40, seed=8)
    base, elig = workloads.constraints(9, 40, 8, 4)
    m.force_path(9)
    m.map_queues_constrained(dev(K), dev(X), dev(base), dev(elig))
    m.map_queues_constrained(dev(K), dev(X), dev(base + np.uint64(1 << 40)), dev(elig))
    m.force_path(0)
    # blocked kernel, one epoch over every CTA (packed-key merge, pair rescan)
    K, X = workloads.cfg4(seed=4, Q=11)
    m.map_queues(dev(K), dev(X))
    # static policy + scoring
    K, X = workloads.cfg2(E=200, seed=5)
    hints, score = workloads.static_hints(K, X), workloads.static_device_scores(4)
    mp = m.static_mappings(dev(hints), dev(score))
    m.score_mappings(dev(K), dev(X), mp)
    # per-socket cost tables
    model = workloads.cost_model(6, 50, 8, 4, sockets=2)
    m.build_costs(model, 4)
    # zero-copy small call on pinned host buffers
    K, X = workloads.cfg1_npb("FT")
    Kp, Xp = torch.from_numpy(K).pin_memory(), torch.from_numpy(X).pin_memory()
    i = torch.empty(1, dtype=torch.uint64).pin_memory()
    ms = torch.empty(1, dtype=torch.uint64).pin_memory()
    mpp = torch.empty((1, 4), dtype=torch.uint8).pin_memory()
    m.map_queues_into(Kp, Xp, i, mpp, ms)
for r in range(3):  # shards of the feasible enumeration
    with Mapper(0, rank=r, world=3) as m:
        K, X = workloads.random_tables(7, 1, 9, 5)
        base, elig = workloads.constraints(7, 1, 9, 5)
        m.map_queues_constrained(dev(K), dev(X), dev(base), dev(elig))
torch.cuda.synchronize()
print("sanitize cases ok")
