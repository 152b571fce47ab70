"""Measure the NEXT-3 variants and the alternative batched kernel on one GPU (not the
driver's bench line): constrained search, mapping scoring, CTA-per-epoch vs flattened
batched kernel. Prints one JSON line per measurement.

    python scripts/bench_variants.py [--reps 10]
"""
import argparse
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_cluster_ajipbf15_b200 import Mapper, workloads  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--reps", type=int, default=10)
args = ap.parse_args()
dev = torch.device("cuda", 0)


def t(x):
    return torch.from_numpy(np.ascontiguousarray(x)).to(dev)


def timed(m, fn, mappings):
    for _ in range(3):
        fn()
    ks = []
    for _ in range(args.reps):
        fn()
        ks.append(m.last_kernel_time_ms()[0])
    k = statistics.median(ks)
    return {"kernel_ms": k, "mappings_per_s": mappings / (k / 1e3)}


def feasible_count(elig, D):
    """Mappings allowed by the masks (product of the eligible-device counts), per epoch."""
    full = (1 << D) - 1
    m = np.where(elig == 0, full, elig.astype(np.int64) & full)
    cnt = np.vectorize(lambda v: bin(int(v)).count("1"))(m)
    return np.prod(cnt.astype(np.float64), axis=1)


def verdict_cfg5_constraints():
    """cfg5 with 3 pinned + 3 masked queues."""
    base, elig = workloads.constraints(77, 1, 12, 8)
    elig[0] = 0
    elig[0, [1, 5, 10]] = [1 << 3, 1 << 0, 1 << 6]
    elig[0, [2, 7, 11]] = [0b00110110, 0b11000001, 0b0111]
    return base, elig


with Mapper(0) as m:
    m.set_timing(1)
    cases = [(name, workloads.constraints(11, *workloads.make(name)[0].shape), "25% queues pinned, 25% masked, "
              "base loads U[0,2^20)") for name in ("cfg5", "cfg4", "cfg2")]
    cases.insert(1, ("cfg5", verdict_cfg5_constraints(), "3 pinned + 3 masked (queue 11 inner), base U[0,2^20)"))
    for name, (base, elig), what in cases:
        K, X = workloads.make(name)
        E, Q, D = K.shape
        N = E * D**Q
        feas = float(feasible_count(elig, D).sum())
        Kd, Xd, Bd, Ed = t(K), t(X), t(base), t(elig)
        r0 = timed(m, lambda: m.map_queues(Kd, Xd), N)
        r1 = timed(m, lambda: m.map_queues_constrained(Kd, Xd, Bd, Ed), feas)
        path = m.launch_info()["path"]
        m.force_path(1)
        r2 = timed(m, lambda: m.map_queues_constrained(Kd, Xd, Bd, Ed), feas)
        m.force_path(0)
        print(json.dumps({"measure": "constrained_mixed_radix", "workload": name, "constraints": what,
                          "full_space_mappings": N, "feasible_mappings": feas,
                          "plain": r0, "mixed_radix": {**r1, "path": path, "unit": "feasible mappings/s"},
                          "full_space_inf_masked": {**r2, "unit": "feasible mappings/s"},
                          "speedup_vs_full_space": r2["kernel_ms"] / r1["kernel_ms"]}), flush=True)
    # policy baselines vs the optimum (PAPER.md L584-587 ROUND_ROBIN, L1088-1116 AUTO_STATIC)
    K, X = workloads.cfg2()
    E, Q, D = K.shape
    Kd, Xd = t(K), t(X)
    opt = m.map_queues(Kd, Xd)[2].double()
    hints, score = workloads.static_hints(K, X), workloads.static_device_scores(D)
    st_map = m.static_mappings(t(hints), t(score))
    rr_map = t(np.tile((np.arange(Q) % D).astype(np.uint8), (E, 1)))
    for label, mp in (("auto_static_hints", st_map), ("round_robin", rr_map)):
        ms = m.score_mappings(Kd, Xd, mp).double()
        ratio = (ms / opt.clamp(min=1)).cpu().numpy()
        nz = (opt > 0).cpu().numpy()
        print(json.dumps({"measure": "policy_vs_optimum", "workload": "cfg2", "policy": label,
                          "makespan_ratio_mean": float(ratio[nz].mean()),
                          "makespan_ratio_median": float(np.median(ratio[nz])),
                          "makespan_ratio_max": float(ratio[nz].max()),
                          "epochs_optimal": float((ms == opt).double().mean()),
                          "note": "makespan of the policy's mapping / the mapper's optimum, per epoch "
                                  "(epochs with optimum 0 excluded from the ratios)"}), flush=True)
    for path, label in ((1, "cta_per_epoch"), (5, "flattened")):
        m.force_path(path)
        r = timed(m, lambda: m.map_queues(Kd, Xd), K.shape[0] * 4**8)
        print(json.dumps({"measure": "batched_kernel", "workload": "cfg2", "kernel": label, **r}), flush=True)
    m.force_path(0)
    E, Q, D = 1_000_000, 8, 4
    K, X = workloads.cfg2(E=E, seed=5)
    mp = np.tile((np.arange(Q) % D).astype(np.uint8), (E, 1))
    base = np.zeros((E, D), np.uint64)
    Kd, Xd, Md, Bd = t(K), t(X), t(mp), t(base)
    out = torch.empty(E, dtype=torch.uint64, device=dev)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    for _ in range(3):
        m.score_mappings(Kd, Xd, Md, Bd)
    ts = []
    for _ in range(args.reps):
        ev0.record()
        m.score_mappings(Kd, Xd, Md, Bd)
        ev1.record()
        torch.cuda.synchronize()
        ts.append(ev0.elapsed_time(ev1))
    ms = statistics.median(ts)
    nbytes = E * (2 * Q * D * 8 + D * 8 + Q + 8)
    print(json.dumps({"measure": "score_mappings", "epochs": E, "Q": Q, "D": D, "call_ms": ms,
                      "epochs_per_s": E / (ms / 1e3), "GB_per_s": nbytes / (ms / 1e3) / 1e9,
                      "note": "call time incl. host overhead; round-robin mappings"}), flush=True)

# ---- NEXT-4: pruned exact search, time-to-solution vs exhaustive ----
with Mapper(0) as m:
    m.set_timing(1)
    for name in ("cfg5", "cfg4", "cfg2", "cfg3"):
        K, X = workloads.make(name)
        E, Q, D = K.shape
        Kd, Xd = t(K), t(X)
        ex = timed(m, lambda: m.map_queues(Kd, Xd), E * D**Q)
        pr = timed(m, lambda: m.map_queues_pruned(Kd, Xd), E * D**Q)
        a = m.map_queues_pruned(Kd, Xd)
        nodes = m.launch_info()["nodes"]  # read before the exhaustive call replaces it
        b = m.map_queues(Kd, Xd)
        same = bool((a[0] == b[0]).all().item() and (a[2] == b[2]).all().item())
        print(json.dumps({"measure": "pruned_vs_exhaustive", "workload": name,
                          "exhaustive_kernel_ms": ex["kernel_ms"], "pruned_kernel_ms": pr["kernel_ms"],
                          "speedup": ex["kernel_ms"] / pr["kernel_ms"], "nodes": nodes,
                          "identical_result": same}), flush=True)
    for seed, (Q, D) in enumerate(((16, 8), (20, 4), (24, 3))):
        K, X = workloads.random_tables(500 + seed, 1, Q, D, hi=1 << 22)
        Kd, Xd = t(K), t(X)
        pr = timed(m, lambda: m.map_queues_pruned(Kd, Xd), D**Q)
        print(json.dumps({"measure": "pruned_large", "Q": Q, "D": D, "mappings": D**Q,
                          "pruned_kernel_ms": pr["kernel_ms"], "nodes": m.launch_info()["nodes"],
                          "exhaustive_estimate_ms": D**Q / 1.15e13 * 1e3}), flush=True)

# ---- NEXT-1: cost-table construction (HBM-bound) and the fused pipeline ----
with Mapper(0) as m:
    m.set_timing(1)
    for E, Q, D in ((100_000, 8, 4), (1_000_000, 2, 3)):
        model = workloads.cost_model(42, E, Q, D)
        dm = {k: (t(v) if isinstance(v, np.ndarray) else v) for k, v in model.items()}
        EQ = E * Q
        nnz = int(model["kernel_ids"].shape[0])
        alg = 4 * nnz + 8 * (EQ + 1) + 8 * EQ + 4 * EQ + 2 * EQ + 2 * 8 * D * EQ
        for _ in range(3):
            m.build_costs(dm, D, device_out=True)
        ks = []
        for _ in range(args.reps):
            m.build_costs(dm, D, device_out=True)
            ks.append(m.last_kernel_time_ms()[0])
        k = statistics.median(ks)
        print(json.dumps({"measure": "build_costs", "E": E, "Q": Q, "D": D, "invocations": nnz,
                          "kernel_ms": k, "algorithmic_bytes": alg, "GB_per_s": alg / (k / 1e3) / 1e9,
                          "frac_of_hbm": alg / (k / 1e3) / 1e9 / 6541.8}), flush=True)
