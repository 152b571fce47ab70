#!/usr/bin/env python
"""bench.py -- queue->device mappings scored per second on B200 (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload cfg5] [--impl mcl|reference]
    python -m torch.distributed.run --nproc-per-node N --master-addr 127.0.0.1 bench.py --gpus N

A step is one mcl_map_queues call: the whole hot path (cost composition, mixed-radix
enumeration, per-device loads, makespan, argmin with lowest-index ties, the cross-GPU
all-reduce when N > 1, and the output decode) on one synthetic workload already resident in
HBM. Default workload: cfg5 = 12 queues x 8 devices (8^12 = 6.9e10 mappings, one epoch),
the largest single-GPU configuration and the one BASELINE.json's scaling target names;
at N GPUs its index space is sharded by contiguous ranges (strong scaling) and the ranks'
packed (makespan, index) keys are combined INSIDE the search kernel over NVLink peer memory
(the fused exchange, include/mcl.h mcl_peer_import; `--collective nccl` uses
ncclAllReduce(MIN) + a decode kernel instead).

Rank 0 prints one JSON line. `value` is whole-job mappings/s from CUDA events over exactly
K timed steps (L2 flushed between steps, outside the events), max over ranks; `e2e` is the
same metric through the C ABI with pinned host buffers (H2D + D2H inside the timed region;
batched workloads stage in pipelined chunks, `e2e.pipelined_chunks`);
`roofline` is the dominant kernel's algorithmic ALU-instruction rate against the B200
ALU-pipe peak; `cpu_baseline` is the CPU oracle timed on a bounded sample of the workload.
`--impl reference` times the oracle instead (this tier's reference arm).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "queue->device mappings scored/sec"
UNIT = "mappings/s"
ALU_LANES_PER_CLK_SM = 64       # B200 ALU pipe: 16 lanes x 4 SMSPs per SM per clock (measured: probe)
ALU_INSTR_PER_MAPPING = 1.5     # floor: 1 VIMNMX forms the makespan + 1/2 VIMNMX3 folds it
L2_FLUSH_BYTES = 256 << 20      # > 126 MB L2
HOLD_US = 200                   # spin ahead of each kernel-duration launch (> host launch latency)
KERNEL_TIMING = ("CUDA events on the mapper's stream around the search launch, in a pass of `steps` "
                 "launches right after the timed steps (L2 flushed before each, as there), each preceded "
                 "by a 200 us spin kernel so the events measure device execution; the timed steps record "
                 "no library events (one timing-event record costs ~2.7 us of host time, "
                 "scripts/host_api_costs.cu, which the step would be charged)")
KERNEL_NAMES = {"blocked_u32": "search_blocked_kernel<u32, D>", "blocked_u32_lean": "search_blocked_kernel<u32, 5, lean>", "blocked_u64": "search_blocked_kernel<u64, D>",
                "generic": "search_generic_kernel", "flat_u32": "search_flat_kernel<u32, D>",
                "small_batched": "search_small_kernel<Q, D>", "batch_u32": "search_batch_kernel<Q, D>"}


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=20)
    p.add_argument("--warmup", type=int, default=5)
    p.add_argument("--workload", default="cfg5", choices=["cfg1", "cfg2", "cfg3", "cfg4", "cfg5"])
    p.add_argument("--impl", default="mcl", choices=["mcl", "reference"])
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--pipeline-chunks", type=int, default=0,
                   help="e2e staging of the host-resident batch: 0 auto, 1 off, n chunks")
    p.add_argument("--cpu-seconds", type=float, default=12.0, help="CPU-oracle sample budget")
    p.add_argument("--collective", default="auto", choices=["auto", "fused", "nccl"],
                   help="cross-GPU combine of a sharded single-epoch search: fused = in-kernel "
                        "exchange over peer memory (NEXT-2), nccl = ncclAllReduce + decode kernel; "
                        "auto = fused when N > 1. An explicit choice also runs it with one rank.")
    return p.parse_args()


def workload(name):
    from paper_conf_cluster_ajipbf15_b200 import workloads

    K, X = workloads.make(name)
    E, Q, D = K.shape
    return K, X, dict(E=E, Q=Q, D=D, N=D**Q, desc=workloads.CONFIGS[name]["desc"])


def is_batched(w):
    return w["E"] > 1


def gpu_local_cpus(device_index):
    """CPUs of the NUMA node the GPU hangs off (sysfs local_cpulist of its PCI device), or
    None when unknown."""
    try:
        import pynvml

        pynvml.nvmlInit()
        bus = pynvml.nvmlDeviceGetPciInfo(pynvml.nvmlDeviceGetHandleByIndex(device_index)).busId
        bus = bus.decode() if isinstance(bus, bytes) else bus
        bus = bus.lower()[-12:]  # domain:bus:device.function as sysfs names it
        text = open(f"/sys/bus/pci/devices/{bus}/local_cpulist").read().strip()
        cpus = set()
        for part in text.split(","):
            a, _, b = part.partition("-")
            cpus.update(range(int(a), int(b or a) + 1))
        cpus &= os.sched_getaffinity(0)
        return cpus or None
    except Exception:
        return None


# ------------------------------------------------------------------ clocks -----------
class ClockSampler:
    """Samples SM clock and throttle reasons with NVML while the timed region runs."""

    REASONS = {
        0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap",
        0x8: "hw_slowdown", 0x10: "sync_boost", 0x20: "sw_thermal_slowdown",
        0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting",
    }

    def __init__(self, device_index):
        self.samples, self.reasons = [], set()
        self.max_mhz = None
        self._stop = threading.Event()
        try:
            import pynvml

            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(device_index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self.nv = None
        self.t = threading.Thread(target=self._run, daemon=True)

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                r = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for bit, name in self.REASONS.items():
                    if r & bit and name != "gpu_idle":
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(0.02)

    def __enter__(self):
        if self.nv:
            self.t.start()
        return self

    def __exit__(self, *exc):
        self._stop.set()
        if self.nv and self.t.is_alive():
            self.t.join()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons)}
        return {"sm_mhz": statistics.median(self.samples), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


# ------------------------------------------------------------------ CPU oracle ---------
def oracle_sample(K, X, w, seconds, threads):
    """Time the oracle (as it stands) on a bounded sample of the workload: a contiguous index
    range of the single epoch, or a slice of the epochs. Returns (mappings/s, sample text)."""
    import oracle

    N, E = w["N"], w["E"]

    def run(n):
        t0 = time.perf_counter()
        if E == 1:
            oracle.oracle_map(K, X, lo=0, hi=min(N, n), threads=threads)
            done = min(N, n)
        else:
            ne = max(1, min(E, n // N))
            oracle.oracle_map(K[:ne], X[:ne], threads=threads)
            done = ne * N
        return done, time.perf_counter() - t0

    n = 1 << 22
    done, dt = run(n)
    while dt < 0.5 and done < w["E"] * N:
        n *= 4
        done, dt = run(n)
    rate = done / dt
    target = int(rate * seconds)
    done, dt = run(max(done, target))
    if E == 1:
        what = f"mapping indices [0, {done}) of the single {w['Q']}x{w['D']} epoch ({done / N:.3%} of it)"
    else:
        what = f"first {done // N} of {E} epochs ({w['Q']}x{w['D']}, {N} mappings each)"
    return done / dt, what, dt


def reference_arm(args, K, X, w, rank, world):
    """--impl reference: the CPU oracle timed on the host cores; rank 0 only."""
    if rank != 0:
        return
    import oracle

    threads = oracle.default_threads()
    total = args.steps + args.warmup
    per_step = max(2.0, min(20.0, 150.0 / max(1, total)))
    rate, what, _ = oracle_sample(K, X, w, 1.0, threads)  # calibration
    n = max(1 << 20, int(rate * per_step))
    times, done_last = [], 0
    for i in range(total):
        t0 = time.perf_counter()
        if w["E"] == 1:
            lo = (i * n) % max(1, w["N"] - n)
            oracle.oracle_map(K, X, lo=lo, hi=min(w["N"], lo + n), threads=threads)
            done = min(w["N"], lo + n) - lo
        else:
            ne = max(1, min(w["E"], n // w["N"]))
            oracle.oracle_map(K[:ne], X[:ne], threads=threads)
            done = ne * w["N"]
        dt = time.perf_counter() - t0
        if i >= args.warmup:
            times.append(dt)
            done_last = done
    ms = 1e3 * statistics.mean(times)
    value = done_last / (ms / 1e3)
    sample = (f"each step: {done_last} mappings of {args.workload} "
              f"({'index range' if w['E'] == 1 else 'epoch slice'}), oracle/oracle.c brute force")
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
        "scaling": "weak" if is_batched(w) else "strong", "vs_baseline": None, "dtype": "u64",
        "data": "synthetic",
        "config": {"workload": args.workload, "desc": w["desc"], "Q": w["Q"], "D": w["D"], "epochs": w["E"]},
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": threads, "kind": "oracle", "sample": sample},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------ our arm ----------
def main():
    args = parse()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    K, X, w = workload(args.workload)
    if args.impl == "reference":
        return reference_arm(args, K, X, w, rank, world)

    import torch
    import torch.distributed as dist

    from paper_conf_cluster_ajipbf15_b200 import Mapper, mcl

    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    # Pinned host arena for the e2e leg, allocated first, in one piece, from the CPUs of the
    # GPU's NUMA node: on the pool's VMs later / separate pinned allocations copied at 14-47
    # instead of 53 GB/s (scripts/e2e_dbg.py), which made the e2e time bimodal by process.
    E0, Q0 = w["E"], w["Q"]
    sizes = [K.nbytes, X.nbytes, E0 * 8, E0 * 8, E0 * Q0]
    offs = [0]
    for n in sizes:
        offs.append(offs[-1] + (n + 255) // 256 * 256)
    prev_cpus = os.sched_getaffinity(0)
    local_cpus = gpu_local_cpus(local)
    if local_cpus:
        os.sched_setaffinity(0, local_cpus)
    arena = torch.empty(offs[-1], dtype=torch.uint8, pin_memory=True)
    os.sched_setaffinity(0, prev_cpus)
    Kh = arena[offs[0]:offs[0] + sizes[0]].view(torch.uint64).view(K.shape)
    Xh = arena[offs[1]:offs[1] + sizes[1]].view(torch.uint64).view(X.shape)
    ih = arena[offs[2]:offs[2] + sizes[2]].view(torch.uint64)
    mh = arena[offs[3]:offs[3] + sizes[3]].view(torch.uint64)
    ph = arena[offs[4]:offs[4] + sizes[4]].view(E0, Q0)
    Kh.copy_(torch.from_numpy(K))
    Xh.copy_(torch.from_numpy(X))
    explicit = args.collective != "auto"
    if world > 1 or explicit:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ.setdefault("MASTER_PORT", "29531")
        dist.init_process_group("nccl", device_id=dev, rank=rank, world_size=world)
    sharded = (world > 1 or explicit) and not is_batched(w)
    comm = None
    if sharded:  # the NCCL communicator: the nccl path, and the fallback of the fused one
        obj = [mcl.mcl_comm_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        comm = mcl.mcl_comm_init(local, world, rank, obj[0])

    # a dedicated stream: the mapper, the L2 flush and the timing events all run on it
    stream = torch.cuda.Stream(dev)
    torch.cuda.set_stream(stream)
    # batched workloads: every rank runs its own full batch (weak scaling, no collective);
    # single-epoch workloads: the index space is sharded across ranks (strong scaling)
    Kd = torch.from_numpy(K).to(dev)
    Xd = torch.from_numpy(X).to(dev)
    E, Q = w["E"], w["Q"]
    idx = torch.empty(E, dtype=torch.uint64, device=dev)
    msp = torch.empty(E, dtype=torch.uint64, device=dev)
    mpg = torch.empty((E, Q), dtype=torch.uint8, device=dev)
    flush = torch.empty(L2_FLUSH_BYTES, dtype=torch.uint8, device=dev)
    flush64 = flush.view(torch.int64)

    def flush_l2(i):
        # write a buffer larger than L2, then read it back: the write evicts everything of
        # ours, the read evicts the write's dirty lines (written back here, not charged to
        # the next kernel's DRAM traffic), leaving L2 clean and holding none of the inputs
        flush.fill_(i & 0xFF)
        flush64.sum()
    mapper = Mapper(local, stream=stream.cuda_stream, nccl_comm=comm, rank=rank if comm else 0,
                    world=world if comm else 1)
    combine = "nccl" if comm else "none"
    if sharded and args.collective != "nccl":
        # fused in-kernel exchange over NVLink peer memory; NCCL stays as the fallback if the
        # slabs cannot be mapped (the choice is agreed by all ranks)
        try:
            mapper.connect_peers(max_epochs=max(1, w["E"]), timeout_ms=60_000)
            ok = 1
        except Exception as exc:  # pragma: no cover
            print(f"[bench] fused exchange unavailable ({exc}); using NCCL", file=sys.stderr)
            ok = 0
        t_ok = torch.tensor([ok], dtype=torch.int32, device=dev)
        dist.all_reduce(t_ok, op=dist.ReduceOp.MIN)
        if int(t_ok[0]):
            combine = "fused"
        elif ok:  # another rank failed: drop the slabs everywhere
            mapper.close()
            mapper = Mapper(local, stream=stream.cuda_stream, nccl_comm=comm, rank=rank, world=world)
    mapper.set_timing(False)

    for _ in range(max(3, args.warmup)):
        mapper.map_queues_into(Kd, Xd, idx, mpg, msp)
    info = mapper.launch_info()

    starts = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    ends = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    launches = 0
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize(dev)
    with ClockSampler(local) as clk:
        for i in range(args.steps):
            flush_l2(i)  # L2 flush between timed steps, outside the events
            starts[i].record(stream)
            mapper.map_queues_into(Kd, Xd, idx, mpg, msp)
            ends[i].record(stream)
            launches += mapper.launch_info()["launches"]
        torch.cuda.synchronize(dev)
    if world > 1:
        dist.barrier()
    step_ms = [s.elapsed_time(e) for s, e in zip(starts, ends)]
    total_ms = sum(step_ms)
    # Kernel-duration pass (outside the timed steps, same launches): a spin kernel holds the
    # stream while the host enqueues the start event and the launch, so the events bracket
    # the search kernel's device execution, not the host launch latency an idle GPU adds.
    mapper.set_timing(True, hold_us=HOLD_US)
    kernel_dev = []
    for i in range(args.steps):
        flush_l2(i)
        mapper.map_queues_into(Kd, Xd, idx, mpg, msp)
        kernel_dev.append(mapper.last_kernel_time_ms()[0])
    mapper.set_timing(False)  # the e2e leg records no library events either
    kern_mean = statistics.mean(kernel_dev)
    t = torch.tensor([total_ms, kern_mean], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    total_ms, kern_mean = float(t[0]), float(t[1])
    ms_per_step = total_ms / args.steps
    mappings_per_step = w["E"] * w["N"] * (world if is_batched(w) else 1)
    value = mappings_per_step / (ms_per_step / 1e3)

    # result agreement across ranks (all ranks hold the identical global argmin)
    res = torch.stack([idx[:1].to(torch.int64), msp[:1].to(torch.int64)]).view(-1)
    if world > 1 and not is_batched(w):
        gathered = [torch.zeros_like(res) for _ in range(world)]
        dist.all_gather(gathered, res)
        assert all((g == res).all() for g in gathered), "ranks disagree on the argmin"

    # ---- e2e through the C ABI with pinned host buffers (H2D + D2H inside the region) ----
    # (host buffers: the pinned arena allocated at start-up)
    e2e_steps = max(10, args.steps)
    mapper.set_pipeline_chunks(args.pipeline_chunks)
    for _ in range(max(3, args.warmup)):
        mapper.map_queues_into(Kh, Xh, ih, ph, mh)
    assert (ih[:1].numpy() == idx[:1].cpu().numpy()).all()
    if world > 1:
        dist.barrier()
    t0 = time.perf_counter()
    for _ in range(e2e_steps):
        mapper.map_queues_into(Kh, Xh, ih, ph, mh)
    e2e_s = torch.tensor([(time.perf_counter() - t0) / e2e_steps], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(e2e_s, op=dist.ReduceOp.MAX)
    e2e_value = mappings_per_step / float(e2e_s[0])
    e2e_chunks = mapper.launch_info()["chunks"]  # pipelined staging (mcl_set_pipeline_chunks)
    h2d = 2 * K.nbytes
    d2h = E * (8 + 8 + Q)

    line = None
    if rank == 0:
        sms = mcl.mcl_device_sms(local)
        clocks = clk.summary()
        max_mhz = clocks.get("sm_max_mhz") or 1965
        # per GPU and launch: the full batch (batched replicas) or this rank's index shard
        mappings_per_launch = w["E"] * w["N"] if is_batched(w) else w["N"] / world
        if info["path"] in ("blocked_u32", "blocked_u32_lean", "blocked_u64", "generic", "flat_u32", "batch_u32"):
            achieved = ALU_INSTR_PER_MAPPING * mappings_per_launch / (kern_mean / 1e3) / 1e12
            peak = ALU_LANES_PER_CLK_SM * sms * max_mhz * 1e6 / 1e12
            roof = {"bound": "alu", "achieved": achieved, "peak": peak, "unit": "Tops/s",
                    "frac": achieved / peak, "traffic": traffic_from_profiles(args.workload),
                    "kernel": KERNEL_NAMES.get(info["path"], info["path"]), "kernel_ms": kern_mean,
                    "kernel_timing": KERNEL_TIMING,
                    "algorithmic": f"{ALU_INSTR_PER_MAPPING} ALU lane-instructions per mapping x "
                                   f"{mappings_per_launch:.4g} mappings per launch",
                    "peak_basis": f"derived: {ALU_LANES_PER_CLK_SM} ALU lanes/clk/SM x {sms} SMs x "
                                  f"{max_mhz} MHz (sm_max); probe-measured rate in peak_measured"}
            try:
                r, per_clk, mhz = mcl.mcl_probe_int_rate(local, 1)
                roof["peak_measured"] = {"vimnmx3_lane_ops_per_s": r, "lane_ops_per_clk_sm": per_clk,
                                         "eff_mhz": mhz, "frac_of_measured": achieved * 1e12 / r}
            except Exception as exc:  # pragma: no cover
                roof["peak_measured"] = {"error": str(exc)}
        else:  # small batched kernel: HBM bound, algorithmic bytes = inputs + outputs
            bytes_per_launch = w["E"] * (2 * Q * w["D"] * 8 + 8 + 8 + Q)
            achieved = bytes_per_launch / (kern_mean / 1e3) / 1e9
            peak = measured_hbm()
            roof = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                    "frac": achieved / peak, "traffic": traffic_from_profiles(args.workload),
                    "kernel": "search_small_kernel", "kernel_ms": kern_mean,
                    "kernel_timing": KERNEL_TIMING}
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
            "scaling": "weak" if is_batched(w) else "strong", "vs_baseline": None, "dtype": "u32",
            "data": "synthetic",
            "config": {"workload": args.workload, "desc": w["desc"], "Q": Q, "D": w["D"],
                       "epochs": w["E"], "mappings_per_step": mappings_per_step,
                       "parallelism": (f"index-range shard x{world} + " + (
                           "in-kernel peer exchange (fused atomicMin over NVLink)" if combine == "fused"
                           else "ncclAllReduce(min)")) if sharded
                       else (f"epoch replicas x{world}" if world > 1 else "1 GPU"),
                       "combine": combine,
                       "l2": "flushed between timed steps (256 MiB write + read-back, outside the events)",
                       "path": info["path"], "ctas": info["ctas"], "threads": info["threads"],
                       "result": {"index": int(idx[0]), "makespan": int(msp[0])}},
            "clocks": clocks,
            "gpu_launches": launches,
            "e2e": {"value": e2e_value, "unit": UNIT, "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
                    "ms_per_step": float(e2e_s[0]) * 1e3, "pipelined_chunks": e2e_chunks,
                    "host_buffers": "one pinned arena allocated at start-up on the GPU's NUMA node"
                    if local_cpus else "one pinned arena allocated at start-up"},
            "roofline": roof,
        }
    mapper.close()
    if comm:
        mcl.mcl_comm_destroy(comm)
    if dist.is_initialized():
        dist.barrier()
        dist.destroy_process_group()
    if rank == 0:
        if world == 1 and not args.no_cpu_baseline:
            import oracle

            threads = oracle.default_threads()
            rate, what, dt = oracle_sample(K, X, w, args.cpu_seconds, threads)
            line["cpu_baseline"] = {"value": rate, "unit": UNIT, "cores": threads, "kind": "oracle",
                                    "sample": f"{what}; {dt:.1f} s on {threads} threads"}
        print(json.dumps(line), flush=True)


def measured_hbm():
    try:
        return float(json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"])
    except Exception:
        return 6650.0  # B200_PROFILING.md fallback


def traffic_from_profiles(workload):
    """dram bytes (read + write) per launch of the dominant kernel, from the committed ncu
    --set full summary (profiles/ncu_traffic.json), else None."""
    try:
        d = json.load(open(os.path.join(ROOT, "profiles", "ncu_traffic.json")))
        return d[workload]["dram_bytes_per_launch"]
    except Exception:
        return None


if __name__ == "__main__":
    main()
