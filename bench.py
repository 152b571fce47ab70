#!/usr/bin/env python
"""bench.py -- queue->device mappings scored per second on B200 (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload cfg5] [--impl mcl|reference]
    python -m torch.distributed.run --nproc-per-node N --master-addr 127.0.0.1 bench.py --gpus N

A step is one mcl_map_queues call: the whole hot path (cost composition, mixed-radix
enumeration, per-device loads, makespan, argmin with lowest-index ties, the cross-GPU
combine when N > 1, and the output decode) on one synthetic workload already resident in
HBM. Headline workload (`value`): cfg5 = 12 queues x 8 devices (8^12 = 6.9e10 mappings, one
epoch), the largest single-GPU configuration and the one BASELINE.json's scaling target
names; at N GPUs its index space is sharded by contiguous ranges (strong scaling) and the
ranks' packed (makespan, index) keys are combined INSIDE the search kernel over NVLink peer
memory (the fused exchange, include/mcl.h mcl_peer_import; `--collective nccl` uses
ncclAllReduce(MIN) + a decode kernel instead). The other four BASELINE configs are measured
in the same run and reported under `configs` (every config reported);
`--only` skips them.

Process plumbing: one process per GPU; torch.distributed with the gloo backend is the
control plane (barriers, the max-over-ranks timing reduction, the exchange of the peer
slabs' IPC handles). The data plane is the library's own: the in-kernel peer exchange, or
an NCCL communicator created only for `--collective nccl`. Ranks beyond the visible GPU
count share GPUs round-robin (a 2-rank run on one GPU proves the N > 1 flow end to end;
its timing is not a scaling number).

Rank 0 prints one JSON line. `value` is whole-job mappings/s from CUDA events over exactly
K timed steps (L2 flushed between steps, outside the events), max over ranks; `e2e` is the
same metric through the C ABI with pinned host buffers (H2D + D2H inside the timed region;
batched workloads stage in pipelined chunks, `e2e.pipelined_chunks`); `roofline` is the
dominant kernel's algorithmic rate against its roofline: `frac` on the 1.5 ALU
lane-instructions per mapping floor (SS7) and `frac_survey` on SURVEY SS8(d)'s 2
integer ops per mapping, both against the derived ALU peak (the probe-measured rates beside
them); `cpu_baseline` is the CPU oracle timed on a bounded sample of the workload on the
host's cores (plus one thread for cfg1-3). `--impl reference` times the oracle instead (this
tier's reference arm).
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
SURVEY_OPS_PER_MAPPING = 2      # one max forms the makespan, one min folds it
L2_FLUSH_BYTES = 256 << 20      # > 126 MB L2
HOLD_US = 200                   # spin ahead of each kernel-duration launch (> host launch latency)
ALL_CONFIGS = ["cfg1", "cfg2", "cfg3", "cfg4", "cfg5"]
ONE_THREAD_CONFIGS = ("cfg1", "cfg2", "cfg3")  # single-thread oracle for cfg1-3
KERNEL_TIMING = ("CUDA events on the mapper's stream around the search launch, in a pass of `steps` "
                 "launches right after the timed steps (L2 flushed before each, as there), each preceded "
                 "by a 200 us spin kernel so the events measure device execution; the timed steps record "
                 "no library events (one timing-event record costs ~2.7 us of host time, "
                 "scripts/archive/host_api_costs.cu, which the step would be charged)")
KERNEL_NAMES = {"blocked_u32": "search_blocked_kernel<u32, D>",
                "blocked_u32_lean": "search_blocked_kernel<u32, 5, lean>",
                "blocked_u64": "search_blocked_kernel<u64, D>",
                "generic": "search_generic_kernel", "flat_u32": "search_flat_kernel<u32, D>",
                "small_batched": "search_small_kernel<Q, D> / search_tiny_kernel<Q, D>",
                "batch_u32": "search_batch_kernel<Q, D>",
                "batch_pool_u32": "search_pool_kernel<Q, D>"}
ALU_PATHS = ("blocked_u32", "blocked_u32_lean", "blocked_u64", "generic", "flat_u32", "batch_u32", "batch_pool_u32")


def parse(argv=None):
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=20)
    p.add_argument("--warmup", type=int, default=5)
    p.add_argument("--workload", default="cfg5", choices=ALL_CONFIGS,
                   help="headline workload (value); the others go under `configs`")
    p.add_argument("--only", action="store_true", help="measure the headline workload only")
    p.add_argument("--impl", default="mcl", choices=["mcl", "reference"])
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--pipeline-chunks", type=int, default=0,
                   help="e2e staging of the host-resident batch: 0 auto, 1 off, n chunks")
    p.add_argument("--cpu-seconds", type=float, default=12.0, help="CPU-oracle sample budget (headline)")
    p.add_argument("--config-cpu-seconds", type=float, default=2.5,
                   help="CPU-oracle sample budget per other config and thread count")
    p.add_argument("--ref-step-seconds", type=float, default=None,
                   help="reference arm: oracle seconds per step (default: ~150 s over all steps, 2-20 s each)")
    p.add_argument("--collective", default="auto", choices=["auto", "fused", "nccl"],
                   help="cross-GPU combine of a sharded single-epoch search: fused = in-kernel "
                        "exchange over peer memory (NEXT-2), nccl = ncclAllReduce + decode kernel; "
                        "auto = fused when N > 1. An explicit choice also runs it with one rank.")
    return p.parse_args(argv)


def workload(name):
    from paper_conf_cluster_ajipbf15_b200 import workloads

    K, X = workloads.make(name)
    E, Q, D = K.shape
    return K, X, dict(name=name, E=E, Q=Q, D=D, N=D**Q, desc=workloads.CONFIGS[name]["desc"])


def is_batched(w):
    return w["E"] > 1


def resident_eligible(w):
    """Decision-sized epochs the resident mapper serves (include/mcl.h mcl_resident_start:
    D^Q <= 4096, Q <= 16, D <= 16, at most 64 epochs per call)."""
    return w["N"] <= 4096 and w["Q"] <= 16 and w["D"] <= 16 and w["E"] <= 64


def is_replicated(w):
    """Workloads every rank runs whole (weak scaling, no collective): epoch batches, and a
    single decision too small to shard (cfg1: 81 mappings; SS8)."""
    return is_batched(w) or w["N"] < (1 << 20)


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
    range of the single epoch, a slice of the epochs, or -- for a single epoch too small to
    time (cfg1: 81 mappings) -- the epoch repeated as a batch of identical decisions, so the
    rate is the search's, not one ctypes call's. Returns (mappings/s, sample text, seconds,
    extra dict)."""
    import oracle

    N, E = w["N"], w["E"]
    tiny = E == 1 and N < (1 << 16)

    def run(n):
        t0 = time.perf_counter()
        if tiny:
            reps = max(1, n // N)
            oracle.oracle_map(np.repeat(K, reps, axis=0), np.repeat(X, reps, axis=0), threads=threads)
            done = reps * N
        elif E == 1:
            oracle.oracle_map(K, X, lo=0, hi=min(N, n), threads=threads)
            done = min(N, n)
        else:
            ne = max(1, min(E, n // N))
            oracle.oracle_map(K[:ne], X[:ne], threads=threads)
            done = ne * N
        return done, time.perf_counter() - t0

    n = 1 << 16 if tiny else 1 << 22
    done, dt = run(n)
    while dt < 0.3 and (tiny or done < E * N):
        n *= 4
        done, dt = run(n)
    rate = done / dt
    done, dt = run(max(done, int(rate * seconds)))
    extra = {}
    if tiny:
        what = f"the single {w['Q']}x{w['D']} epoch repeated {done // N} times as one batch"
        t0 = time.perf_counter()
        for _ in range(200):
            oracle.oracle_map(K, X, threads=threads)
        extra["latency_us_per_call"] = (time.perf_counter() - t0) / 200 * 1e6
        extra["latency_note"] = "one oracle_map call on the single epoch through ctypes (Python overhead included)"
    elif E == 1:
        what = f"mapping indices [0, {done}) of the single {w['Q']}x{w['D']} epoch ({done / N:.3%} of it)"
    else:
        what = f"first {done // N} of {E} epochs ({w['Q']}x{w['D']}, {N} mappings each)"
    return done / dt, what, dt, extra


def cpu_baseline(K, X, w, seconds, threads):
    rate, what, dt, extra = oracle_sample(K, X, w, seconds, threads)
    d = {"value": rate, "unit": UNIT, "cores": threads, "kind": "oracle",
         "sample": f"{what}; {dt:.1f} s on {threads} thread{'s' if threads > 1 else ''}"}
    d.update(extra)
    return d


def reference_arm(args, rank):
    """--impl reference: the CPU oracle timed on the host cores; rank 0 only."""
    if rank != 0:
        return
    import oracle

    K, X, w = workload(args.workload)
    threads = oracle.default_threads()
    total = args.steps + args.warmup
    per_step = args.ref_step_seconds or max(2.0, min(20.0, 150.0 / max(1, total)))
    rate, _, _, _ = oracle_sample(K, X, w, 1.0, threads)  # calibration
    n = max(1 << 20, int(rate * per_step))
    tiny = w["E"] == 1 and w["N"] < (1 << 16)
    times, done_last = [], 0
    for i in range(total):
        t0 = time.perf_counter()
        if tiny:
            reps = max(1, n // w["N"])
            oracle.oracle_map(np.repeat(K, reps, axis=0), np.repeat(X, reps, axis=0), threads=threads)
            done = reps * w["N"]
        elif w["E"] == 1:
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
    kind = "repeated epoch" if tiny else ("index range" if w["E"] == 1 else "epoch slice")
    sample = f"each step: {done_last} mappings of {args.workload} ({kind}), oracle/oracle.c brute force"
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
        "scaling": "weak" if is_replicated(w) else "strong", "vs_baseline": None, "dtype": "u64",
        "data": "synthetic",
        "config": {"workload": args.workload, "desc": w["desc"], "Q": w["Q"], "D": w["D"], "epochs": w["E"]},
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": threads, "kind": "oracle", "sample": sample},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------ our arm ----------
class Ctx:
    """Per-process state shared by the config measurements."""

    def __init__(self, args):
        self.args = args
        self.world = int(os.environ.get("WORLD_SIZE", "1"))
        self.rank = int(os.environ.get("RANK", "0"))
        self.local = int(os.environ.get("LOCAL_RANK", "0"))
        self.explicit = args.collective != "auto"
        self.dist = None
        self.comm = None
        self.arena = None
        self.fused_failed = False  # the fused exchange failed once: NCCL for the rest of the run


def max_over_ranks(ctx, values):
    """Element-wise max over ranks of a list of floats (gloo control plane, CPU tensors)."""
    if ctx.world == 1:
        return list(values)
    import torch

    t = torch.tensor(values, dtype=torch.float64)
    ctx.dist.all_reduce(t, op=ctx.dist.ReduceOp.MAX)
    return t.tolist()


def barrier(ctx):
    if ctx.world > 1:
        ctx.dist.barrier()


def roofline(w, info, kern_ms, sms, max_mhz, world, mcl, dev_index):
    """The dominant kernel's algorithmic rate against its roofline (SS7)."""
    if info["path"] in ALU_PATHS:
        per_launch = w["E"] * w["N"] if is_replicated(w) else w["N"] / world
        mps = per_launch / (kern_ms / 1e3)
        peak = ALU_LANES_PER_CLK_SM * sms * max_mhz * 1e6 / 1e12
        achieved = ALU_INSTR_PER_MAPPING * mps / 1e12
        survey = SURVEY_OPS_PER_MAPPING * mps / 1e12
        roof = {"bound": "alu", "achieved": achieved, "peak": peak, "unit": "Tops/s",
                "frac": achieved / peak,
                "achieved_survey": survey, "frac_survey": survey / peak,
                "traffic": traffic_from_profiles(w["name"]),
                "kernel": KERNEL_NAMES.get(info["path"], info["path"]), "kernel_ms": kern_ms,
                "kernel_timing": KERNEL_TIMING,
                "algorithmic": f"frac: {ALU_INSTR_PER_MAPPING} ALU lane-instructions per mapping (the floor "
                               f"with the 3-input VIMNMX3 fold, DESIGN.md SS7); frac_survey: "
                               f"{SURVEY_OPS_PER_MAPPING} integer ops per mapping (SURVEY SS8(d)); x "
                               f"{per_launch:.4g} mappings per launch",
                "peak_basis": f"derived: {ALU_LANES_PER_CLK_SM} ALU lanes/clk/SM x {sms} SMs x "
                              f"{max_mhz} MHz (sm_max); probe-measured rates in peak_measured"}
        try:
            pm = {}
            for op, name in ((0, "vimnmx2"), (1, "vimnmx3")):
                r, per_clk, mhz = mcl.mcl_probe_int_rate(dev_index, op)
                pm[name] = {"lane_ops_per_s": r, "lane_ops_per_clk_sm": per_clk, "eff_mhz": mhz}
            pm["frac_of_measured_vimnmx3"] = achieved * 1e12 / pm["vimnmx3"]["lane_ops_per_s"]
            pm["frac_survey_of_measured_vimnmx2"] = survey * 1e12 / pm["vimnmx2"]["lane_ops_per_s"]
            roof["peak_measured"] = pm
        except Exception as exc:  # pragma: no cover
            roof["peak_measured"] = {"error": str(exc)}
        return roof
    if w["N"] < 256 and w["E"] == 1:  # cfg1: 81 mappings, one decision
        return {"bound": "latency", "kernel": KERNEL_NAMES.get(info["path"], info["path"]),
                "kernel_ms": kern_ms, "kernel_timing": KERNEL_TIMING,
                "note": "81 mappings per call: launch + sync latency bound, no throughput roofline (SURVEY SS8(d))"}
    # small batched kernel: HBM bound, algorithmic bytes = inputs + outputs
    bytes_per_launch = w["E"] * (2 * w["Q"] * w["D"] * 8 + 8 + 8 + w["Q"])
    achieved = bytes_per_launch / (kern_ms / 1e3) / 1e9
    peak = measured_hbm()
    return {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
            "frac": achieved / peak, "traffic": traffic_from_profiles(w["name"]),
            "kernel": KERNEL_NAMES.get(info["path"], info["path"]), "kernel_ms": kern_ms,
            "kernel_timing": KERNEL_TIMING,
            "algorithmic": f"{2 * w['Q'] * w['D'] * 8 + 16 + w['Q']} B per epoch (K + X in, index + makespan "
                           f"+ mapping out) x {w['E']} epochs"}


def measure(ctx, name):
    """One config on this rank's GPU: warm-up, K timed steps (device resident), the
    kernel-duration pass, and the e2e leg through host buffers. Returns rank 0's entry (or
    None on other ranks)."""
    import torch

    from paper_conf_cluster_ajipbf15_b200 import Mapper, mcl

    args, world, rank = ctx.args, ctx.world, ctx.rank
    dev, dev_index = ctx.dev, ctx.dev_index
    K, X, w = workload(name)
    E, Q, D = w["E"], w["Q"], w["D"]
    sharded = (world > 1 or ctx.explicit) and not is_replicated(w)

    # host buffers of the e2e leg: views into the pinned arena allocated at start-up
    sizes = [K.nbytes, X.nbytes, E * 8, E * 8, E * Q]
    offs = [0]
    for n in sizes:
        offs.append(offs[-1] + (n + 255) // 256 * 256)
    arena = ctx.arena
    Kh = arena[offs[0]:offs[0] + sizes[0]].view(torch.uint64).view(K.shape)
    Xh = arena[offs[1]:offs[1] + sizes[1]].view(torch.uint64).view(X.shape)
    ih = arena[offs[2]:offs[2] + sizes[2]].view(torch.uint64)
    mh = arena[offs[3]:offs[3] + sizes[3]].view(torch.uint64)
    ph = arena[offs[4]:offs[4] + sizes[4]].view(E, Q)
    Kh.copy_(torch.from_numpy(K))
    Xh.copy_(torch.from_numpy(X))

    stream = ctx.stream
    Kd = torch.from_numpy(K).to(dev)
    Xd = torch.from_numpy(X).to(dev)
    idx = torch.empty(E, dtype=torch.uint64, device=dev)
    msp = torch.empty(E, dtype=torch.uint64, device=dev)
    mpg = torch.empty((E, Q), dtype=torch.uint8, device=dev)
    torch.cuda.synchronize(dev)
    flush, flush64 = ctx.flush, ctx.flush64

    def flush_l2(i):
        # write a buffer larger than L2, then read it back: the write evicts everything of
        # ours, the read evicts the write's dirty lines (written back here, not charged to
        # the next kernel's DRAM traffic), leaving L2 clean and holding none of the inputs
        flush.fill_(i & 0xFF)
        flush64.sum()

    comm = ctx.comm if sharded else None
    mapper = Mapper(dev_index, stream=stream.cuda_stream, nccl_comm=comm,
                    rank=rank if sharded else 0, world=world if sharded else 1)
    combine = "nccl" if comm else "none"
    if sharded and args.collective != "nccl" and not ctx.fused_failed:
        # fused in-kernel exchange over NVLink peer memory, validated by one sharded call
        # against the same call's answer on a single GPU; all ranks agree (gloo) -- if any
        # rank cannot map the slabs or the exchange fails, every rank falls back to an NCCL
        # communicator instead of failing the run
        ok = 1
        try:
            mapper.connect_peers(max_epochs=1, timeout_ms=20_000)
            Kv, Xv = Kd[:1], Xd[:1]
            vi, _, vm = mapper.map_queues(Kv, Xv, with_mapping=False)
            with Mapper(dev_index, stream=stream.cuda_stream) as solo:
                si, _, sm = solo.map_queues(Kv, Xv, with_mapping=False)
            ok = int(bool((vi == si).all() and (vm == sm).all()))
        except Exception as exc:  # pragma: no cover
            print(f"[bench] fused exchange unavailable ({exc})", file=sys.stderr)
            ok = 0
        if -max_over_ranks(ctx, [-ok])[0] < 1:  # min over ranks
            print("[bench] fused exchange unusable on some rank: NCCL communicator instead", file=sys.stderr)
            ctx.fused_failed = True
            mapper.close()
        else:
            combine = "fused"
    if sharded and combine == "none":  # --collective nccl, or the fused exchange's fallback
        if ctx.comm is None:
            obj = [mcl.mcl_comm_unique_id() if rank == 0 else None]
            ctx.dist.broadcast_object_list(obj, src=0)
            ctx.comm = mcl.mcl_comm_init(dev_index, world, rank, obj[0])
        if mapper.handle:
            mapper.close()
        mapper = Mapper(dev_index, stream=stream.cuda_stream, nccl_comm=ctx.comm, rank=rank, world=world)
        combine = "nccl"
    mapper.set_timing(False)

    for _ in range(max(3, args.warmup)):
        mapper.map_queues_into(Kd, Xd, idx, mpg, msp)
    info = mapper.launch_info()

    starts = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    ends = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    launches = 0
    barrier(ctx)
    torch.cuda.synchronize(dev)
    with ClockSampler(dev_index) as clk:
        for i in range(args.steps):
            flush_l2(i)  # L2 flush between timed steps, outside the events
            starts[i].record(stream)
            mapper.map_queues_into(Kd, Xd, idx, mpg, msp)
            ends[i].record(stream)
            launches += mapper.launch_info()["launches"]
        torch.cuda.synchronize(dev)
    barrier(ctx)
    total_ms = sum(s.elapsed_time(e) for s, e in zip(starts, ends))
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

    # result agreement across ranks (all ranks hold the identical global argmin)
    agree = None
    if world > 1 and sharded:
        res = torch.tensor([int(idx[0].item()), int(msp[0].item())], dtype=torch.int64)
        gathered = [torch.zeros_like(res) for _ in range(world)]
        ctx.dist.all_gather(gathered, res)
        agree = all(bool((g == res).all()) for g in gathered)
        assert agree, f"ranks disagree on the argmin: {[g.tolist() for g in gathered]}"

    # ---- e2e through the C ABI with pinned host buffers (H2D + D2H inside the region) ----
    e2e_steps = max(10, args.steps)
    mapper.set_pipeline_chunks(args.pipeline_chunks)
    for _ in range(max(3, args.warmup)):
        mapper.map_queues_into(Kh, Xh, ih, ph, mh)
    assert (ih[:1].numpy() == idx[:1].cpu().numpy()).all()
    barrier(ctx)
    t0 = time.perf_counter()
    for _ in range(e2e_steps):
        mapper.map_queues_into(Kh, Xh, ih, ph, mh)
    e2e_s = (time.perf_counter() - t0) / e2e_steps
    e2e_chunks = mapper.launch_info()["chunks"]  # pipelined staging (mcl_set_pipeline_chunks)
    result = {"index": int(idx[0].item()), "makespan": int(msp[0].item())}
    # ---- decision-sized searches: the same through the resident mapper (mcl_resident_*,
    # one warp left on the GPU serving a pinned host mailbox; no launch per call) ----
    e2e_launch_s, res_s = e2e_s, None
    if resident_eligible(w) and not sharded and not os.environ.get("MCL_BENCH_NO_RESIDENT"):
        # (MCL_BENCH_NO_RESIDENT=1 under profilers that serialise launches: a resident
        # kernel then only returns after its idle timeout)
        Kn, Xn = Kh.numpy(), Xh.numpy()
        outs = (ih.numpy(), ph.numpy(), mh.numpy())
        mapper.resident_start(Q, D, max_epochs=E)
        try:
            for _ in range(max(3, args.warmup) * 10):
                mapper.resident_map(Kn, Xn, out=outs)
            assert int(outs[0][0]) == result["index"] and int(outs[2][0]) == result["makespan"]
            barrier(ctx)
            t0 = time.perf_counter()
            for _ in range(e2e_steps * 10):
                mapper.resident_map(Kn, Xn, out=outs)
            res_s = (time.perf_counter() - t0) / (e2e_steps * 10)
        finally:
            mapper.resident_stop()
        e2e_s = res_s  # the call a user makes for a single decision
    mapper.close()

    total_ms, kern_mean, e2e_s, e2e_launch_s = max_over_ranks(ctx, [total_ms, kern_mean, e2e_s, e2e_launch_s])
    ms_per_step = total_ms / args.steps
    mappings_per_step = E * w["N"] * (world if is_replicated(w) else 1)
    value = mappings_per_step / (ms_per_step / 1e3)
    e2e_value = mappings_per_step / e2e_s
    if rank != 0:
        return None
    sms = mcl.mcl_device_sms(dev_index)
    clocks = clk.summary()
    max_mhz = clocks.get("sm_max_mhz") or 1965
    entry = {
        "value": value, "unit": UNIT, "ms_per_step": ms_per_step,
        "scaling": "weak" if is_replicated(w) else "strong",
        "config": {"workload": name, "desc": w["desc"], "Q": Q, "D": D, "epochs": E,
                   "mappings_per_step": mappings_per_step,
                   "parallelism": (f"index-range shard x{world} + " + (
                       "in-kernel peer exchange (fused atomicMin over NVLink)" if combine == "fused"
                       else "ncclAllReduce(min)")) if sharded
                   else ((f"epoch replicas x{world}" if is_batched(w) else f"decision replicas x{world}")
                         if world > 1 else "1 GPU"),
                   "combine": combine,
                   "l2": "flushed between timed steps (256 MiB write + read-back, outside the events)",
                   "path": info["path"], "ctas": info["ctas"], "threads": info["threads"],
                   "result": result},
        "clocks": clocks,
        "gpu_launches": launches,
        "e2e": {"value": e2e_value, "unit": UNIT, "h2d_bytes_per_step": K.nbytes + X.nbytes,
                # resident: one three-word record per epoch (kernels.h ResidentArgs)
                "d2h_bytes_per_step": E * 24 if res_s is not None else E * (8 + 8 + Q),
                "ms_per_step": e2e_s * 1e3,
                "api": ("mcl_resident_map (resident warp; inputs read in place over PCIe, results "
                        "written back to the pinned mailbox)" if res_s is not None
                        else "mcl_map_queues on pinned host buffers"),
                "pipelined_chunks": e2e_chunks,
                "host_buffers": "one pinned arena allocated at start-up on the GPU's NUMA node"
                if ctx.local_cpus else "one pinned arena allocated at start-up"},
        "roofline": roofline(w, info, kern_mean, sms, max_mhz, world, mcl, dev_index),
    }
    if agree is not None:
        entry["ranks_agree"] = agree
    if name == "cfg1":
        entry["latency_us"] = {"device_resident_launch": ms_per_step * 1e3,
                               "host_buffers_launch": e2e_launch_s * 1e6,
                               "host_buffers_resident": res_s * 1e6 if res_s is not None else None}
    return entry


def arena_bytes(names):
    """Bytes of the pinned host arena: the largest config's inputs + outputs."""
    from paper_conf_cluster_ajipbf15_b200 import workloads

    best = 0
    for n in names:
        c = workloads.CONFIGS[n]
        E, Q, D = c["E"], c["Q"], c["D"]
        tot = 0
        for b in (E * Q * D * 8, E * Q * D * 8, E * 8, E * 8, E * Q):
            tot += (b + 255) // 256 * 256
        best = max(best, tot)
    return best


def main():
    args = parse()
    ctx = Ctx(args)
    if args.impl == "reference":
        return reference_arm(args, ctx.rank)

    import torch
    import torch.distributed as dist

    from paper_conf_cluster_ajipbf15_b200 import mcl

    ndev = torch.cuda.device_count()
    ctx.dev_index = ctx.local % max(1, ndev)  # ranks beyond the visible GPUs share them
    torch.cuda.set_device(ctx.dev_index)
    ctx.dev = torch.device("cuda", ctx.dev_index)
    names = [args.workload] + ([] if args.only else [n for n in ALL_CONFIGS if n != args.workload])
    # Pinned host arena for the e2e legs, allocated first, in one piece, from the CPUs of the
    # GPU's NUMA node: on the pool's VMs later / separate pinned allocations copied at 14-47
    # instead of 53 GB/s (scripts/archive/e2e_dbg.py), which made the e2e time bimodal by process.
    prev_cpus = os.sched_getaffinity(0)
    ctx.local_cpus = gpu_local_cpus(ctx.dev_index)
    if ctx.local_cpus:
        os.sched_setaffinity(0, ctx.local_cpus)
    ctx.arena = torch.empty(arena_bytes(names), dtype=torch.uint8, pin_memory=True)
    os.sched_setaffinity(0, prev_cpus)
    if ctx.world > 1 or ctx.explicit:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ.setdefault("MASTER_PORT", "29531")
        dist.init_process_group("gloo", rank=ctx.rank, world_size=ctx.world)  # control plane only
        ctx.dist = dist
    if args.collective == "nccl":  # the NCCL data plane: a communicator of the library's own
        obj = [mcl.mcl_comm_unique_id() if ctx.rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        ctx.comm = mcl.mcl_comm_init(ctx.dev_index, ctx.world, ctx.rank, obj[0])

    # a dedicated stream: the mapper, the L2 flush and the timing events all run on it
    ctx.stream = torch.cuda.Stream(ctx.dev)
    torch.cuda.set_stream(ctx.stream)
    ctx.flush = torch.empty(L2_FLUSH_BYTES, dtype=torch.uint8, device=ctx.dev)
    ctx.flush64 = ctx.flush.view(torch.int64)

    entries = {}
    t_all = time.perf_counter()
    for n in names:
        entries[n] = measure(ctx, n)
    # after every timed region: what CUDA events report around a kernel that does nothing,
    # timed as the configs' kernel_ms are (the share of a short kernel's kernel_ms that no
    # kernel can avoid on this platform; SS12)
    floor = None
    if ctx.rank == 0:
        try:
            k_us, e_us = mcl.mcl_probe_launch_floor(ctx.dev_index, 30)
            floor = {"empty_kernel_us": k_us, "events_only_us": e_us,
                     "note": "CUDA events around an empty 148 x 512 kernel after a 200 us hold "
                             "(mcl_probe_launch_floor), as kernel_ms is timed; not subtracted anywhere"}
        except Exception as exc:  # pragma: no cover
            floor = {"error": str(exc)}
    if ctx.comm:
        mcl.mcl_comm_destroy(ctx.comm)
    if dist.is_initialized():
        dist.barrier()
        dist.destroy_process_group()
    if ctx.rank != 0:
        return
    head = entries[args.workload]
    line = {
        "metric": METRIC, "value": head["value"], "unit": UNIT, "n_gpus": ctx.world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": head["ms_per_step"],
        "higher_is_better": True, "scaling": head["scaling"], "vs_baseline": None, "dtype": "u32",
        "data": "synthetic", "config": head["config"], "clocks": head["clocks"],
        "gpu_launches": head["gpu_launches"], "e2e": head["e2e"], "roofline": head["roofline"],
    }
    if "ranks_agree" in head:
        line["ranks_agree"] = head["ranks_agree"]
    if floor is not None:
        line["launch_floor"] = floor
    others = {n: e for n, e in entries.items() if n != args.workload}
    if ctx.world == 1 and not args.no_cpu_baseline:
        import oracle

        threads = oracle.default_threads()
        K, X, w = workload(args.workload)
        line["cpu_baseline"] = cpu_baseline(K, X, w, args.cpu_seconds, threads)
        for n, e in others.items():
            K, X, w = workload(n)
            e["cpu_baseline"] = cpu_baseline(K, X, w, args.config_cpu_seconds, threads)
            if n in ONE_THREAD_CONFIGS:
                e["cpu_baseline_1t"] = cpu_baseline(K, X, w, args.config_cpu_seconds, 1)
    if others:
        line["configs"] = others
    line["bench_wall_s"] = time.perf_counter() - t_all
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
