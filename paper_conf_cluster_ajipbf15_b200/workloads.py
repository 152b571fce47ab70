"""Seeded synthetic inputs for the mapper (the five BASELINE.json configs + test families).

This module only DRAWS inputs; it holds none of the mapper's arithmetic (no cost
composition, no loads, no makespans). It is the one module shared by the CUDA path's
tests/bench and the oracle's tests, as DESIGN.md "Input recipe" describes. Magnitudes are
assumptions shaped by the paper, not values the paper prints.

Every generator returns ``(K, X)``: ``uint64`` arrays ``[E, Q, D]`` in integer
nanoseconds, C order. Device 0 is the "CPU" (data resident on the host, so X[:, :, 0] = 0,
PAPER.md L1293-1301 / L1349-1361); devices >= 1 are "GPUs".
"""
from __future__ import annotations

import math

import numpy as np

# Fig. 3: GPU-over-CPU relative time per SNU-NPB benchmark; five of
# six favour the CPU, EP favours the GPU (CPU up to 20x slower, L2058-2060).
NPB_RATIO = {"BT": 4.0, "CG": 1.6, "EP": 0.05, "FT": 1.8, "MG": 3.5, "SP": 1.5}
NPB_SEED = {"BT": 100, "CG": 101, "EP": 102, "FT": 103, "MG": 104, "SP": 105}
MIB = 1 << 20
H2D_BYTES_PER_NS = 5.0  # 5 GB/s PCIe-2-era host->device, expressed in bytes per ns


def cfg1_npb(name: str = "FT", seed: int | None = None):
    """cfg1: 4 queues x 3 devices (CPU, GPU0, GPU1), one epoch, SNU-NPB-like."""
    rng = np.random.default_rng(NPB_SEED[name] if seed is None else seed)
    Q, D = 4, 3
    r = NPB_RATIO[name]
    K = np.zeros((1, Q, D), dtype=np.uint64)
    X = np.zeros((1, Q, D), dtype=np.uint64)
    for q in range(Q):
        kc = int(rng.integers(5_000_000, 50_000_001))
        K[0, q, 0] = kc
        nbytes = 64 * MIB if name == "FT" else int(rng.integers(4 * MIB, 16 * MIB + 1))
        for g in (1, 2):
            eps = rng.uniform(-0.02, 0.02)
            K[0, q, g] = int(round(kc * r * (1.0 + eps)))
            X[0, q, g] = int(math.ceil(nbytes / H2D_BYTES_PER_NS))
    return K, X


def cfg1_random(seed: int, Q: int = 4, D: int = 3, hi: int = 1 << 20):
    rng = np.random.default_rng(seed)
    K = rng.integers(0, hi, size=(1, Q, D), dtype=np.uint64)
    X = rng.integers(0, hi, size=(1, Q, D), dtype=np.uint64)
    X[:, :, 0] = 0
    return K, X


def cfg2(E: int = 10_000, seed: int = 2, Q: int = 8, D: int = 4, adversarial: float = 0.05):
    """cfg2: 8 queues x 4 devices, batch of E epochs. K log-uniform in [1e3, 2^20) ns,
    X[:, :, 1:] uniform in {0..2^19}; a fraction of adversarial epochs (all-equal, zeros,
    one-hot cheap device)."""
    rng = np.random.default_rng(seed)
    lo, hi = math.log(1e3), math.log(float(1 << 20))
    K = np.floor(np.exp(rng.uniform(lo, hi, size=(E, Q, D)))).astype(np.uint64)
    K = np.minimum(K, np.uint64((1 << 20) - 1))
    X = rng.integers(0, (1 << 19) + 1, size=(E, Q, D), dtype=np.uint64)
    X[:, :, 0] = 0
    n_adv = int(E * adversarial)
    if n_adv:
        which = rng.choice(E, size=n_adv, replace=False)
        for t, e in enumerate(which):
            kind = t % 3
            if kind == 0:  # all-equal: maximal ties
                c = int(rng.integers(1, 1 << 19))
                K[e] = c
                X[e] = 0
            elif kind == 1:  # all zero: every mapping ties at 0
                K[e] = 0
                X[e] = 0
            else:  # one device is much cheaper for every queue
                d = int(rng.integers(0, D))
                K[e] = (1 << 19)
                X[e] = 0
                K[e, :, d] = rng.integers(1, 64, size=Q, dtype=np.uint64)
    return K, X


def cfg3(E: int = 1_000_000, seed: int = 3):
    """cfg3: FDM-Seismology-shaped, 2 queues x 3 devices, E epochs alternating the
    column-major regime (all-CPU best) and the row-major regime (two GPUs best, large
    transfer costs), PAPER.md L2229-2251 (Fig. 9) and L2304-2326 (Fig. 10)."""
    rng = np.random.default_rng(seed)
    Q, D = 2, 3
    K = np.zeros((E, Q, D), dtype=np.float64)
    X = np.zeros((E, Q, D), dtype=np.float64)
    col = (np.arange(E) % 2) == 0
    nc, nr = int(col.sum()), int((~col).sum())
    # column-major epochs
    kc = rng.uniform(1.0e8, 1.4e8, size=(nc, Q))
    K[col, :, 0] = kc
    K[col, :, 1:] = kc[:, :, None] * rng.uniform(1.3, 1.5, size=(nc, Q, 2))
    X[col, :, 1:] = kc[:, :, None] * rng.uniform(1.2, 1.4, size=(nc, Q, 2))
    # row-major epochs
    kg = rng.uniform(2.0e8, 2.5e8, size=(nr, Q, 2))
    xg = rng.uniform(1.5e8, 2.0e8, size=(nr, Q, 2))
    K[~col, :, 1:] = kg
    X[~col, :, 1:] = xg
    K[~col, :, 0] = (kg[:, :, 0] + xg[:, :, 0]) * rng.uniform(1.1, 1.3, size=(nr, Q))
    return np.rint(K).astype(np.uint64), np.rint(X).astype(np.uint64)


def cfg4(seed: int = 4, Q: int = 16, D: int = 4):
    """cfg4: 16 queues x 4 devices (4.3e9 mappings), one epoch. K, X[:, 1:] uniform in
    {0 .. 2^24-1}."""
    rng = np.random.default_rng(seed)
    K = rng.integers(0, 1 << 24, size=(1, Q, D), dtype=np.uint64)
    X = rng.integers(0, 1 << 24, size=(1, Q, D), dtype=np.uint64)
    X[:, :, 0] = 0
    return K, X


def cfg5(seed: int = 7, Q: int = 12, D: int = 8):
    """cfg5: 12 queues x 8 devices (6.9e10 mappings), one epoch. K, X[:, 1:] uniform in
    {0 .. 2^22-1}."""
    rng = np.random.default_rng(seed)
    K = rng.integers(0, 1 << 22, size=(1, Q, D), dtype=np.uint64)
    X = rng.integers(0, 1 << 22, size=(1, Q, D), dtype=np.uint64)
    X[:, :, 0] = 0
    return K, X


def random_tables(seed: int, E: int, Q: int, D: int, hi: int = 1 << 20, x_cpu_zero: bool = True):
    """Generic uniform tables for property / parity sweeps."""
    rng = np.random.default_rng(seed)
    K = rng.integers(0, hi, size=(E, Q, D), dtype=np.uint64)
    X = rng.integers(0, hi, size=(E, Q, D), dtype=np.uint64)
    if x_cpu_zero:
        X[:, :, 0] = 0
    return K, X


def small_int_tables(seed: int, E: int, Q: int, D: int, hi: int = 8):
    """Tiny integer costs: many exact ties, exercises the lowest-index rule."""
    rng = np.random.default_rng(seed)
    K = rng.integers(0, hi, size=(E, Q, D), dtype=np.uint64)
    X = rng.integers(0, hi, size=(E, Q, D), dtype=np.uint64)
    return K, X


CONFIGS = {
    "cfg1": dict(Q=4, D=3, E=1, desc="4 queues x 3 devices (1 CPU + 2 GPU, SNU-NPB-like), 81 mappings, single epoch"),
    "cfg2": dict(Q=8, D=4, E=10_000, desc="8 queues x 4 devices (65,536 mappings), batch of 10^4 scheduling epochs"),
    "cfg3": dict(Q=2, D=3, E=1_000_000, desc="FDM-Seismology-shaped: 2 queues x 3 devices, batch of 10^6 epochs"),
    "cfg4": dict(Q=16, D=4, E=1, desc="16 queues x 4 devices (4.3e9 mappings), single epoch"),
    "cfg5": dict(Q=12, D=8, E=1, desc="12 queues x 8 devices (6.9e10 mappings), single epoch"),
}


def make(name: str, **kw):
    """Inputs of a named BASELINE config."""
    if name == "cfg1":
        return cfg1_npb(**kw)
    return {"cfg2": cfg2, "cfg3": cfg3, "cfg4": cfg4, "cfg5": cfg5}[name](**kw)


def constraints(seed: int, E: int, Q: int, D: int, pin_frac: float = 0.25, mask_frac: float = 0.25,
                base_hi: int = 1 << 20):
    """Seeded constraints for the constrained variant (NEXT-3): per-device base loads
    (queues outside the pool, SCHED_OFF) uniform in [0, base_hi), and per
    queue an eligible-device mask: a fraction pinned to one device, a fraction restricted to
    a random non-empty subset, the rest unconstrained (mask 0)."""
    rng = np.random.default_rng(seed)
    base = rng.integers(0, base_hi, size=(E, D), dtype=np.uint64)
    elig = np.zeros((E, Q), dtype=np.uint16)
    u = rng.random((E, Q))
    pins = u < pin_frac
    elig[pins] = (1 << rng.integers(0, D, size=int(pins.sum()))).astype(np.uint16)
    sub = (u >= pin_frac) & (u < pin_frac + mask_frac)
    masks = rng.integers(1, 1 << D, size=int(sub.sum())).astype(np.uint16)
    elig[sub] = masks
    return base, elig


def cost_model(seed: int, E: int, Q: int, D: int, n_kernels: int = 64, max_kernels: int = 16,
               cached_frac: float = 0.1, sockets: int = 1):
    """Seeded inputs of the cost-table construction step (NEXT-1), shaped by the paper:
    a kernel profile table whose GPU/CPU time ratios span Fig. 3's
    range (0.05x .. 4x, L1391-1401, L2058-2060); 1..max_kernels invocations per (epoch,
    queue) (a kernel epoch, L1142-1158); working sets log-uniform in 1 KiB .. 256 MiB (Fig. 6
    axis, L1854-1876) resident on the host or a GPU; bandwidth curves sampled at powers of
    two from 1 KiB to 1 GiB, latency-bound at small sizes ("from being latency bound to
    bandwidth bound", L896-898); device 0 is the CPU device working on host memory.
    With ``sockets`` > 1 the curves are per (socket, device), [S, D, M] ("all the CPU
    socket-device combinations", L897-901): socket 0 is near the GPUs and every further
    socket reaches them through an inter-socket link at 0.55-0.8 of the bandwidth and a
    longer latency (the paper's node: GPUs with affinity to one socket, L1349-1361); each
    queue's host memory is on a random socket (``host_socket`` [E, Q])."""
    rng = np.random.default_rng(seed)
    cpu = rng.integers(100_000, 10_000_000, size=n_kernels)
    profile = np.zeros((n_kernels, D), dtype=np.uint64)
    profile[:, 0] = cpu
    for d in range(1, D):
        ratio = np.exp(rng.uniform(math.log(0.05), math.log(4.0), size=n_kernels))
        profile[:, d] = np.maximum(1, np.rint(cpu * ratio)).astype(np.uint64)
    counts = rng.integers(1, max_kernels + 1, size=E * Q)
    offsets = np.zeros(E * Q + 1, dtype=np.uint64)
    offsets[1:] = np.cumsum(counts)
    kernel_ids = rng.integers(0, n_kernels, size=int(offsets[-1])).astype(np.uint32)
    nbytes = np.exp(rng.uniform(math.log(1024), math.log(256 * MIB), size=(E, Q))).astype(np.uint64)
    source = np.where(rng.random((E, Q)) < 0.5, -1, rng.integers(1, max(2, D), size=(E, Q))).astype(np.int32)
    if D == 1:
        source[:] = -1
    cached = np.where(rng.random((E, Q)) < cached_frac, rng.integers(0, 1 << D, size=(E, Q)), 0).astype(np.uint16)
    sizes = (1024 * (2 ** np.arange(21))).astype(np.uint64)
    peak_h2d = rng.uniform(5.0, 12.0, size=D)      # GB/s == bytes/ns
    peak_d2h = peak_h2d * rng.uniform(0.8, 1.0, size=D)
    half = 65536.0
    s = sizes.astype(np.float64)
    h2d = (peak_h2d[:, None] * s[None, :] / (s[None, :] + half)).astype(np.float64)
    d2h = (peak_d2h[:, None] * s[None, :] / (s[None, :] + half)).astype(np.float64)
    model = dict(profile=profile, offsets=offsets, kernel_ids=kernel_ids, bytes=nbytes, source=source,
                 cached=cached, sizes=sizes, h2d_bw=h2d, d2h_bw=d2h, host_shared=1)
    if sockets > 1:
        far = rng.uniform(0.55, 0.8, size=(sockets, D))
        far[0] = 1.0
        lat = 1.0 + 2.0 * (np.arange(sockets) > 0)  # the far sockets' longer latency ...
        model["h2d_bw"] = np.stack([far[k][:, None] * peak_h2d[:, None] * s[None, :] / (s[None, :] + half * lat[k])
                                    for k in range(sockets)]).astype(np.float64)
        model["d2h_bw"] = np.stack([far[k][:, None] * peak_d2h[:, None] * s[None, :] / (s[None, :] + half * lat[k])
                                    for k in range(sockets)]).astype(np.float64)
        model["host_socket"] = rng.integers(0, sockets, size=(E, Q)).astype(np.uint8)
    return model


def static_hints(K, X):
    """SCHED_COMPUTE_BOUND / SCHED_MEMORY_BOUND / SCHED_IO_BOUND hints (Table I, PAPER.md
    L1100-1116) a programmer would annotate the queues of a synthetic epoch with -- input
    synthesis for the SCHED_AUTO_STATIC baseline, [E, Q] uint8: I/O-bound (2) when moving the
    queue's data to a GPU costs more on average than its kernels there, else compute-bound
    (0) when some GPU runs its kernels faster than the CPU (device 0), else memory-bound (1).
    D = 1 (no GPU): every queue is compute-bound."""
    K = np.asarray(K)
    X = np.asarray(X)
    if K.shape[-1] < 2:
        return np.zeros(K.shape[:-1], np.uint8)
    gk, gx = K[..., 1:].astype(np.float64), X[..., 1:].astype(np.float64)
    io = gx.mean(-1) > gk.mean(-1)
    compute = K[..., 1:].min(-1) < K[..., 0]
    return np.where(io, 2, np.where(compute, 0, 1)).astype(np.uint8)


def static_device_scores(D: int):
    """Device-profile cost of each hint class on each device ([3, D] uint64, lower is
    better; device 0 = the CPU): compute-bound work is 4x faster on a GPU,
    memory-bound work 2x faster on the CPU (the SNU-NPB pattern of Fig. 3),
    I/O-bound queues cost nothing to keep on the host-resident CPU. Every GPU has the same
    profile (a homogeneous node), so the static policy sends all compute-bound queues to the
    first GPU -- the load imbalance the dynamic mapper avoids (L1096-1100)."""
    s = np.ones((3, D), np.uint64)
    s[0, 0], s[1, 0], s[2, 0] = 4, 1, 0
    s[1, 1:] = 2
    return s
