"""bench.py's driver contract: the reference arm (the CPU oracle, this tier's reference)
runs without a GPU and prints one JSON line with the contract's keys; the roofline
bookkeeping matches the formulas DESIGN.md SS7 states; on a GPU box the default invocation
prints the headline line with every other config under `configs`."""
from __future__ import annotations

import json
import os
import subprocess
import sys

import pytest

from conftest import ROOT, cuda_available

sys.path.insert(0, ROOT)
import bench  # noqa: E402


def _run(args, timeout=600):
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py")] + args, capture_output=True,
                         text=True, timeout=timeout, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [ln for ln in out.stdout.strip().splitlines() if ln.startswith("{")]
    assert len(lines) == 1, out.stdout
    return json.loads(lines[0])


def test_reference_arm_line_cpu():
    d = _run(["--impl", "reference", "--workload", "cfg1", "--steps", "3", "--warmup", "3",
              "--ref-step-seconds", "0.2"])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
              "scaling", "vs_baseline", "dtype", "data", "config", "cpu_baseline", "e2e"):
        assert k in d, k
    assert d["impl"] == "reference" and d["value"] > 0 and d["steps"] == 3 and d["warmup"] == 3
    assert d["config"]["workload"] == "cfg1" and d["cpu_baseline"]["kind"] == "oracle"
    assert d["e2e"] == {"value": d["value"], "unit": d["unit"], "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}


def test_roofline_bookkeeping():
    class FakeMcl:
        @staticmethod
        def mcl_probe_int_rate(dev, op):
            return (1.8e13, 64.0, 1965.0)

    w = dict(name="cfg5", E=1, Q=12, D=8, N=8**12)
    r = bench.roofline(w, {"path": "blocked_u32"}, 6.0, 148, 1965, 1, FakeMcl, 0)
    mps = 8**12 / 6e-3
    peak = 64 * 148 * 1965e6 / 1e12
    assert r["bound"] == "alu" and abs(r["peak"] - peak) < 1e-9
    assert abs(r["frac"] - 1.5 * mps / 1e12 / peak) < 1e-12
    assert abs(r["frac_survey"] - 2 * mps / 1e12 / peak) < 1e-12
    # sharded: per launch is this rank's share of the index space
    r8 = bench.roofline(w, {"path": "blocked_u32"}, 0.75, 148, 1965, 8, FakeMcl, 0)
    assert abs(r8["achieved"] - 1.5 * 8**12 / 8 / 0.75e-3 / 1e12) < 1e-9
    # batched HBM-bound kernel: algorithmic bytes per epoch = 2*Q*D*8 in + 8 + 8 + Q out
    w3 = dict(name="cfg3", E=10**6, Q=2, D=3, N=9)
    r3 = bench.roofline(w3, {"path": "small_batched"}, 0.02, 148, 1965, 1, FakeMcl, 0)
    assert r3["bound"] == "hbm" and abs(r3["achieved"] - 10**6 * 114 / 2e-5 / 1e9) < 1e-6
    w1 = dict(name="cfg1", E=1, Q=4, D=3, N=81)
    assert bench.roofline(w1, {"path": "small_batched"}, 0.006, 148, 1965, 1, FakeMcl, 0)["bound"] == "latency"


def test_replication_rules():
    assert bench.is_replicated(dict(E=10, N=65536)) and bench.is_replicated(dict(E=1, N=81))
    assert not bench.is_replicated(dict(E=1, N=8**12))


@pytest.mark.gpu
def test_default_bench_line_gpu():
    if not cuda_available():
        pytest.fail("no CUDA device")
    d = _run(["--steps", "3", "--warmup", "3", "--no-cpu-baseline"], timeout=900)
    assert d["config"]["workload"] == "cfg5" and d["value"] > 0 and d["gpu_launches"] >= 3
    assert set(d["configs"]) == {"cfg1", "cfg2", "cfg3", "cfg4"}
    for name, e in d["configs"].items():
        assert e["value"] > 0 and e["e2e"]["value"] > 0 and "roofline" in e and "clocks" in e, name
    assert d["roofline"]["bound"] == "alu" and 0 < d["roofline"]["frac"] < 1.05
    assert "frac_survey" in d["roofline"] and d["clocks"]["sm_mhz"]
    # the live launch floor: an empty kernel costs more than the events alone, and far less
    # than any search kernel the line reports
    lf = d["launch_floor"]
    assert 0 < lf["events_only_us"] < lf["empty_kernel_us"] < 50, lf
    assert lf["empty_kernel_us"] * 1e-3 < d["configs"]["cfg1"]["roofline"]["kernel_ms"] * 1.5
