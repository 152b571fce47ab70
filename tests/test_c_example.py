"""The C ABI from plain C: examples/map_queues.c compiles against include/mcl.h and
libmcl.so alone (CPU test), and on a GPU returns the hand-solved optima of DESIGN.md
Appendix A cases E and F, the hand-solved constrained optimum with a pinned queue, the static
policy's mapping and makespan, and reports a 2^48 entry as MCL_E_RANGE (GPU test)."""
from __future__ import annotations

import os
import subprocess

import pytest

from conftest import cuda_available

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_cluster_ajipbf15_b200")


def build_example(tmp_path):
    from paper_conf_cluster_ajipbf15_b200 import build

    build.build()
    exe = str(tmp_path / "map_queues")
    subprocess.run(["gcc", "-O2", "-Wall", "-Werror", "-I", os.path.join(ROOT, "include"),
                    os.path.join(ROOT, "examples", "map_queues.c"), "-L", PKG, "-lmcl",
                    f"-Wl,-rpath,{PKG}", "-o", exe], check=True, capture_output=True, text=True)
    return exe


def test_c_example_compiles_against_the_abi(tmp_path):
    assert os.path.exists(build_example(tmp_path))


@pytest.mark.gpu
def test_c_example_runs(tmp_path):
    if not cuda_available():
        pytest.fail("no CUDA device: the -m gpu tests must run on a GPU box")
    r = subprocess.run([build_example(tmp_path)], capture_output=True, text=True, timeout=120)
    assert r.returncode == 0, r.stdout + r.stderr
    assert "epoch 0: index 44 makespan 200 mapping 1 1 2 2" in r.stdout
    assert "epoch 1: index 1 makespan 350 mapping 0 0 0 1" in r.stdout
    assert "pinned queue 0: MCL_OK: success index 13 makespan 2000 mapping 0 1 1 1" in r.stdout
    assert "static policy: MCL_OK: success mapping 1 1 1 1 makespan 400" in r.stdout
    assert "resident: MCL_OK: success agrees" in r.stdout
    assert "entry 2^48: MCL_E_RANGE" in r.stdout
    assert r.stdout.strip().endswith("OK")
